"""The exact bound checker must itself catch violations (tester's pin)."""
import numpy as np

from tests.boundcheck import violations


def test_abs_edge():
    eps = 1e-3
    x = np.array([0.0, 0.0, 1.0], np.float64)
    y = np.array([eps, np.nextafter(eps, 1), 1.0], np.float64)
    assert list(violations(x, y, "abs", eps)) == [1]
    # float32: float32(1e-3) > 1e-3 exactly, so it violates
    assert list(violations(np.zeros(1, np.float32), np.array([1e-3], np.float32), "abs", 1e-3)) == [0]


def test_rel_sign_and_factor():
    eps = 1e-3
    x = np.array([2.0, 2.0, -2.0, 2.0], np.float64)
    y = np.array([2.0 * (1 + eps), np.nextafter(2.0 * (1 + eps), 9), 2.0, 2.0 / (1 + eps)])
    bad = list(violations(x, y, "rel", eps))
    assert 1 in bad and 2 in bad and 0 not in bad


def test_nonfinite_must_be_exact():
    x = np.array([np.inf, np.nan, -np.inf], np.float32)
    y = x.copy()
    assert violations(x, y, "abs", 1e-3).size == 0
    y[0] = np.float32(3.4e38)
    assert list(violations(x, y, "abs", 1e-3)) == [0]
    xn = np.array([0xFFC00001], np.uint32).view(np.float32)
    assert violations(xn, np.array([0x7FC00001], np.uint32).view(np.float32), "rel", 1e-3).size == 0
    assert violations(xn, xn, "rel", 1e-3).size == 1


def test_noa_uses_finite_range():
    x = np.array([0.0, 10.0, np.inf], np.float64)
    y = np.array([0.01, 10.0, np.inf])
    assert violations(x, y, "noa", 1e-3).size == 0
    y[0] = np.nextafter(0.01, 1)
    assert list(violations(x, y, "noa", 1e-3)) == [0]
