"""Pins for the oracle's quantizers (O0/O1) and the whole pipeline's bound.

The error bounds are checked exactly (tests/boundcheck.py, tolerance 0,
against the user's double epsilon as a rational) on every element; special
cases reduce to closed forms (P:88 bins, P:102 denormals, P:104 NaN sign).
"""
import math

import numpy as np
import pytest

import synth
from tests.boundcheck import violations


# ---------------- closed forms ----------------

def test_abs_power_of_two_bins_exact(orc):
    """eps = 2^-k, v = j*2^(1-k): bin j, exact reconstruction (values are
    reconstructed to the bin center; bin width 2 eps)."""
    for k in (3, 10, 20):
        j = np.arange(-3000, 3001)
        for dt, bits in ((np.float32, 32), (np.float64, 64)):
            v = (j * 2.0 ** (1 - k)).astype(dt)
            q = orc.quantize(v, "abs", 2.0 ** -k)
            want = np.where(j >= 0, 2 * j, -2 * j - 1).astype(q.dtype)   # zigzag(j), R8
            assert np.array_equal(q, want)
            P = orc.params(v, "abs", 2.0 ** -k)
            assert np.array_equal(orc.dequantize(q, P), v)


def test_abs_denormals_and_zero_map_to_bin0(orc):
    """the ABS bound is at least the smallest normal, so denormals are
    always quantized to zero; -0 decodes as +0."""
    den = np.array([0x00000001, 0x807FFFFF, 0x80000000, 0x00000000], np.uint32).view(np.float32)
    q = orc.quantize(den, "abs", float(np.finfo(np.float32).tiny))
    assert np.all(q == 0)
    P = orc.params(den, "abs", 1e-3)
    y = orc.dequantize(orc.quantize(den, "abs", 1e-3), P)
    assert np.all(y.view(np.uint32) == 0)


def test_abs_bound_below_min_normal_is_rejected(orc):
    with pytest.raises(orc.OracleError) as e:
        orc.params(np.ones(4, np.float32), "abs", 1e-39)
    assert e.value.code == orc.ERR_BOUND
    for bad in (0.0, -1.0, math.nan, math.inf):
        with pytest.raises(orc.OracleError):
            orc.params(np.ones(4, np.float32), "abs", bad)


def test_eps_rounds_down_into_float32(orc):
    """Reading R1: eps_eff is the largest binary32 <= eps (round-to-nearest
    would give float32(1e-3) > 1e-3 and admit exact violations)."""
    P = orc.params(np.ones(1, np.float32), "abs", 1e-3)
    assert float(P.eps_eff_f) <= 1e-3
    assert float(np.nextafter(np.float32(P.eps_eff_f), np.float32(1))) > 1e-3
    P = orc.params(np.ones(1, np.float32), "rel", 1e-3)
    assert float(P.c_lo_f) - 1.0 <= 1e-3 < float(np.nextafter(np.float32(P.c_lo_f), np.float32(2))) - 1.0


def test_rel_unit_values_are_bin0(orc):
    """REL: log2(1) = 0 -> bin 0 -> reconstruction pow2(0) = 1 exactly;
    the word is payload 1 + (0<<1 | sign) in the negative-NaN range with the
    sign+exponent bits inverted (R10, R11)."""
    v = np.array([1.0, -1.0], np.float32)
    q = orc.quantize(v, "rel", 1e-3)
    assert list(q) == [(0xFF800000 | 1) ^ 0xFF800000, (0xFF800000 | 2) ^ 0xFF800000]
    P = orc.params(v, "rel", 1e-3)
    assert np.array_equal(orc.dequantize(q, P), v)


def test_rel_specials(orc):
    """zeros, denormals, inf are lossless; negative NaNs become positive."""
    bits = np.array([0x00000000, 0x80000000, 0x00000001, 0x807FFFFF, 0x7F800000,
                     0xFF800000, 0x7FC00001, 0xFFC00001, 0xFF800001], np.uint32)
    v = bits.view(np.float32)
    P = orc.params(v, "rel", 1e-3)
    y = orc.dequantize(orc.quantize(v, "rel", 1e-3, P), P).view(np.uint32)
    assert list(y) == [0x00000000, 0x80000000, 0x00000001, 0x807FFFFF, 0x7F800000,
                       0xFF800000, 0x7FC00001, 0x7FC00001, 0x7F800001]


def test_noa_minmax_over_finite(orc):
    """P:92 min/max; reading R2: over finite values only."""
    x = synth.adversarial_f32()
    P = orc.params(x, "noa", 1e-3)
    f = x[np.isfinite(x)].astype(np.float64)
    assert P.range == f.max() - f.min()


def test_noa_equals_abs_with_derived_bound(orc):
    """NOA 'is then used for quantization as if it were passed directly
    to ABS' -> identical chunk bytes (only header fields differ)."""
    x = synth.generate(synth.CONFIGS["cesm"], slab=(0, 20)).numpy()
    P = orc.params(x, "noa", 1e-3)
    a = orc.compress(x, "noa", 1e-3)
    b = orc.compress(x, "abs", float(P.eps_eff_f))
    assert a[48:] == b[48:] and a[24:32] == b[24:32]
    assert np.frombuffer(a[32:40], np.float64)[0] == P.range


def test_noa_constant_input_is_raw_words(orc):
    x = np.full(5000, 3.25, np.float32)
    s = orc.compress(x, "noa", 1e-3)
    assert s[7] & orc.FLAG_RAWWORDS
    assert np.array_equal(orc.decompress(s), x)


# ---------------- portable log2 / pow2 ----------------

def test_log2p_pow2p_exact_at_powers_of_two(orc):
    for k in range(-126, 128):
        assert orc.log2p_f32(2.0 ** k) == k
        assert orc.pow2p_f32(float(k)) == 2.0 ** k
    for k in range(-1022, 1024, 7):
        assert orc.log2p_f64(2.0 ** k) == k
        assert orc.pow2p_f64(float(k)) == 2.0 ** k


def test_log2p_pow2p_accuracy(orc):
    """Accuracy pins for the atanh/Taylor approximations (quality, not bytes):
    a wrong coefficient or a dropped term exceeds these bounds."""
    import mpmath
    mpmath.mp.prec = 120
    rng = np.random.default_rng(4)
    a32 = np.exp(rng.uniform(-80, 80, 2000)).astype(np.float32)
    for a in a32:
        ex = float(mpmath.log(mpmath.mpf(float(a)), 2))
        assert abs(orc.log2p_f32(float(a)) - ex) <= 4e-7 * max(1.0, abs(ex))
    for y in rng.uniform(-120, 120, 2000).astype(np.float32):
        ex = mpmath.power(2, mpmath.mpf(float(y)))
        assert abs(orc.pow2p_f32(float(y)) / float(ex) - 1) <= 1e-6
    for a in np.exp(rng.uniform(-600, 600, 2000)):
        ex = float(mpmath.log(mpmath.mpf(float(a)), 2))
        assert abs(orc.log2p_f64(float(a)) - ex) <= 1e-15 * max(1.0, abs(ex))
    for y in rng.uniform(-1000, 1000, 2000):
        ex = mpmath.power(2, mpmath.mpf(float(y)))
        assert abs(orc.pow2p_f64(float(y)) / float(ex) - 1) <= 2e-15


# ---------------- whole-pipeline bound, brute force ----------------

CASES = [(b, dt) for b in ("abs", "rel", "noa") for dt in (np.float32, np.float64)]


def _field(dt, n, seed):
    spec = synth.FieldSpec("t", (n,), "f32" if dt == np.float32 else "f64", seed, A=3.0, tau=0.01)
    return synth.generate(spec).numpy()


@pytest.mark.parametrize("bound,dt", CASES)
@pytest.mark.parametrize("eps", [1e-1, 1e-3, 1e-4, 0.37])
def test_bound_holds_on_every_element(orc, bound, dt, eps):
    x = np.concatenate([_field(dt, 9000, 11),
                        synth.adversarial_f32() if dt == np.float32 else synth.adversarial_f64()])
    # values sitting exactly on / next to bin edges (P:29 rounding issue)
    e2 = 2 * eps
    edges = (np.arange(-50, 50) * e2 + eps).astype(dt)
    near = np.concatenate([np.nextafter(edges, dt(np.inf)), edges, np.nextafter(edges, dt(-np.inf))])
    x = np.concatenate([x, near]).astype(dt)
    s = orc.compress(x, bound, eps)
    y = orc.decompress(s)
    assert y.dtype == x.dtype and y.size == x.size
    assert violations(x, y, bound, eps).size == 0
    # determinism: compressing again gives the same bytes
    assert orc.compress(x, bound, eps) == s


@pytest.mark.parametrize("bound,dt", CASES)
def test_huge_ranges_do_not_overflow(orc, bound, dt):
    """cuSZp's pre-quantization can overflow on huge values; here huge
    values (up to T_MAX) must be stored losslessly, never wrapped."""
    fi = np.finfo(dt)
    x = np.array([fi.max, -fi.max, fi.max / 3, 1e-3, -7.5, fi.tiny, 1.0], dtype=dt)
    x = np.tile(x, 700)
    y = orc.decompress(orc.compress(x, bound, 1e-3))
    assert violations(x, y, bound, 1e-3).size == 0


def test_unquantizable_fraction_reported(orc):
    """P:98 reports 0.7% average at ABS 1E-3 on real data; on the synthetic
    fields it is far lower (reported, parity unpinned)."""
    x = synth.generate(synth.CONFIGS["nyx"], slab=(100, 102)).numpy()
    q = orc.quantize(x, "abs", 1e-3)
    frac = float(np.mean(q >= (1 << 23)))
    assert frac < 0.007
