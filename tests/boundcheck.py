"""Exact error-bound checker (test side; independent of oracle/ and the CUDA path).

Checks the paper's definitions with tolerance 0 against the user's epsilon
as an exact rational (the double actually passed to the API):
  ABS  x - eps <= y <= x + eps
  REL  same sign, |x|/(1+eps) <= |y| <= |x|(1+eps)
  NOA  |x - y| <= eps * (max - min), finite max/min
Non-finite inputs (outside the definitions) must be reproduced bit-exactly,
except that REL makes negative NaNs positive (reading R20).
Vectorised in float64/longdouble; every element within a relative 1e-9 of
its limit is re-checked with fractions.Fraction.
"""
from __future__ import annotations

from fractions import Fraction

import numpy as np


def _uint(a):
    return a.view(np.uint32) if a.dtype == np.float32 else a.view(np.uint64)


def violations(x: np.ndarray, y: np.ndarray, bound: str, eps: float) -> np.ndarray:
    """Return indices of elements that violate the bound (empty = OK)."""
    assert x.shape == y.shape and x.dtype == y.dtype
    bad = np.zeros(x.shape, dtype=bool)
    fin = np.isfinite(x)
    # --- non-finite inputs: bit-exact (REL: NaN sign cleared) ---
    nf = ~fin
    if nf.any():
        xb, yb = _uint(x)[nf], _uint(y)[nf]
        if bound == "rel":
            signmask = np.uint32(0x7FFFFFFF) if x.dtype == np.float32 else np.uint64(0x7FFFFFFFFFFFFFFF)
            isnan = np.isnan(x[nf])
            want = np.where(isnan, xb & signmask, xb)
        else:
            want = xb
        bad[np.flatnonzero(nf)[yb != want]] = True
    if not fin.any():
        return np.flatnonzero(bad)
    xf = x[fin].astype(np.longdouble)
    yf = y[fin].astype(np.longdouble)
    idx = np.flatnonzero(fin)
    ynotfin = ~np.isfinite(y[fin])
    bad[idx[ynotfin]] = True
    E = Fraction(eps)
    if bound in ("abs", "noa"):
        if bound == "noa":
            xv = x[fin]
            xv = np.where(xv == 0, 0, xv)
            R = Fraction(float(xv.max())) - Fraction(float(xv.min()))
            limF = E * R
        else:
            limF = E
        lim = np.longdouble(float(limF))
        err = np.abs(xf - yf)
        suspicious = (err > lim * (1 - 1e-9)) | ynotfin
        for j in np.flatnonzero(suspicious):
            if not np.isfinite(y[fin][j]):
                bad[idx[j]] = True
                continue
            e = abs(Fraction(float(x[fin][j])) - Fraction(float(y[fin][j])))
            if e > limF:
                bad[idx[j]] = True
    elif bound == "rel":
        ax, ay = np.abs(xf), np.abs(yf)
        one_eps = 1 + np.longdouble(eps)
        sign_bad = (np.signbit(x[fin]) != np.signbit(y[fin])) & (x[fin] != 0)
        bad[idx[sign_bad]] = True
        lo_ok = ay * one_eps >= ax * (1 + 1e-9)
        hi_ok = ay <= ax * one_eps * (1 - 1e-9)
        suspicious = ~(lo_ok & hi_ok) & ~sign_bad
        for j in np.flatnonzero(suspicious):
            xv, yv = float(x[fin][j]), float(y[fin][j])
            if not np.isfinite(yv):
                bad[idx[j]] = True
                continue
            if xv == 0:
                if not (yv == 0):
                    bad[idx[j]] = True
                continue
            if (xv < 0) != (yv < 0) or yv == 0:
                bad[idx[j]] = True
                continue
            AX, AY = abs(Fraction(xv)), abs(Fraction(yv))
            if not (AX <= AY * (1 + E) and AY <= AX * (1 + E)):
                bad[idx[j]] = True
    else:
        raise ValueError(bound)
    return np.flatnonzero(bad)
