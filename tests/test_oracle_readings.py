"""Pins for the oracle's readings R3 (NOA bound), R5 (REL bin scale) and R12
(tail padding), each checked against something other than the oracle itself:
exact rational arithmetic (fractions / mpmath), closed forms at powers of two,
a hand-derived known-answer stream (tests/golden/kav5_tail.txt) and a property
of the paper's REL quantizer on smooth data (few values are unquantizable).

Mutation evidence ("What's weak" #1): each of
  * REL inv_w = 1/lw instead of 0.5/lw            (R5)
  * NOA eps_abs scaled by 0.75                    (R3)
  * tail padded with 0 instead of the last word   (R12)
applied to oracle/pfpl_oracle.c makes at least one test here fail.
"""
import os
from fractions import Fraction

import mpmath
import numpy as np
import pytest

import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _golden(name):
    d = {}
    for line in open(os.path.join(GOLD, name)):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        k, v = line.split(":", 1)
        d[k.strip()] = v.strip()
    return d


def _hex(s):
    return bytes.fromhex(s.replace(" ", ""))


def _f32_bits(x) -> int:
    return int(np.array([x], np.float32).view(np.uint32)[0])


def _largest_f32_le(q: Fraction) -> np.float32:
    """Largest binary32 <= q (q > 0), by exact comparison."""
    f = np.float32(float(q))
    while Fraction(float(f)) > q:
        f = np.nextafter(f, np.float32(0))
    while Fraction(float(np.nextafter(f, np.float32(np.inf)))) <= q:
        f = np.nextafter(f, np.float32(np.inf))
    return f


def _largest_f64_le(q: Fraction) -> float:
    f = float(q)
    while Fraction(f) > q:
        f = float(np.nextafter(f, 0.0))
    while Fraction(float(np.nextafter(f, np.inf))) <= q:
        f = float(np.nextafter(f, np.inf))
    return f


# ---------------------------------------------------------------------------
# R5: REL bin scale ("multiplying by 0.5/log(eps)" is garbled; reading:
# bin = rint(log2|v| * 0.5/log2(c_lo)), reconstruction 2^(bin * 2 log2(c_lo)))
# ---------------------------------------------------------------------------

def _rel_word(bin_: int, sign: int, bits: int) -> int:
    """R10/R11 word of a REL bin: payload 1 + (zigzag(bin) << 1 | sign) in the
    negative-NaN range, sign+exponent bits inverted."""
    zz = (bin_ << 1) if bin_ >= 0 else ((-bin_) << 1) - 1
    if bits == 32:
        return (0xFF800000 | (1 + ((zz << 1) | sign))) ^ 0xFF800000
    return (0xFFF0000000000000 | (1 + ((zz << 1) | sign))) ^ 0xFFF0000000000000


@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("eps", [1e-1, 1e-2, 1e-3, 1e-4])
def test_rel_power_of_two_bins(orc, dt, eps):
    """v = +-2^k: log2|v| = k exactly, so the bin is rint(k / (2 log2 c_lo)),
    computed here in 120-bit arithmetic from c_lo = largest T <= 1 + eps (R1).
    Exponents whose exact quotient sits within 0.05 of a rounding tie are
    skipped (the float chain may legitimately round them either way).  The
    value must be quantized (not stored raw) and reconstruct within 1+eps."""
    mpmath.mp.prec = 120
    bits = 32 if dt == np.float32 else 64
    if dt == np.float32:
        c_lo = _largest_f32_le(Fraction(1) + Fraction(eps))
        ks = range(-126, 128)
    else:
        c_lo = _largest_f64_le(Fraction(1) + Fraction(eps))
        ks = range(-1022, 1024, 3)
    w_exact = 2 * mpmath.log(mpmath.mpf(float(c_lo)), 2)
    vals, want = [], []
    for k in ks:
        qv = mpmath.mpf(k) / w_exact
        fl = mpmath.floor(qv)
        if abs(qv - fl - mpmath.mpf(0.5)) < 0.05:
            continue
        b = int(mpmath.nint(qv))
        for sign in (0, 1):
            vals.append((-1.0 if sign else 1.0) * 2.0 ** k)
            want.append(_rel_word(b, sign, bits))
    x = np.array(vals, dtype=dt)
    q = orc.quantize(x, "rel", eps)
    assert [int(v) for v in q] == want
    P = orc.params(x, "rel", eps)
    y = orc.dequantize(q, P)
    ratio = np.abs(y.astype(np.float64) / x.astype(np.float64))
    # reconstruction within a factor 1+eps; generous 2 ulp slack on the check
    assert np.all(ratio <= 1 + eps * (1 + 1e-6)) and np.all(ratio >= 1 / (1 + eps * (1 + 1e-6)))


@pytest.mark.parametrize("eps", [1e-2, 1e-3, 1e-4])
def test_rel_smooth_field_is_almost_all_quantized(orc, eps):
    """on smooth scientific data only a small fraction of values is
    unquantizable.  REL on a smooth, zero-crossing Hurricane-shaped slab:
    among the normal finite values, >= 99% must be bins (R10 format), and the
    stream must compress (a wrong bin scale makes every value fail the verify
    and be stored raw while every bound test stays green)."""
    x = synth.generate(synth.CONFIGS["hurricane"], slab=(10, 12)).numpy()
    q = orc.quantize(x, "rel", eps)
    normal = (np.abs(x) >= np.finfo(np.float32).tiny) & np.isfinite(x)
    is_bin = (q >= 1) & (q <= 0x007FFFFF)
    frac_bins = float(np.mean(is_bin[normal]))
    assert frac_bins >= 0.99, frac_bins
    s = orc.compress(x, "rel", eps)
    assert len(s) < 0.5 * x.nbytes


# ---------------------------------------------------------------------------
# R3: NOA derived bound (P:92 abs = eps * (max - min)), rounded down twice in
# f64, then R1 into the data type
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("eps", [1e-1, 1e-2, 1e-3, 1e-4, 0.37])
def test_noa_bound_is_tight_and_sound(orc, dt, eps):
    """The header's q-constant is eps_eff; exactly (rationals) it must satisfy
    eps_eff <= eps * (max - min) (soundness) and be the largest value of
    the data type below that bound up to the slack of two f64 round-downs (R3):
    nextup(eps_eff) > eps * (max - min) * (1 - 2^-50).  R is the f64 range."""
    spec = synth.CONFIGS["cesm"] if dt == np.float32 else synth.CONFIGS["miranda"]
    x = synth.generate(spec, slab=(3, 5)).numpy()
    x = x.astype(dt)
    x[7] = np.inf
    x[11] = np.nan                      # R2: min/max over finite values only
    s = orc.compress(x, "noa", eps)
    f = x[np.isfinite(x)]
    mn, mx = float(f.min()), float(f.max())
    B = Fraction(eps) * (Fraction(mx) - Fraction(mn))
    qc = int.from_bytes(s[24:32], "little")
    if dt == np.float32:
        assert qc >> 32 == 0
        ee = np.array([qc], np.uint32).view(np.float32)[0]
        up = np.nextafter(ee, np.float32(np.inf))
    else:
        ee = np.array([qc], np.uint64).view(np.float64)[0]
        up = np.nextafter(ee, np.inf)
    assert Fraction(float(ee)) <= B
    assert Fraction(float(up)) > B * (1 - Fraction(1, 2 ** 50))
    assert np.frombuffer(s[32:40], np.float64)[0] == mx - mn


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_noa_equals_abs_with_exact_bound(orc, dt):
    """the NOA bound 'is then used for quantization as if it were passed
    directly to ABS'.  f32: the ABS bound is computed independently of the
    oracle (largest binary32 <= eps*(max-min), exact rationals).  f64: every
    double within ~2^-50 of the exact bound is admissible under R3's two
    round-downs, so the header's value is used after checking it lies in
    [B (1 - 2^-50), B] exactly.  The chunk bytes of NOA and of ABS with that
    bound must be identical."""
    spec = synth.CONFIGS["cesm"] if dt == np.float32 else synth.CONFIGS["miranda"]
    x = synth.generate(spec, slab=(0, 6)).numpy().astype(dt)
    eps = 1e-3
    f = x[np.isfinite(x)]
    B = Fraction(eps) * (Fraction(float(f.max())) - Fraction(float(f.min())))
    a = orc.compress(x, "noa", eps)
    if dt == np.float32:
        ee = float(_largest_f32_le(B))
        # R3's slack matters only when B is within ~2^-50 of a binary32 value
        assert Fraction(ee) < B * (1 - Fraction(1, 2 ** 48))
    else:
        ee = float(np.frombuffer(a[24:32], np.float64)[0])
        assert B * (1 - Fraction(1, 2 ** 50)) <= Fraction(ee) <= B
    b = orc.compress(x, "abs", ee)
    assert a[48:] == b[48:] and a[24:32] == b[24:32]
    assert a[6] == 2 and b[6] == 0


# ---------------------------------------------------------------------------
# R12: the tail chunk is padded with its last word
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("tag,dt", [("f32", np.float32), ("f64", np.float64)])
def test_kav5_compressed_tail_chunk(orc, tag, dt):
    g = _golden("kav5_tail.txt")
    eps = 2.0 ** int(g[f"{tag}_eps_log2"])
    n = int(g[f"{tag}_n"])
    cw = 16384 // np.dtype(dt).itemsize
    x = np.zeros(n, dt)
    x[cw:] = 2.0 ** -9
    s = orc.compress(x, "abs", eps)
    sizes = [int(v) for v in g[f"{tag}_sizes"].split()]
    assert len(s) == int(g[f"{tag}_stream_bytes"])
    assert list(np.frombuffer(s[48:48 + 4 * len(sizes)], np.uint32)) == sizes
    body = s[48 + 4 * len(sizes):]
    assert body == _hex(g[f"{tag}_payload0"]) + _hex(g[f"{tag}_payload1"])
    assert np.array_equal(orc.decompress(s), x)


# ---------------------------------------------------------------------------
# R7: REL verification against the user's bound, on values at the bin edges
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("eps", [2.0 ** -10, 2.0 ** -4, 1e-3])
def test_rel_bin_edge_values_hold_the_bound(orc, dt, eps):
    """Values within a few ulps of r_b (1+eps) and r_b / (1+eps), where r_b is
    the reconstruction of bin b: exactly the values whose acceptance depends
    on how the REL check rounds (R7).  eps = 2^-k makes 1+eps exactly
    representable, so c_lo = 1+eps and fl(a/c_lo) can round below a/(1+eps).
    Every element must satisfy |x|/(1+eps) <= |y| <= |x|(1+eps) exactly."""
    from tests.boundcheck import violations
    bits = 32 if dt == np.float32 else 64
    P = orc.params(np.ones(1, dt), "rel", eps)
    bins = np.concatenate([np.arange(-400, 400, 7), np.arange(2000, 2200, 13)])
    words = np.array([_rel_word(int(b), 0, bits) for b in bins],
                     dtype=np.uint32 if bits == 32 else np.uint64)
    r = orc.dequantize(words, P).astype(np.float64)
    r = r[np.isfinite(r) & (r > np.finfo(dt).tiny * 4) & (r < np.finfo(dt).max / 4)]
    centers = np.concatenate([(r * (1 + eps)).astype(dt), (r / (1 + eps)).astype(dt)])
    vals = [centers]
    up = down = centers
    for _ in range(12):
        up = np.nextafter(up, dt(np.inf))
        down = np.nextafter(down, dt(0))
        vals += [up, down]
    x = np.concatenate(vals).astype(dt)
    x = np.concatenate([x, -x])
    y = orc.decompress(orc.compress(x, "rel", eps))
    assert violations(x, y, "rel", eps).size == 0
    # the edges are really exercised: a good share of these values are bins
    q = orc.quantize(x, "rel", eps)
    assert np.mean((q >= 1) & (q <= (0x007FFFFF if bits == 32 else 0x000FFFFFFFFFFFFF))) > 0.3
