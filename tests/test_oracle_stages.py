"""Pins for the oracle's lossless stages (O3-O5) and stream layout (O6-O7).

Each pin checks the oracle against something other than itself: the paper's
worked example, hand-derived known answers (tests/golden/), the
mathematical definition of base -2 numerals, numpy's packbits/unpackbits for
the bit transpose, and round-trip/size invariants.
"""
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

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


# ---------------- O3: delta + negabinary ----------------

def test_p125_worked_example(orc):
    g = _golden("p125_delta_example.txt")
    q = np.array([int(v) for v in g["input"].split()], dtype=np.uint64)
    want_d = [int(v) for v in g["residual"].split()]
    want_nb = [int(v, 2) for v in g["negabinary_binary"].split()]
    for bits in (32, 64):
        r = orc.delta_encode(q, bits)
        assert list(r[:4]) == want_nb
        # magnitude-sign (zigzag) variant of the residual, flag A1
        r_ms = orc.delta_encode(q, bits, ms=True)
        assert list(r_ms[:4]) == [2 * d if d >= 0 else -2 * d - 1 for d in want_d]


def _negabinary_value(r: int, bits: int) -> int:
    """Definition of a base -2 numeral: sum_i digit_i * (-2)^i."""
    return sum(((r >> i) & 1) * (-2) ** i for i in range(bits))


@settings(max_examples=200, deadline=None)
@given(st.lists(st.integers(0, 2**32 - 1), min_size=2, max_size=64))
def test_negabinary_is_base_minus_two_f32(orc, vals):
    q = np.array(vals, dtype=np.uint64)
    r = orc.delta_encode(q, 32)
    prev = 0
    for i, v in enumerate(vals):
        d = (v - prev) % 2**32
        # base -2 value equals the residual modulo 2^32
        assert _negabinary_value(int(r[i]), 32) % 2**32 == d
        prev = v
    assert np.array_equal(orc.delta_decode(r, 32), q)
    assert np.array_equal(orc.delta_decode(orc.delta_encode(q, 32, True), 32, True), q)


@settings(max_examples=100, deadline=None)
@given(st.lists(st.integers(0, 2**64 - 1), min_size=2, max_size=64))
def test_negabinary_is_base_minus_two_f64(orc, vals):
    q = np.array(vals, dtype=np.uint64)
    r = orc.delta_encode(q, 64)
    prev = 0
    for i, v in enumerate(vals):
        assert _negabinary_value(int(r[i]), 64) % 2**64 == (v - prev) % 2**64
        prev = v
    assert np.array_equal(orc.delta_decode(r, 64), q)


def test_small_residuals_have_leading_zeros(orc):
    """small positive and negative negabinary values both have many
    leading zero bits (the property the later stages exploit)."""
    for d in range(-8, 9):
        q = np.array([0, d % 2**32], dtype=np.uint64)
        r = int(orc.delta_encode(q, 32)[1])
        assert r < 32


# ---------------- O4: bit shuffle ----------------

def _numpy_shuffle(r: np.ndarray, bits: int) -> np.ndarray:
    """Independent transpose: numpy unpackbits/packbits, MSB plane first,
    element i -> bit (i%8) of byte i//8 within its plane (reading R13)."""
    dt = ">u4" if bits == 32 else ">u8"
    be = r.astype(dt)                                     # big-endian -> MSB first
    B = np.unpackbits(be.view(np.uint8)).reshape(len(r), bits)   # [elem, plane]
    return np.packbits(B.T.copy(), axis=1, bitorder="little").reshape(-1)


@pytest.mark.parametrize("bits,cw", [(32, 4096), (64, 2048)])
def test_shuffle_matches_numpy_transpose(orc, bits, cw):
    rng = np.random.default_rng(1)
    for scale in (2, 2**9, 2**31, None):
        if scale is None:
            r = rng.integers(0, 2**63, size=cw, dtype=np.uint64) * 2 + 1
            if bits == 32:
                r &= np.uint64(0xFFFFFFFF)
        else:
            r = rng.integers(0, scale, size=cw, dtype=np.uint64)
        S = orc.shuffle(r, bits)
        assert S.size == 16384
        assert np.array_equal(S, _numpy_shuffle(r, bits))
        assert np.array_equal(orc.unshuffle(S, cw, bits), r)


# ---------------- O5: zero / repeat elimination ----------------

def test_rze_known_answers(orc):
    g = _golden("kav_rze.txt")
    X = np.zeros(16384, np.uint8)
    X[0] = 0x5A
    assert orc.rze_encode(X) == _hex(g["kav2"])
    assert orc.rze_encode(np.zeros(16384, np.uint8)) == _hex(g["kav3"])
    rng = np.random.default_rng(2)
    X4 = rng.integers(1, 256, size=16384).astype(np.uint8)
    out = orc.rze_encode(X4)
    pre = _hex(g["kav4_prefix"])
    assert len(out) == int(g["kav4_size"])
    assert out[:len(pre)] == pre and out[len(pre):] == X4.tobytes()
    for payload, X in ((_hex(g["kav2"]), None), (_hex(g["kav3"]), np.zeros(16384, np.uint8))):
        dec, used = orc.rze_decode(payload)
        assert used == len(payload)
        if X is not None:
            assert np.array_equal(dec, X)


def _popc(b: bytes) -> int:
    return sum(bin(x).count("1") for x in b)


@pytest.mark.parametrize("density", [0.0, 0.001, 0.03, 0.3, 1.0])
def test_rze_sizes_and_roundtrip(orc, density):
    """Bitmap sizes input/8 -> 2048/256/32/4 ("the size of the bitmap is
    always the size of the input divided by 8", applied 4 times) and each
    Z section's length equals the popcount of its bitmap."""
    rng = np.random.default_rng(int(density * 1000) + 3)
    X = (rng.integers(1, 256, size=16384) * (rng.random(16384) < density)).astype(np.uint8)
    out = orc.rze_encode(X)
    nz = int(np.count_nonzero(X))
    M4 = out[:4]
    n4 = _popc(M4)
    assert len(out) >= 4 + nz
    # Z1 is exactly the non-zero bytes, in order, at the end of the payload
    assert out[len(out) - nz:] == X[X != 0].tobytes()
    dec, used = orc.rze_decode(out)
    assert used == len(out) and np.array_equal(dec, X)
    # a truncated payload must be rejected, never over-read
    if len(out) > 4:
        bad, k = orc.rze_decode(out[:-1])
        assert k < 0
    assert n4 <= 32


# ---------------- O6/O7: chunk + stream ----------------

def test_kav1_stream(orc):
    g = _golden("kav1_abs_f32.txt")
    eps = 2.0 ** int(g["eps_log2"])
    n = int(g["n"])
    x = np.full(n, -2.0 ** -9, dtype=np.float32)
    x[:4] = [0, 2.0 ** -9, 3 * 2.0 ** -9, -2.0 ** -9]
    s = orc.compress(x, "abs", eps)
    assert len(s) == int(g["stream_bytes"])
    assert s[:4] == b"PFPL" and s[4] == 1 and s[5] == 0 and s[6] == 0 and s[7] == 0
    assert int.from_bytes(s[8:16], "little") == n
    assert np.frombuffer(s[16:24], np.float64)[0] == eps
    assert s[24:32] == _hex(g["qconst"])[::-1] + b"\0" * 4
    assert int.from_bytes(s[40:44], "little") == 16384
    payload = _hex(g["payload"])
    assert int.from_bytes(s[48:52], "little") == len(payload)
    assert s[52:] == payload
    assert np.array_equal(orc.decompress(s), x)
    s4 = orc.compress(x[:4], "abs", eps)
    assert len(s4) == int(g["n4_stream_bytes"])
    assert int.from_bytes(s4[48:52], "little") == 16 and s4[52:] == x[:4].tobytes()


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_random_bits_are_stored_raw(orc, dtype):
    """incompressible chunks are emitted uncompressed, capping the
    expansion at header + size table."""
    rng = np.random.default_rng(5)
    n = 3 * (16384 // np.dtype(dtype).itemsize) + 17
    u = rng.integers(0, 2**62, size=n, dtype=np.int64).astype(np.uint64) * 3 + 12345
    x = (u.astype(np.uint32) if dtype == np.float32 else u).view(dtype)
    x = np.where(np.isfinite(x), x, 1.5).astype(dtype)
    s = orc.compress(x, "abs", 1e-30 if dtype == np.float64 else 1e-30)
    C = -(-x.nbytes // 16384)
    assert len(s) == 48 + 4 * C + x.nbytes == orc.max_compressed_bytes(n, dtype)
    sizes = np.frombuffer(s[48:48 + 4 * C], np.uint32)
    assert list(sizes[:-1]) == [16384] * (C - 1) and sizes[-1] == x.nbytes - 16384 * (C - 1)
    assert s[48 + 4 * C:] == x.tobytes()


def test_empty_input(orc):
    for dt in (np.float32, np.float64):
        s = orc.compress(np.zeros(0, dt), "abs", 1e-3)
        assert len(s) == 48
        assert orc.decompress(s).size == 0


def test_random_access_chunk_decode(orc):
    """the decoder locates chunk c by a prefix sum of the stored sizes;
    a one-chunk stream built from chunk c's table entry and payload decodes
    to the same values as that slice of the full decode."""
    import synth
    x = synth.generate(synth.CONFIGS["cesm"], slab=(0, 40)).numpy()   # 144000 values
    s = orc.compress(x, "abs", 1e-3)
    full = orc.decompress(s)
    C = -(-x.nbytes // 16384)
    sizes = np.frombuffer(s[48:48 + 4 * C], np.uint32).astype(np.int64)
    offs = 48 + 4 * C + np.concatenate([[0], np.cumsum(sizes)])
    for c in (0, 5, C - 1):
        m = min(4096, x.size - c * 4096)
        hdr = bytearray(s[:48])
        hdr[8:16] = m.to_bytes(8, "little")
        sub = bytes(hdr) + int(sizes[c]).to_bytes(4, "little") + s[offs[c]:offs[c + 1]]
        assert np.array_equal(orc.decompress(sub), full[c * 4096:c * 4096 + m])


def test_corrupt_streams_are_rejected(orc):
    import synth
    x = synth.generate(synth.CONFIGS["cesm"], slab=(0, 8)).numpy()
    s = orc.compress(x, "abs", 1e-3)
    with pytest.raises(orc.OracleError):
        orc.decompress(s[:-1])
    with pytest.raises(orc.OracleError):
        orc.decompress(b"XFPL" + s[4:])
    rng = np.random.default_rng(0)
    for _ in range(200):
        b = bytearray(s)
        i = int(rng.integers(48, len(b)))
        b[i] ^= 1 << int(rng.integers(0, 8))
        try:
            orc.decompress(bytes(b))          # must not crash or over-read
        except orc.OracleError:
            pass
