"""GPU <-> oracle parity through the C ABI (bit-for-bit identical
compressed and decompressed output on CPUs and GPUs).

Three checks per case: (1) GPU stream bytes == oracle stream bytes; (2) the
GPU decodes the oracle's stream to the oracle's values, bit for bit; (3)
every decoded value satisfies its bound exactly (tests/boundcheck.py).
"""
import numpy as np
import pytest
import torch

import synth
from tests.boundcheck import violations

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pk():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_fallinadcb25_b200 as pk
    return pk


def _bits(a: np.ndarray):
    return a.view(np.uint32 if a.dtype == np.float32 else np.uint64)


def _check(pk, orc, x: np.ndarray, bound: str, eps: float, ms: bool = False):
    xd = torch.from_numpy(x).cuda()
    s_gpu = pk.compress(xd, bound, eps, ms=ms).cpu().numpy().tobytes()
    s_cpu = orc.compress(x, bound, eps, ms=ms)
    if s_gpu != s_cpu:
        a, b = np.frombuffer(s_gpu, np.uint8), np.frombuffer(s_cpu, np.uint8)
        k = min(a.size, b.size)
        first = int(np.flatnonzero(a[:k] != b[:k])[0]) if np.any(a[:k] != b[:k]) else k
        raise AssertionError(f"stream mismatch ({bound}, {x.dtype}, n={x.size}): "
                             f"len gpu={len(s_gpu)} cpu={len(s_cpu)} first diff at byte {first}")
    y_cpu = orc.decompress(s_cpu)
    buf = torch.frombuffer(bytearray(s_cpu), dtype=torch.uint8).cuda()
    y_gpu = pk.decompress(buf).cpu().numpy()
    assert np.array_equal(_bits(y_gpu), _bits(y_cpu)), f"decoded values differ ({bound})"
    assert violations(x, y_gpu, bound, eps).size == 0
    return s_cpu


SIZES = [1, 31, 32, 33, 4095, 4096, 4097, 3 * 4096 + 17, 20000]


@pytest.mark.parametrize("bound", ["abs", "rel", "noa"])
@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("eps", [1e-2, 1e-3])
def test_small_fields_all_sizes(pk, orc, bound, dt, eps):
    for n in SIZES:
        spec = synth.FieldSpec("t", (n,), "f32" if dt == np.float32 else "f64", 3, A=0.5, tau=0.01)
        x = synth.generate(spec).numpy()
        _check(pk, orc, x, bound, eps)


@pytest.mark.parametrize("bound", ["abs", "rel", "noa"])
@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("eps", [1e-1, 1e-2, 1e-4, 0.37])
def test_adversarial(pk, orc, bound, dt, eps):
    x = synth.adversarial_f32() if dt == np.float32 else synth.adversarial_f64()
    _check(pk, orc, x, bound, eps)


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_random_bits_raw_and_constants(pk, orc, dt):
    rng = np.random.default_rng(7)
    n = 5 * (16384 // np.dtype(dt).itemsize) + 3
    u = rng.integers(0, 2**63, size=n, dtype=np.int64).astype(np.uint64)
    x = (u.astype(np.uint32) if dt == np.float32 else u).view(dt)
    for bound in ("abs", "rel", "noa"):
        _check(pk, orc, x, bound, 1e-3)
        _check(pk, orc, np.full(n, 2.5, dt), bound, 1e-3)
        _check(pk, orc, np.zeros(n, dt), bound, 1e-3)


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_magnitude_sign_residuals(pk, orc, dt):
    spec = synth.FieldSpec("t", (40000,), "f32" if dt == np.float32 else "f64", 5, A=1.0, tau=0.01)
    x = synth.generate(spec).numpy()
    for bound in ("abs", "rel", "noa"):
        _check(pk, orc, x, bound, 1e-3, ms=True)


def test_empty(pk, orc):
    for dt in (np.float32, np.float64):
        for bound in ("abs", "rel", "noa"):
            x = np.zeros(0, dt)
            s = pk.compress(torch.zeros(0, dtype=torch.float32 if dt == np.float32 else torch.float64,
                                        device="cuda"), bound, 1e-3)
            assert s.cpu().numpy().tobytes() == orc.compress(x, bound, 1e-3)


CONFIGS = [("cesm", "abs", 1e-3), ("hurricane", "rel", 1e-3), ("miranda", "abs", 1e-4),
           ("miranda", "rel", 1e-4), ("miranda", "noa", 1e-4), ("nyx", "abs", 1e-3),
           ("nyx", "noa", 1e-3), ("nyx_rough", "abs", 1e-3), ("cesm", "abs", 1e-2),
           ("hurricane", "rel", 1e-2), ("miranda", "noa", 1e-2)]


@pytest.mark.parametrize("name,bound,eps", CONFIGS)
def test_full_size_configs(pk, orc, name, bound, eps):
    """BASELINE.json configs at full size, in the launch configuration bench.py
    times: full stream bytes compared with the oracle (multi-threaded), GPU
    decode of the oracle stream compared bitwise, exact bound on every element."""
    spec = synth.CONFIGS[name]
    xd = synth.generate(spec, device="cuda")
    x = xd.cpu().numpy()
    s_gpu = pk.compress(xd, bound, eps).cpu().numpy().tobytes()
    s_cpu = orc.compress(x, bound, eps, nthreads=max(1, len(__import__("os").sched_getaffinity(0))))
    assert len(s_gpu) == len(s_cpu) and s_gpu == s_cpu
    y = pk.decompress(torch.frombuffer(bytearray(s_cpu), dtype=torch.uint8).cuda()).cpu().numpy()
    y_cpu = orc.decompress(s_cpu, nthreads=8)
    assert np.array_equal(_bits(y), _bits(y_cpu))
    assert violations(x, y, bound, eps).size == 0


def test_capacity_and_corruption(pk, orc):
    x = synth.generate(synth.CONFIGS["cesm"], device="cuda", slab=(0, 16))
    full = pk.compress(x, "abs", 1e-3)
    out = torch.empty(full.numel() - 1, dtype=torch.uint8, device="cuda")
    with pytest.raises(pk.PFPLError) as e:
        pk.compress(x, "abs", 1e-3, out=out)
    assert e.value.code == -3
    with pytest.raises(pk.PFPLError):
        pk.compress(x, "abs", 1e-40)
    with pytest.raises(pk.PFPLError):
        pk.decompress(full[:-1].clone())
    rng = np.random.default_rng(1)
    for _ in range(100):
        b = full.clone()
        i = int(rng.integers(48, b.numel()))
        b[i] ^= 1 << int(rng.integers(0, 8))
        try:
            pk.decompress(b)
        except pk.PFPLError:
            pass
    torch.cuda.synchronize()


def test_async_api(pk, orc):
    x = synth.generate(synth.CONFIGS["cesm"], device="cuda", slab=(0, 32))
    out = torch.empty(pk.max_compressed_bytes(x.numel(), torch.float32), dtype=torch.uint8,
                      device="cuda")
    res = torch.zeros(2, dtype=torch.int64, device="cuda")
    pk.compress_async(x, out, res, "abs", 1e-3)
    nb = int(res[0].item())
    assert out[:nb].cpu().numpy().tobytes() == orc.compress(x.cpu().numpy(), "abs", 1e-3)
    y = torch.empty_like(x)
    pk.decompress_async(out[:nb], out[:48].cpu().numpy().tobytes(), y, res)
    assert int(res[1].item()) == 0
    assert torch.equal(y, pk.decompress(out[:nb]))


@pytest.mark.parametrize("bound", ["abs", "noa"])
def test_shards_assemble_to_single_stream(pk, orc, bound):
    """chunk-aligned shards + gathered sizes give a stream
    byte-identical to the single-device one (P:141 chunks are independent)."""
    spec = synth.CONFIGS["cesm"]
    xd = synth.generate(spec, device="cuda")
    single = pk.compress(xd, bound, 1e-3).cpu().numpy().tobytes()
    for world in (2, 3):
        mm = pk.minmax(xd) if bound == "noa" else None
        parts, tables, hdr = [], [], None
        for r in range(world):
            e0, e1 = synth.chunk_slab(spec, r, world)
            tab, pay, h = pk.compress_shard(xd[e0:e1].contiguous(), e0 // 4096, xd.numel(), bound,
                                            1e-3, mnmx=mm)
            tables.append(tab.cpu().numpy().tobytes())
            parts.append(pay.cpu().numpy().tobytes())
            hdr = hdr or h
            assert h == hdr
        assert hdr + b"".join(tables) + b"".join(parts) == single


@pytest.mark.parametrize("name,bound,eps", [("miranda", "abs", 1e-4), ("nyx_rough", "abs", 1e-3),
                                            ("hurricane", "rel", 1e-3)])
def test_repeat_determinism(pk, name, bound, eps):
    """Back-to-back async calls must reproduce the same stream and decode exactly:
    guards the encoder's arena / IO-queue hand-off and the look-back (a missing
    release of the Z2 bytes once showed up here as ~5% of runs differing)."""
    x = synth.generate(synth.CONFIGS[name], device="cuda")
    ref = pk.compress(x, bound, eps).clone()
    hdr = ref[:48].cpu().numpy().tobytes()
    out = torch.empty(pk.max_compressed_bytes(x.numel(), x.dtype), dtype=torch.uint8, device="cuda")
    rc = torch.zeros(4, dtype=torch.int64, device="cuda")
    rd = torch.zeros(4, dtype=torch.int64, device="cuda")
    y0 = pk.decompress(ref).clone()
    y = torch.empty_like(x)
    for i in range(40):
        if i % 10 == 0:
            out.fill_(0xA5)
        pk.compress_async(x, out, rc, bound, eps)
        pk.decompress_async(ref, hdr, y, rd)
        torch.cuda.synchronize()
        n = int(rc[0])
        assert n == ref.numel() and torch.equal(out[:n], ref), f"rep {i}: stream differs"
        assert int(rd[1]) == 0 and torch.equal(y, y0), f"rep {i}: decode differs"


# ---- encoder statistics (pfpl_last_stats): unquantizable values, raw chunks
def _oracle_unquantizable(orc, x: np.ndarray, bound: str, eps: float) -> int:
    """Values the oracle's quantizer (O1) stores losslessly: words outside the bin
    range of the stream format (R8 ABS/NOA zigzag bins below the normal range, R10 REL
    bins 1 + payload), or every value in raw-words mode (R4)."""
    P = orc.params(x, bound, eps)
    if P.flags & 1:
        return x.size
    w = orc.quantize(x, bound, eps, P).astype(np.uint64)
    lim = np.uint64(2**23 if x.dtype == np.float32 else 2**52)
    if bound == "rel":
        return int(np.count_nonzero(~((w >= 1) & (w < lim))))
    return int(np.count_nonzero(w >= lim))


def _raw_chunks(stream: bytes, x: np.ndarray) -> int:
    cw = 16384 // x.itemsize
    C = -(-x.size // cw)
    sizes = np.frombuffer(stream[48:48 + 4 * C], np.uint32)
    raw = [(min(cw, x.size - c * cw) * x.itemsize) for c in range(C)]
    return int(np.count_nonzero(sizes == np.array(raw, np.uint32)))


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_stats_match_oracle(pk, orc, dt):
    rng = np.random.default_rng(11)
    adv = synth.adversarial_f32() if dt == np.float32 else synth.adversarial_f64()
    n = 3 * (16384 // np.dtype(dt).itemsize) + 5
    u = rng.integers(0, 2**63, size=n, dtype=np.int64).astype(np.uint64)
    rnd = (u.astype(np.uint32) if dt == np.float32 else u).view(dt)
    spec = synth.FieldSpec("t", (20000,), "f32" if dt == np.float32 else "f64", 3, A=0.5, tau=0.01)
    fld = synth.generate(spec).numpy()
    fld[::97] = np.inf                      # a sprinkle of unquantizable values in a smooth field
    cases = [(adv, b, e) for b in ("abs", "rel", "noa") for e in (1e-1, 1e-4)]
    cases += [(rnd, b, 1e-3) for b in ("abs", "rel", "noa")]
    cases += [(fld, b, 1e-3) for b in ("abs", "rel", "noa")]
    cases += [(np.zeros(0, dt), "abs", 1e-3)]
    for x, bound, eps in cases:
        s = pk.compress(torch.from_numpy(x).cuda(), bound, eps).cpu().numpy().tobytes()
        st = pk.last_stats()
        want_u = _oracle_unquantizable(orc, x, bound, eps)
        assert st["unquantizable"] == want_u, (bound, eps, x.size, st, want_u)
        assert st["raw_chunks"] == _raw_chunks(s, x), (bound, eps, x.size, st)


# ---- verify mode (pfpl_decompress_verify)
def _metrics_ref(x: np.ndarray, y: np.ndarray, bound: str, eps: float, rng_noa: float):
    xd, yd = x.astype(np.float64), y.astype(np.float64)
    fin = np.isfinite(xd)
    d = np.abs(xd[fin] - yd[fin])
    nz = xd[fin] != 0
    lim = {"abs": np.full(d.shape, eps), "rel": eps * np.abs(xd[fin]),
           "noa": np.full(d.shape, eps * rng_noa)}[bound]
    nonfin_bad = ~fin & ~((np.isnan(xd) & np.isnan(yd)) | (xd == yd))
    return dict(n_finite=int(fin.sum()), max_abs_err=float(d.max()) if d.size else 0.0,
                max_rel_err=float((d[nz] / np.abs(xd[fin][nz])).max()) if nz.any() else 0.0,
                sum_sq_err=float((d * d).sum()), violations=int((~(d <= lim)).sum() + nonfin_bad.sum()),
                value_min=float(xd[fin].min()) if fin.any() else 0.0,
                value_max=float(xd[fin].max()) if fin.any() else 0.0)


@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("bound", ["abs", "rel", "noa"])
def test_decompress_verify_metrics(pk, orc, dt, bound):
    """Metrics from the decode epilogue equal numpy's on the oracle-decoded values (max
    and counts exactly, the f64 sum up to summation order); zero violations; a perturbed
    original is caught value by value."""
    spec = synth.FieldSpec("t", (3 * 4096 + 1000,), "f32" if dt == np.float32 else "f64", 5, A=0.5, tau=0.01)
    cases = [synth.generate(spec).numpy(),
             synth.adversarial_f32() if dt == np.float32 else synth.adversarial_f64()]
    rng = np.random.default_rng(3)
    u = rng.integers(0, 2**63, size=2 * (16384 // np.dtype(dt).itemsize) + 7, dtype=np.int64).astype(np.uint64)
    cases.append((u.astype(np.uint32) if dt == np.float32 else u).view(dt))     # raw chunks
    for ci, x in enumerate(cases):
        eps = 1e-3
        s = orc.compress(x, bound, eps)
        P = orc.params(x, bound, eps)
        y_ref = orc.decompress(s)
        buf = torch.frombuffer(bytearray(s), dtype=torch.uint8).cuda()
        xg = torch.from_numpy(x).cuda()
        y, m = pk.decompress_verify(buf, xg)
        assert np.array_equal(_bits(y.cpu().numpy()), _bits(y_ref))
        ref = _metrics_ref(x, y_ref, bound, eps, P.range)
        assert m["n"] == x.size and m["n_finite"] == ref["n_finite"]
        assert m["violations"] == 0 == ref["violations"]
        assert m["max_abs_err"] == ref["max_abs_err"] and m["max_rel_err"] == ref["max_rel_err"]
        assert m["value_min"] == ref["value_min"] and m["value_max"] == ref["value_max"]
        assert m["sum_sq_err"] == pytest.approx(ref["sum_sq_err"], rel=1e-12, abs=1e-300)
        # a corrupted original: every changed finite value is outside the bound
        x2 = x.copy()
        idx = np.flatnonzero(np.isfinite(x2))[::501][:7]
        x2[idx] = x2[idx] * 3 + 10
        _, m2 = pk.decompress_verify(buf, torch.from_numpy(x2).cuda())
        ref2 = _metrics_ref(x2, y_ref, bound, eps, P.range)
        assert m2["violations"] == ref2["violations"]
        if ci == 0:
            assert m2["violations"] == len(idx)


def test_full_size_16gib(pk, orc):
    """BASELINE.json configs[4] (16 GiB f32, n = 2^32, ABS 1E-3) at full size on one GPU, in
    bench's launch configuration: the size table must account for the whole stream, the whole
    stream must equal the oracle's (when the host has ~64 GiB free) and decode to the oracle's
    values, and sampled chunks (first, last, 62 random) must be byte-identical to the oracle's encoding of
    the same 4096 values (ABS constants depend only on eps, so a lone chunk's payload is the
    chunk's payload in any stream) and decode to the oracle's values bit for bit."""
    free, _ = torch.cuda.mem_get_info()
    if free < 60 * 2**30:
        pytest.skip("needs ~60 GiB of free device memory")
    spec = synth.CONFIGS["big16g"]
    x = synth.generate(spec, device="cuda")
    n = x.numel()
    assert n == 2**32
    s = pk.compress(x, "abs", 1e-3)
    C = n // 4096
    table = s[48:48 + 4 * C].cpu().numpy().view(np.uint32).astype(np.int64)
    offs = np.concatenate([[0], np.cumsum(table)])
    base = 48 + 4 * C
    assert base + int(offs[-1]) == s.numel()
    y = pk.decompress(s)
    # the whole stream against the oracle on all host cores (~25 s of CPU work), when the
    # host has room for the field, both decodes and the stream (~50 GiB)
    import os
    host_free = os.sysconf("SC_AVPHYS_PAGES") * os.sysconf("SC_PAGE_SIZE")
    if host_free >= 64 * 2**30:
        nt = max(1, len(os.sched_getaffinity(0)))
        xh = x.cpu().numpy()
        s_orc = orc.compress(xh, "abs", 1e-3, nthreads=nt)
        assert s.cpu().numpy().tobytes() == s_orc          # all 1,048,576 chunks
        y_orc = orc.decompress(s_orc, nthreads=nt)
        assert np.array_equal(y.cpu().numpy().view(np.uint32), y_orc.view(np.uint32))
        del xh, s_orc, y_orc
    rng = np.random.default_rng(4)
    for c in [0, C - 1] + list(rng.integers(1, C - 1, size=62)):
        c = int(c)
        xc = x[c * 4096:(c + 1) * 4096].cpu().numpy()
        ref = orc.compress(xc, "abs", 1e-3)
        assert int(table[c]) == len(ref) - 52, c
        got = s[base + int(offs[c]):base + int(offs[c + 1])].cpu().numpy().tobytes()
        assert got == ref[52:], c
        yc = y[c * 4096:(c + 1) * 4096].cpu().numpy()
        assert np.array_equal(yc.view(np.uint32), orc.decompress(ref).view(np.uint32)), c
    del x, y, s
    torch.cuda.empty_cache()


def _rel_edge_values(orc, dt, eps):
    """Values within 12 ulps of r_b (1+eps) and r_b / (1+eps) for many bins b (the REL
    bins' edges, where the exact check decides; R7), plus the largest/smallest
    exponents (pow2p's clamps) -- the inputs that probe the encoder's REL fast path."""
    bits = 32 if dt == np.float32 else 64
    P = orc.params(np.ones(1, dt), "rel", eps)
    bins = np.concatenate([np.arange(-400, 400, 7), np.arange(2000, 2200, 13),
                           np.arange(30000, 44000, 997)])
    zz = np.where(bins >= 0, 2 * bins, -2 * bins - 1).astype(np.int64)
    mask = 0xFF800000 if bits == 32 else 0xFFF0000000000000
    words = [((mask | (1 + (int(z) << 1))) ^ mask) for z in zz if (1 + (int(z) << 1)) < (1 << (22 if bits == 32 else 51))]
    r = orc.dequantize(np.array(words, dtype=np.uint32 if bits == 32 else np.uint64), P).astype(np.float64)
    r = r[np.isfinite(r) & (r > 0)]
    with np.errstate(over="ignore"):
        centers = np.concatenate([(r * (1 + eps)).astype(dt), (r / (1 + eps)).astype(dt)])
    centers = centers[np.isfinite(centers) & (centers > 0)]
    vals = [centers]
    up = down = centers
    for _ in range(12):
        up = np.nextafter(up, dt(np.inf))
        down = np.nextafter(down, dt(0))
        vals += [up, down]
    fi = np.finfo(dt)
    extremes = np.array([fi.max, fi.max / 1.5, fi.tiny, fi.tiny * 1.5, fi.tiny * 3, 2.0 ** (fi.maxexp - 2)], dt)
    x = np.concatenate(vals + [extremes]).astype(dt)
    x = np.concatenate([x, -x])
    return x[np.isfinite(x)]


@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("eps", [2.0 ** -10, 1e-1, 1e-2, 1e-3, 1e-4, 1e-6])
def test_rel_bin_edges_and_extremes(pk, orc, dt, eps):
    """REL parity where the encoder's fast path must defer to the exact quantizer: bin
    edges (|s - k| close to 1/2) and the exponent extremes (pow2p's inf/0 clamps)."""
    x = _rel_edge_values(orc, dt, eps)
    cw = 16384 // np.dtype(dt).itemsize
    x = np.resize(x, ((x.size + cw - 1) // cw) * cw)     # full chunks: the fast-path layout
    _check(pk, orc, x, "rel", eps)


def _tier_mix(dt, bound: str, eps: float, seed: int = 11) -> np.ndarray:
    """Blocks of 1024 values (one encoder warp's share of a chunk, f32 and f64) whose
    bin-domain residuals are ~2^k, with k cycling so that neighbouring warps of a chunk
    sit in different transpose tiers (P <= 8, 16, 32 and, for f64, the high-half tiers)
    and the largest k overflow into unquantizable (raw) words."""
    rng = np.random.default_rng(seed)
    ks = [0, 3, 5, 6, 9, 12, 14, 17, 20, 23, 26, 30] if dt == np.float32 else \
         [0, 5, 9, 14, 20, 26, 30, 33, 36, 39, 44, 47, 52, 60]
    order = np.concatenate([rng.permutation(len(ks)) for _ in range(8 if dt == np.float32 else 10)])
    out = []
    for j in order:
        r = float(2.0 ** ks[j])
        u = rng.uniform(-r, r, 1024) + np.arange(1024) * 0.25
        if bound == "rel":
            step = 2.0 * np.log2(1.0 + eps)
            with np.errstate(over="ignore"):
                v = np.exp2(np.clip(step * u, -2000.0, 2000.0)) * rng.choice([-1.0, 1.0], 1024)
        else:
            v = 2.0 * eps * u
        out.append(v)
    with np.errstate(over="ignore"):
        return np.concatenate(out).astype(dt)


@pytest.mark.parametrize("bound", ["abs", "rel", "noa"])
@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_every_plane_tier_per_warp(pk, orc, bound, dt):
    """The three level-1 code shapes (one copy per tier for f32 ABS, the
    windowed path for f32 NOA and f64 ABS/NOA, the staged path for REL) on chunks whose
    warps run different tiers, plus a ragged tail: same bytes as the oracle."""
    eps = 1e-2 if bound == "rel" else 1e-3
    x = _tier_mix(dt, bound, eps)
    _check(pk, orc, x, bound, eps)
    _check(pk, orc, x[: x.size - 777], bound, eps)


@pytest.mark.gpu
@pytest.mark.parametrize("bound", ["abs", "noa"])
@pytest.mark.parametrize("ms", [False, True])
def test_f32_abs_both_encoder_forms(pk, orc, ms, bound):
    """The f32 ABS encoder's two forms (the first residual of a chunk, taken
    against q[-1] = 0, split into single-byte extra planes, or not) write the
    oracle's bytes.  A large-magnitude smooth field leaves the hint for the split form, a
    small-magnitude one for the plain form, so this sequence runs both."""
    n = 4096 * 300 + 77
    xb = synth.generate(synth.FieldSpec("t", (n,), "f32", 11, A=0.4, tau=0.001)).numpy()
    xs = synth.generate(synth.FieldSpec("t", (n,), "f32", 12, A=0.02, tau=0.001)).numpy()
    if bound == "noa":
        # NOA bins are relative to the range: a large relative bound keeps them small
        eb, es = 1e-4, 1e-1
    else:
        eb, es = 1e-3, 1e-3
    forms = []
    for x, e in ((xb, eb), (xb, eb), (xs, es), (xs, es), (xb, eb), (xb, eb)):
        forms.append(pk.f32_encoder_form(bound))
        _check(pk, orc, x, bound, e, ms=ms)
    assert forms[1] == 1 and forms[3] == 0 and forms[5] == 1, forms
    # the decoder follows the same hint (pfpl_decompress): with it at 1, decode the oracle's
    # stream of the small-magnitude field (no foldable planes) and of the large one
    assert pk.f32_encoder_form(bound) == 1
    for x, e in ((xs, es), (xb, eb)):
        s_cpu = orc.compress(x, bound, e, ms=ms)
        y = pk.decompress(torch.frombuffer(bytearray(s_cpu), dtype=torch.uint8).cuda()).cpu().numpy()
        assert np.array_equal(_bits(y), _bits(orc.decompress(s_cpu)))

