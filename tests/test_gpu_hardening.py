"""Round-2 GPU checks: corrupt-stream safety of the decoder at scale, the async
status word, the host-pipeline and batch argument checks, and full-size
incompressible input (every chunk raw).

Corrupt streams must come back as PFPL_ERR_CORRUPT (-4) or decode without
error (a flipped value byte is a valid stream) -- never a CUDA fault (-6),
which would mean a read outside the payload (chunk data is located by
the size-table prefix; corrupt input never reads out of bounds).
"""
import numpy as np
import pytest
import torch

import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def pk():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_fallinadcb25_b200 as pk
    return pk


def _decode_status(pk, buf) -> int:
    try:
        pk.decompress(buf)
        return 0
    except pk.PFPLError as e:
        return e.code


@pytest.mark.parametrize("rows", [128, 160])
def test_fuzz_large_stream_never_faults(pk, rows):
    """>= 200 single-bit flips in a 128 MiB NYX-shaped stream (8192 chunks, ~11 per
    decoder CTA, so every CTA's payload ring wraps): flips aimed at the M4 bitmaps,
    the Z4/Z3 prefixes, the size table and random payload bytes.  128 MiB: the decoder's
    IO warps sum the size table themselves; 160 MiB: the offsets come from
    size_scan_kernel (pfpl_internal.h kFusedScanChunks)."""
    spec = synth.CONFIGS["nyx"]
    x = synth.generate(spec, device="cuda", slab=(0, rows))
    ref = pk.compress(x, "abs", 1e-3).clone()
    y0 = pk.decompress(ref).clone()
    C = x.numel() // 4096
    table = ref[48:48 + 4 * C].cpu().numpy().view(np.uint32).astype(np.int64)
    base = 48 + 4 * C
    offs = base + np.concatenate([[0], np.cumsum(table)])
    comp = np.flatnonzero(table < 16384)
    rng = np.random.default_rng(2024)
    trials = []
    for _ in range(80):                       # M4 of a compressed chunk (late chunks too)
        c = int(comp[rng.integers(0, comp.size)])
        trials.append(("m4", int(offs[c]) + int(rng.integers(0, 4))))
    for _ in range(60):                       # Z4 / Z3 / Z2 prefix bytes
        c = int(comp[rng.integers(0, comp.size)])
        trials.append(("prefix", int(offs[c]) + 4 + int(rng.integers(0, max(1, min(64, table[c] - 4))))))
    for _ in range(40):                       # size table
        trials.append(("table", 48 + int(rng.integers(0, 4 * C))))
    for _ in range(40):                       # anywhere in the payload
        trials.append(("payload", int(rng.integers(base, ref.numel()))))
    detected = {"m4": 0, "prefix": 0, "table": 0, "payload": 0}
    for kind, pos in trials:
        b = ref.clone()
        b[pos] ^= 1 << int(rng.integers(0, 8))
        st = _decode_status(pk, b)
        assert st in (0, -4), (kind, pos, st)
        detected[kind] += st == -4
    torch.cuda.synchronize()
    assert detected["table"] == 40                      # the size sum no longer matches
    assert detected["m4"] >= 72, detected               # n4 changes the section sizes
    assert torch.equal(pk.decompress(ref), y0)          # the context is healthy


def test_async_status_word_reports_capacity(pk, orc):
    """pfpl_compress_async with a capacity that holds the header and table but not
    the payload: the status word ((int32*)result)[2] is PFPL_ERR_CAPACITY and
    result[0] still reports the size the stream needs (include/pfpl.h)."""
    x = synth.generate(synth.CONFIGS["cesm"], device="cuda", slab=(0, 32))
    need = len(orc.compress(x.cpu().numpy(), "abs", 1e-3))
    C = -(-x.numel() // 4096)
    cap = 48 + 4 * C + 64
    assert cap < need
    out = torch.zeros(cap, dtype=torch.uint8, device="cuda")
    res = torch.zeros(2, dtype=torch.int64, device="cuda")
    pk.compress_async(x, out, res, "abs", 1e-3)
    r = res.cpu().numpy()
    assert int(r[0]) == need
    assert int(np.int32(np.uint32(int(r[1]) & 0xFFFFFFFF))) == -3
    # and a sufficient capacity reports 0
    out2 = torch.zeros(need, dtype=torch.uint8, device="cuda")
    pk.compress_async(x, out2, res, "abs", 1e-3)
    r = res.cpu().numpy()
    assert int(r[0]) == need and int(r[1]) == 0


def test_decompress_host_strict_table(pk, orc):
    """pfpl_decompress_host checks the stream like pfpl_decompress: trailing bytes,
    a header-only stream with extra bytes, and table entries that exceed a chunk's
    raw size are PFPL_ERR_CORRUPT, found on the host before any device buffer is
    sized from the table."""
    x = synth.generate(synth.CONFIGS["cesm"], slab=(0, 40)).numpy()
    s = orc.compress(x, "abs", 1e-3)
    good = torch.frombuffer(bytearray(s), dtype=torch.uint8)
    want = torch.from_numpy(orc.decompress(s))
    assert torch.equal(pk.decompress_host(good), want)
    for bad in (s + b"\0",
                orc.compress(np.zeros(0, np.float32), "abs", 1e-3) + b"\0\0\0\0"):
        with pytest.raises(pk.PFPLError) as e:
            pk.decompress_host(torch.frombuffer(bytearray(bad), dtype=torch.uint8))
        assert e.value.code == -4
    C = -(-x.size // 4096)
    b = bytearray(s)
    # entry 0 -> everything (sizes sum unchanged if entry 1 absorbs the difference)
    t = np.frombuffer(bytes(b[48:48 + 4 * C]), np.uint32).copy()
    t[1] += t[0] - 2
    t[0] = 2
    b[48:48 + 4 * C] = t.tobytes()
    with pytest.raises(pk.PFPLError) as e:
        pk.decompress_host(torch.frombuffer(b, dtype=torch.uint8))
    assert e.value.code == -4
    # seg_chunks far beyond C is clamped (one segment), not an overflow
    assert torch.equal(pk.decompress_host(good, seg_chunks=2**62), want)
    y = pk.compress_host(torch.from_numpy(x), "abs", 1e-3, seg_chunks=2**62)
    assert bytes(y.numpy()) == s


def test_batch_validates_every_field_first(pk):
    """pfpl_compress_batch returns argument errors before anything is enqueued:
    with a misaligned third field, the first two outputs stay untouched."""
    xs = [synth.generate(synth.CONFIGS["cesm"], device="cuda", slab=(i, i + 8)) for i in range(3)]
    big = torch.empty(xs[2].numel() + 1, dtype=torch.float32, device="cuda")
    xs[2] = big[1:]                                     # 4-byte offset: not 16-byte aligned
    outs = [torch.full((pk.max_compressed_bytes(x.numel(), torch.float32),), 0xA5, dtype=torch.uint8,
                       device="cuda") for x in xs]
    with pytest.raises(pk.PFPLError) as e:
        pk.compress_batch(xs, "abs", 1e-3, outs=outs)
    assert e.value.code == -5
    torch.cuda.synchronize()
    for o in outs:
        assert bool((o == 0xA5).all())
    with pytest.raises(pk.PFPLError) as e:
        pk.compress_batch(xs[:2] + [xs[0]], "abs", -1.0, outs=outs)
    assert e.value.code == -2


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_full_size_incompressible_stream(pk, orc, dt):
    """256 MiB of random bits (every chunk raw; a raw slice fills most of
    the encoder's payload arena, so the arena wraps on every chunk): stream bytes
    equal the oracle's, the decode is bit-exact."""
    n = (256 << 20) // np.dtype(dt).itemsize
    g = torch.Generator(device="cuda").manual_seed(99)
    bits = torch.randint(-2**31, 2**31 - 1, (n * np.dtype(dt).itemsize // 4,), dtype=torch.int32,
                         device="cuda", generator=g)
    xd = bits.view(torch.float32 if dt == np.float32 else torch.float64)
    x = xd.cpu().numpy()
    s_gpu = pk.compress(xd, "abs", 1e-3).cpu().numpy().tobytes()
    s_cpu = orc.compress(x, "abs", 1e-3, nthreads=max(1, len(__import__("os").sched_getaffinity(0))))
    assert s_gpu == s_cpu
    C = n * np.dtype(dt).itemsize // 16384
    assert len(s_gpu) == 48 + 4 * C + x.nbytes
    y = pk.decompress(torch.frombuffer(bytearray(s_cpu), dtype=torch.uint8).cuda())
    assert torch.equal(y.view(torch.int32), bits)


@pytest.mark.parametrize("name,bound,eps", [("nyx", "abs", 1e-3), ("hurricane", "rel", 1e-3),
                                            ("miranda", "noa", 1e-4)])
def test_gpu_and_cpu_codec_interchange(pk, name, bound, eps):
    """P:43 (data compressed on one device, decompressed on another): at full size the
    GPU library and the multi-core CPU codec (NEXT-2) write the same stream, and each
    decodes the other's stream to the same values."""
    from paper_conf_ipps_fallinadcb25_b200 import cpu
    xd = synth.generate(synth.CONFIGS[name], device="cuda")
    x = xd.cpu().numpy()
    s_gpu = pk.compress(xd, bound, eps).cpu().numpy().tobytes()
    s_cpu = cpu.compress(x, bound, eps)
    assert s_gpu == s_cpu
    y_cpu = cpu.decompress(s_gpu)
    y_gpu = pk.decompress(torch.frombuffer(bytearray(s_cpu), dtype=torch.uint8).cuda()).cpu().numpy()
    assert np.array_equal(y_cpu.view(np.uint8), y_gpu.view(np.uint8))
