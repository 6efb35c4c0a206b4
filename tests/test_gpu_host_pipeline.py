"""Host-resident (out-of-core) pipeline, pfpl_compress_host / pfpl_decompress_host
(SURVEY 8(f) NEXT-4).  The segmented H2D -> kernel -> D2H path must give the
oracle's stream byte for byte for every segment size, including
segments that end on a ragged tail and NOA's two-pass min/max, and
decode the oracle's stream to the oracle's values bit for bit."""
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


@pytest.mark.parametrize("bound", ["abs", "rel", "noa"])
@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_host_pipeline_matches_oracle(pk, orc, bound, dt):
    cw = 4096 if dt == np.float32 else 2048
    for n in (0, 1, cw - 1, 7 * cw + 123, 9 * cw):
        spec = synth.FieldSpec("t", (max(n, 1),), "f32" if dt == np.float32 else "f64", 5,
                               A=0.5, tau=0.01)
        x = synth.generate(spec).numpy()[:n].copy()
        ref = orc.compress(x, bound, 1e-3)
        y_ref = orc.decompress(ref)
        xt = torch.from_numpy(x).pin_memory()
        for seg in (1, 2, 3, 0):
            s = pk.compress_host(xt, bound, 1e-3, seg_chunks=seg)
            assert s.numpy().tobytes() == ref, (bound, dt, n, seg)
            buf = torch.frombuffer(bytearray(ref), dtype=torch.uint8)
            y = pk.decompress_host(buf, seg_chunks=seg).numpy()
            assert np.array_equal(_bits(y), _bits(y_ref)), (bound, dt, n, seg)
        assert violations(x, y, bound, 1e-3).size == 0


def test_host_pipeline_pageable_and_full_config(pk):
    """CESM-shaped field (1,583 chunks, ragged tail) from PAGEABLE host memory
    equals the device path's stream; round trip equals the device decoder."""
    spec = synth.CONFIGS["cesm"]
    x = synth.generate(spec)
    dev = pk.compress(x.cuda(), "abs", 1e-3).cpu()
    for seg in (100, 0):
        host = pk.compress_host(x.contiguous(), "abs", 1e-3, seg_chunks=seg,
                                out=torch.empty(pk.max_compressed_bytes(x.numel(), torch.float32),
                                                dtype=torch.uint8))
        assert torch.equal(host, dev)
        y = pk.decompress_host(host.clone(), seg_chunks=seg)
        assert torch.equal(y, pk.decompress(dev.cuda()).cpu())


def test_host_pipeline_errors(pk):
    x = torch.randn(50000, dtype=torch.float32)
    full = pk.compress_host(x, "abs", 1e-3)
    small = torch.empty(full.numel() - 1, dtype=torch.uint8)
    with pytest.raises(pk.PFPLError) as ei:
        pk.compress_host(x, "abs", 1e-3, out=small, seg_chunks=2)
    assert ei.value.code == -3
    bad = full.clone()
    bad[48:52] = torch.tensor([255, 255, 255, 0], dtype=torch.uint8)   # chunk 0 size 16 MiB
    with pytest.raises(pk.PFPLError) as ei:
        pk.decompress_host(bad)
    assert ei.value.code == -4


@pytest.mark.parametrize("bound", ["abs", "rel", "noa"])
@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_compress_batch_matches_oracle(pk, orc, bound, dt):
    """pfpl_compress_batch: every field's stream equals the oracle's for that
    field alone (fields of mixed sizes, an empty one, ragged tails; more fields
    than internal streams so lanes are reused)."""
    cw = 4096 if dt == np.float32 else 2048
    sizes = [3 * cw + 5, 0, 1, cw, 11 * cw + 777, 2 * cw - 1, 5]
    xs = []
    for i, n in enumerate(sizes):
        spec = synth.FieldSpec("t", (max(n, 1),), "f32" if dt == np.float32 else "f64", 20 + i,
                               A=0.5, tau=0.01)
        xs.append(synth.generate(spec).numpy()[:n].copy())
    outs = pk.compress_batch([torch.from_numpy(x).cuda() for x in xs], bound, 1e-3)
    refs = [orc.compress(x, bound, 1e-3) for x in xs]
    for x, o, r in zip(xs, outs, refs):
        assert o.cpu().numpy().tobytes() == r, (bound, dt, x.size)
    # pfpl_decompress_batch on the oracle's streams gives the oracle's values
    ys = pk.decompress_batch([torch.frombuffer(bytearray(r), dtype=torch.uint8).cuda() for r in refs])
    for x, y, r in zip(xs, ys, refs):
        assert np.array_equal(_bits(y.cpu().numpy()), _bits(orc.decompress(r))), (bound, dt, x.size)


def test_compress_batch_capacity(pk):
    xs = [torch.randn(30000, device="cuda") for _ in range(3)]
    outs = [torch.empty(pk.max_compressed_bytes(30000, torch.float32), dtype=torch.uint8, device="cuda")
            for _ in range(3)]
    outs[1] = outs[1][:1000]
    with pytest.raises(pk.PFPLError) as ei:
        pk.compress_batch(xs, "abs", 1e-3, outs=outs)
    assert ei.value.code == -3


def test_decompress_batch_corrupt(pk):
    xs = [torch.randn(30000, device="cuda") for _ in range(3)]
    outs = [o.clone() for o in pk.compress_batch(xs, "abs", 1e-3)]
    with pytest.raises(pk.PFPLError) as ei:
        pk.decompress_batch([outs[0], outs[1][:-5], outs[2]])
    assert ei.value.code == -4
    ys = pk.decompress_batch(outs)
    for x, y in zip(xs, ys):
        assert torch.equal(y, pk.decompress(pk.compress(x, "abs", 1e-3)))


def test_release_scratch_then_reuse(pk):
    """pfpl_release_scratch frees the pipeline and lane caches; the next calls
    re-create them and give the same bytes."""
    x = torch.randn(70000, dtype=torch.float32)
    a = pk.compress_host(x, "abs", 1e-3, seg_chunks=2).clone()
    b = [o.cpu() for o in pk.compress_batch([x.cuda(), x[:5000].cuda()], "noa", 1e-3)]
    assert pk.lib().pfpl_release_scratch() == 0
    assert torch.equal(pk.compress_host(x, "abs", 1e-3, seg_chunks=2), a)
    b2 = [o.cpu() for o in pk.compress_batch([x.cuda(), x[:5000].cuda()], "noa", 1e-3)]
    assert all(torch.equal(u, v) for u, v in zip(b, b2))
    assert torch.equal(pk.decompress_host(a), pk.decompress(a.cuda()).cpu())
