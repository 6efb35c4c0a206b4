"""World-size-2 gloo test of the multi-GPU exchange logic on CPU.

The per-shard kernels need a GPU, so the shard compressor is a CPU stand-in
built on the oracle (NOA shard = ABS with the NOA-derived bound); what is
under test is dist.py's partitioning, the NOA min/max all-reduce, the size
all-gather, the offsets and the assembly: the assembled stream must be
byte-identical to the single-device oracle stream.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _field():
    import synth
    return synth.generate(synth.CONFIGS["cesm"], slab=(0, 37)).numpy()   # 133200 f32, tail chunk


def _worker(rank, world, port, bound, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ipps_fallinadcb25_b200 import dist as pdist
        x = _field()
        eps = 1e-3
        full = oracle.compress(x, bound, eps)
        fc, nch, e0, e1 = pdist.shard_chunks(x.size, 4, rank, world)
        xl = torch.from_numpy(x[e0:e1].copy())

        def minmax_fn(t):
            a = t.numpy().astype(np.float64)
            a = a[np.isfinite(a)]
            return torch.tensor([a.min(), a.max()], dtype=torch.float64)

        def shard_fn(t, first_chunk, n_total, b, e, ms, mm):
            xs = t.numpy()
            if b == "noa":
                P = oracle.params(np.array([mm[0].item(), mm[1].item()], np.float32), "noa", e)
                s = oracle.compress(xs, "abs", float(P.eps_eff_f))
            else:
                s = oracle.compress(xs, b, e)
            C = -(-xs.size // 4096)
            tab = torch.frombuffer(bytearray(s[48:48 + 4 * C]), dtype=torch.uint8)
            pay = torch.frombuffer(bytearray(s[48 + 4 * C:]) or bytearray(1), dtype=torch.uint8)
            if len(s) == 48 + 4 * C:
                pay = pay[:0]
            return tab, pay, full[:48]

        r = pdist.compress_sharded(xl, x.size, bound, eps, minmax_fn=minmax_fn, shard_fn=shard_fn)
        parts = [None] * world
        dist.all_gather_object(parts, (r.header, r.table.numpy().tobytes(), r.payload.numpy().tobytes(),
                                       r.table_offset, r.payload_offset, r.total_bytes))
        if rank == 0:
            stream = pdist.assemble_on_host(parts)
            ok = stream == full
            offs_ok = all(stream[p[3]:p[3] + len(p[1])] == p[1] and stream[p[4]:p[4] + len(p[2])] == p[2]
                          for p in parts)
            q.put((ok, offs_ok, parts[0][5] == len(full)))
        dist.barrier()          # neither rank tears down the pair while the other still uses it
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("bound", ["abs", "noa"])
def test_two_rank_assembly_matches_single_stream(bound):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, bound, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=240)
        assert p.exitcode == 0
    ok, offs_ok, total_ok = q.get(timeout=10)
    assert ok and offs_ok and total_ok


def test_shard_plan_covers_every_chunk_once():
    from paper_conf_ipps_fallinadcb25_b200 import dist as pdist
    for n in (0, 1, 4095, 4096, 4097, 6480000):
        for world in (1, 2, 3, 8):
            spans = [pdist.shard_chunks(n, 4, r, world) for r in range(world)]
            assert spans[0][2] == 0 and spans[-1][3] == n
            for a, b in zip(spans, spans[1:]):
                assert a[3] == b[2] and a[0] + a[1] == b[0]
            assert all(s[2] % 4096 == 0 for s in spans)
