"""Workload for compute-sanitizer runs (memcheck / racecheck / synccheck).

    PFPL_GRID_LIMIT=8 compute-sanitizer --tool racecheck python tools/sanitize_cases.py --small
    compute-sanitizer --tool memcheck python tools/sanitize_cases.py --fuzz 200 --mb 100

--small: every (bound, dtype) encode + decode on ~200-chunk fields, a random-bits
(all raw) field and a short fuzz.  With PFPL_GRID_LIMIT=8 each persistent CTA
handles ~25 chunks, so the encoder's payload arena and IO queue and the decoder's
ring and payload queue all wrap many times (the hand-offs the tools check).
--fuzz K --mb M: K single-bit flips (M4 bitmaps, prefixes, table, payload) in an
M-MiB NYX-shaped stream; every decode must return OK or PFPL_ERR_CORRUPT.
Prints one summary line; exits non-zero on a wrong result.
"""
from __future__ import annotations

import argparse
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
import paper_conf_ipps_fallinadcb25_b200 as pk  # noqa: E402


def small() -> int:
    n_ok = 0
    for dt, tdt in (("f32", torch.float32), ("f64", torch.float64)):
        n = 200 * (16384 // (4 if dt == "f32" else 8)) + 77
        spec = synth.FieldSpec("t", (n,), dt, 5, A=2.0, tau=0.01)
        x = synth.generate(spec, device="cuda")
        for bound in ("abs", "rel", "noa"):
            s1 = pk.compress(x, bound, 1e-3).clone()
            s2 = pk.compress(x, bound, 1e-3)
            assert torch.equal(s1, s2), (dt, bound)
            y = pk.decompress(s1)
            assert y.numel() == n
            n_ok += 1
        g = torch.Generator(device="cuda").manual_seed(5)
        rb = torch.randint(-2**31, 2**31 - 1, (40 * 4096,), dtype=torch.int32, device="cuda",
                           generator=g).view(tdt)
        s = pk.compress(rb, "abs", 1e-3)
        assert torch.equal(pk.decompress(s).view(torch.int32), rb.view(torch.int32))
        n_ok += 1
    return n_ok


def fuzz(k: int, mb: int) -> tuple:
    rows = max(1, (mb << 20) // (512 * 512 * 4))
    x = synth.generate(synth.CONFIGS["nyx"], device="cuda", slab=(0, rows))
    ref = pk.compress(x, "abs", 1e-3).clone()
    y0 = pk.decompress(ref).clone()
    C = x.numel() // 4096
    table = ref[48:48 + 4 * C].cpu().numpy().view(np.uint32).astype(np.int64)
    offs = 48 + 4 * C + np.concatenate([[0], np.cumsum(table)])
    comp = np.flatnonzero(table < 16384)
    rng = np.random.default_rng(7)
    det = 0
    for i in range(k):
        kind = i % 4
        if kind == 0:
            pos = int(offs[comp[rng.integers(0, comp.size)]]) + int(rng.integers(0, 4))
        elif kind == 1:
            c = comp[rng.integers(0, comp.size)]
            pos = int(offs[c]) + 4 + int(rng.integers(0, max(1, min(64, table[c] - 4))))
        elif kind == 2:
            pos = 48 + int(rng.integers(0, 4 * C))
        else:
            pos = int(rng.integers(48 + 4 * C, ref.numel()))
        b = ref.clone()
        b[pos] ^= 1 << int(rng.integers(0, 8))
        try:
            pk.decompress(b)
        except pk.PFPLError as e:
            assert e.code == -4, (i, pos, e.code)
            det += 1
    assert torch.equal(pk.decompress(ref), y0)
    return det, k


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--small", action="store_true")
    ap.add_argument("--fuzz", type=int, default=0)
    ap.add_argument("--mb", type=int, default=100)
    a = ap.parse_args()
    pk.lib()
    out = []
    if a.small:
        out.append(f"small cases ok: {small()}")
        out.append("small fuzz detected %d/%d" % fuzz(48, 3))
    if a.fuzz:
        out.append(f"fuzz {a.mb} MiB detected %d/%d" % fuzz(a.fuzz, a.mb))
    torch.cuda.synchronize()
    print("SANITIZE_CASES OK:", "; ".join(out),
          f"grid_limit={os.environ.get('PFPL_GRID_LIMIT', 'none')}")
