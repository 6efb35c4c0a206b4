"""Run the hot path a few times for ncu / nsight captures (not a benchmark)."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_fallinadcb25_b200 as pk
import synth

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="nyx")
ap.add_argument("--bound", default="abs")
ap.add_argument("--eps", type=float, default=1e-3)
ap.add_argument("--iters", type=int, default=3)
ap.add_argument("--what", default="both")
a = ap.parse_args()
x = synth.generate(synth.CONFIGS[a.config], device="cuda")
torch.cuda.synchronize()
for _ in range(a.iters):
    s = pk.compress(x, a.bound, a.eps)
    if a.what in ("both", "decode"):
        y = pk.decompress(s)
torch.cuda.synchronize()
print("ok", s.numel(), x.numel() * x.element_size() / s.numel())
