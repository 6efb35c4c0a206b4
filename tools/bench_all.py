"""Compress/decompress GB/s, ratio and roofline fraction for every BASELINE.json
config on one GPU (CUDA events, median of K runs after W warm-ups; inputs in
HBM).  Prints a markdown table and writes gpurun_out/bench_all.json."""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_fallinadcb25_b200 as pk
import synth

PEAK = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6650.0
CASES = [("cesm", "abs", 1e-3), ("nyx", "abs", 1e-3), ("nyx", "noa", 1e-3), ("nyx_rough", "abs", 1e-3),
         ("hurricane", "rel", 1e-3), ("miranda", "abs", 1e-4), ("miranda", "rel", 1e-4), ("miranda", "noa", 1e-4)]
if len(sys.argv) > 1 and sys.argv[1] == "big":
    CASES = [("big16g", "abs", 1e-3)]
K, W = 10, 3
res = []
print("| config | bound | MB | ratio | compress GB/s | decompress GB/s | compress roofline | decompress roofline |")
print("|---|---|---|---|---|---|---|---|")
for name, bound, eps in CASES:
    spec = synth.CONFIGS[name]
    x = synth.generate(spec, device="cuda")
    out = torch.empty(pk.max_compressed_bytes(x.numel(), x.dtype), dtype=torch.uint8, device="cuda")
    y = torch.empty_like(x)
    for _ in range(W):
        s = pk.compress(x, bound, eps, out=out)
        pk.decompress(s, out=y)
    tc, td = [], []
    for _ in range(K):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record()
        s = pk.compress(x, bound, eps, out=out)      # includes the D2H of the 8-byte size
        e[1].record()
        pk.decompress(s, out=y)
        e[2].record()
        torch.cuda.synchronize()
        tc.append(e[0].elapsed_time(e[1])); td.append(e[1].elapsed_time(e[2]))
    nb = x.numel() * x.element_size()
    c_ms, d_ms = statistics.median(tc), statistics.median(td)
    traffic = nb + s.numel() + (nb if bound == "noa" else 0)
    r = dict(config=spec.name, bound=bound, eps=eps, mb=nb / 1e6, ratio=nb / s.numel(),
             compress_gbs=nb / c_ms / 1e6, decompress_gbs=nb / d_ms / 1e6,
             compress_roofline=traffic / c_ms / 1e6 / PEAK, decompress_roofline=(nb + s.numel()) / d_ms / 1e6 / PEAK)
    res.append(r)
    print(f"| {r['config']} | {bound.upper()} {eps:g} | {r['mb']:.0f} | {r['ratio']:.2f} | {r['compress_gbs']:.0f} | "
          f"{r['decompress_gbs']:.0f} | {100*r['compress_roofline']:.1f}% | {100*r['decompress_roofline']:.1f}% |", flush=True)
    del x, out, y
    torch.cuda.empty_cache()
os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open("gpurun_out/bench_all%s.json" % ("_big" if len(sys.argv) > 1 else ""), "w"), indent=1)
