"""Compress/decompress GB/s, ratio and roofline fraction for every BASELINE.json
config on one GPU.  Device time = CUDA events around the async C-ABI calls
(median of K after W warm-ups; inputs resident in HBM); `api` = the blocking
pfpl_compress call (adds its host sync + 8-byte D2H).  Prints a markdown table,
writes gpurun_out/bench_all.json.   usage: bench_all.py [big] [case-filter | name:bound:eps ...]"""
import json, os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_fallinadcb25_b200 as pk
import synth

PEAK = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6650.0
CASES = [("cesm", "abs", 1e-3), ("nyx", "abs", 1e-3), ("nyx", "noa", 1e-3), ("nyx_rough", "abs", 1e-3),
         ("hurricane", "rel", 1e-3), ("miranda", "abs", 1e-4), ("miranda", "rel", 1e-4), ("miranda", "noa", 1e-4)]
args = sys.argv[1:]
big = bool(args) and args[0] == "big"
if big:
    CASES = [("big16g", "abs", 1e-3)]
    args = args[1:]
if args:
    # "name:bound:eps" adds an ad-hoc case; other args filter the table's cases
    extra = [(a.split(":")[0], a.split(":")[1], float(a.split(":")[2])) for a in args if a.count(":") == 2]
    CASES = [c for c in CASES if any(a in f"{c[0]}_{c[1]}" for a in args)] + extra
K, W = 10, 3
res = []
print("| config | bound | MB | ratio | compress GB/s | decompress GB/s | compress roofline | decompress roofline | api compress GB/s |")
print("|---|---|---|---|---|---|---|---|---|")
for name, bound, eps in CASES:
    spec = synth.CONFIGS[name]
    x = synth.generate(spec, device="cuda")
    out = torch.empty(pk.max_compressed_bytes(x.numel(), x.dtype), dtype=torch.uint8, device="cuda")
    rc = torch.zeros(4, dtype=torch.int64, device="cuda")
    rd = torch.zeros(4, dtype=torch.int64, device="cuda")
    y = torch.empty_like(x)
    s = pk.compress(x, bound, eps, out=out)
    hdr = s[:48].cpu().numpy().tobytes()
    nbytes_s = s.numel()
    for _ in range(W):
        pk.compress_async(x, out, rc, bound, eps)
        pk.decompress_async(out[:nbytes_s], hdr, y, rd)
    torch.cuda.synchronize()
    assert os.environ.get("PFPL_NOCHECK") or (int(rc[0]) == nbytes_s and int(rd[1]) == 0)
    tc, td, ta = [], [], []
    for _ in range(K):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record()
        pk.compress_async(x, out, rc, bound, eps)
        e[1].record()
        pk.decompress_async(out[:nbytes_s], hdr, y, rd)
        e[2].record()
        torch.cuda.synchronize()
        tc.append(e[0].elapsed_time(e[1])); td.append(e[1].elapsed_time(e[2]))
    for _ in range(K):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        e[0].record()
        pk.compress(x, bound, eps, out=out)
        e[1].record()
        torch.cuda.synchronize()
        ta.append(e[0].elapsed_time(e[1]))
    nb = x.numel() * x.element_size()
    c_ms, d_ms, a_ms = statistics.median(tc), statistics.median(td), statistics.median(ta)
    traffic = nb + nbytes_s + (nb if bound == "noa" else 0)
    r = dict(config=spec.name, bound=bound, eps=eps, mb=nb / 1e6, ratio=nb / nbytes_s,
             compress_gbs=nb / c_ms / 1e6, decompress_gbs=nb / d_ms / 1e6, api_compress_gbs=nb / a_ms / 1e6,
             compress_roofline=traffic / c_ms / 1e6 / PEAK, decompress_roofline=(nb + nbytes_s) / d_ms / 1e6 / PEAK)
    res.append(r)
    print(f"| {r['config']} | {bound.upper()} {eps:g} | {r['mb']:.0f} | {r['ratio']:.2f} | {r['compress_gbs']:.0f} | "
          f"{r['decompress_gbs']:.0f} | {100*r['compress_roofline']:.1f}% | {100*r['decompress_roofline']:.1f}% | "
          f"{r['api_compress_gbs']:.0f} |", flush=True)
    del x, out, y
    torch.cuda.empty_cache()
os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open("gpurun_out/bench_all%s.json" % ("_big" if big else ""), "w"), indent=1)
