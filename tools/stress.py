"""Repeat compress/decompress of one config many times and check that every
stream is byte-identical to the first and every decode is exact (catches
races in the look-back / arena / ring protocols).  usage: stress.py CONFIG BOUND EPS REPS"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_fallinadcb25_b200 as pk
import synth
name, bound, eps, reps = sys.argv[1], sys.argv[2], float(sys.argv[3]), int(sys.argv[4])
x = synth.generate(synth.CONFIGS[name], device="cuda")
out = torch.empty(pk.max_compressed_bytes(x.numel(), x.dtype), dtype=torch.uint8, device="cuda")
rc = torch.zeros(4, dtype=torch.int64, device="cuda")
rd = torch.zeros(4, dtype=torch.int64, device="cuda")
y = torch.empty_like(x)
ref = pk.compress(x, bound, eps).clone()
hdr = ref[:48].cpu().numpy().tobytes()
bad = 0
for i in range(reps):
    out.fill_(0xA5) if i % 8 == 0 else None
    pk.compress_async(x, out, rc, bound, eps)
    pk.decompress_async(ref, hdr, y, rd)
    torch.cuda.synchronize()
    n = int(rc[0])
    ok = n == ref.numel() and torch.equal(out[:n], ref) and int(rd[1]) == 0 and torch.equal(y.view(torch.int32) if y.dtype == torch.float32 else y.view(torch.int64), pk.decompress(ref).view(y.dtype).view(torch.int32) if y.dtype == torch.float32 else pk.decompress(ref).view(torch.int64)) if i % 16 == 0 else (n == ref.numel() and torch.equal(out[:n], ref) and int(rd[1]) == 0)
    if not ok:
        bad += 1
        print(f"rep {i}: MISMATCH n={n} ref={ref.numel()} dec_status={int(rd[1])}", flush=True)
print(f"{name} {bound} {eps}: {reps} reps, {bad} bad")
