import sys, os, torch
sys.path.insert(0, os.getcwd())
import paper_conf_ipps_fallinadcb25_b200 as pk, synth
spec = synth.CONFIGS["big16g"]
for rows in (64, 256, 1024):
    x = synth.generate(spec, device="cuda", slab=(0, rows))
    out = torch.empty(pk.max_compressed_bytes(x.numel(), x.dtype), dtype=torch.uint8, device="cuda")
    rc = torch.zeros(4, dtype=torch.int64, device="cuda")
    for _ in range(3): pk.compress_async(x, out, rc, "abs", 1e-3)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    ts = []
    for _ in range(7):
        e0.record(); pk.compress_async(x, out, rc, "abs", 1e-3); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1))
    ts.sort(); t = ts[3]
    print(rows, x.numel() * 4 / 1e6, "MB", "ratio", x.numel() * 4 / int(rc[0]), "GB/s", x.numel() * 4 / t / 1e6)
    del x, out
