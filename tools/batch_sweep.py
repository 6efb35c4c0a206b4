"""Multi-field batch (pfpl_compress_batch) vs one pfpl_compress per field, on 33
CESM-shaped 1800x3600 f32 fields (CESM-ATM has 33 per timestep).  Prints one
JSON line; host-timed around the blocking calls (both synchronise once per call)."""
import json
import statistics
import time

import torch

import paper_conf_ipps_fallinadcb25_b200 as pk
import synth

base = synth.CONFIGS["cesm"]
xs = [synth.generate(synth.FieldSpec(base.name, base.shape, "f32", 100 + i, A=0.3, tau=1e-3),
                     device="cuda").view(-1) for i in range(33)]
nbytes = sum(x.numel() * 4 for x in xs)
outs = [torch.empty(pk.max_compressed_bytes(x.numel(), torch.float32), dtype=torch.uint8, device="cuda")
        for x in xs]
res = {}
for bound in ("abs", "noa", "rel"):
    seq, bat, dseq, dbat = [], [], [], []
    ys = [torch.empty_like(x) for x in xs]
    for it in range(6):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        a = [pk.compress(x, bound, 1e-3, out=o).numel() for x, o in zip(xs, outs)]
        t1 = time.perf_counter()
        bs = pk.compress_batch(xs, bound, 1e-3, outs=outs)
        t2 = time.perf_counter()
        b = [o.numel() for o in bs]
        assert a == b
        torch.cuda.synchronize()
        t3 = time.perf_counter()
        for s_, y in zip(bs, ys):
            pk.decompress(s_, out=y)
        t4 = time.perf_counter()
        pk.decompress_batch(bs, outs=ys)
        t5 = time.perf_counter()
        if it:
            seq.append(t1 - t0)
            bat.append(t2 - t1)
            dseq.append(t4 - t3)
            dbat.append(t5 - t4)
    res[bound] = {"sequential_gbs": nbytes / statistics.median(seq) / 1e9,
                  "batch_gbs": nbytes / statistics.median(bat) / 1e9, "ratio": nbytes / sum(b),
                  "decompress_sequential_gbs": nbytes / statistics.median(dseq) / 1e9,
                  "decompress_batch_gbs": nbytes / statistics.median(dbat) / 1e9}
print(json.dumps({"fields": 33, "bytes": nbytes, "eps": 1e-3, **res}))
