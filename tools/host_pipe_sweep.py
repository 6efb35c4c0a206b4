"""Segment-size sweep of the host-resident pipeline (pfpl_compress_host /
pfpl_decompress_host) on the NYX-shaped field; prints one JSON line per size."""
import json
import statistics
import time

import torch

import paper_conf_ipps_fallinadcb25_b200 as pk
import synth

x = synth.generate(synth.CONFIGS["nyx"], device="cuda").view(-1)
xh = x.cpu().pin_memory()
nbytes = xh.numel() * 4
oh = torch.empty(pk.max_compressed_bytes(xh.numel(), torch.float32), dtype=torch.uint8).pin_memory()
yh = torch.empty_like(xh).pin_memory()
# raw copy rates for context
d = torch.empty_like(x)
for name, fn in (("h2d", lambda: d.copy_(xh, non_blocking=True)), ("d2h", lambda: yh.copy_(d, non_blocking=True))):
    ts = []
    for _ in range(4):
        torch.cuda.synchronize(); t = time.perf_counter(); fn(); torch.cuda.synchronize()
        ts.append(time.perf_counter() - t)
    print(json.dumps({"copy": name, "gbs": nbytes / statistics.median(ts[1:]) / 1e9}))
for seg in (256, 512, 1024, 2048, 4096, 8192):
    tc, td = [], []
    for it in range(5):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        hb = pk.compress_host(xh, "abs", 1e-3, out=oh, seg_chunks=seg).numel()
        t1 = time.perf_counter()
        pk.decompress_host(oh[:hb], out=yh, seg_chunks=seg)
        t2 = time.perf_counter()
        if it:
            tc.append(t1 - t0)
            td.append(t2 - t1)
    print(json.dumps({"seg_chunks": seg, "compress_gbs": nbytes / statistics.median(tc) / 1e9,
                      "decompress_gbs": nbytes / statistics.median(td) / 1e9}))
