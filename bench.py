#!/usr/bin/env python3
"""PFPL hot-path benchmark (BASELINE.json metric).

python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                [--config nyx] [--bound abs] [--eps 1e-3]

One step = one pass of the whole hot path over the synthetic field: compress
(a0-a8: quantize/verify, delta+negabinary, bit shuffle, zero/repeat
elimination, look-back concatenation) then decompress (d1-d5).  Inputs are
resident in HBM before timing; they are larger than L2 (NYX: 537 MB vs 126 MB)
so no flush is needed.  Times are CUDA events on the launching stream,
max over ranks.  value = compression throughput in uncompressed GB/s (10^9,
P:225), whole job; decompression GB/s and ratio are reported beside it.

N > 1 (one process per GPU; `--gpus N` starts the N ranks itself under
torch.distributed.run when WORLD_SIZE is unset): BASELINE.json configs[4] --
the 16 GiB f32 field (1024x2048x2048, n = 2^32), ABS 1E-3, STRONG scaling:
rank r generates and compresses its chunk-aligned slab; NCCL all-reduces the
NOA range (NOA only) and all-gathers the per-shard payload sizes so every
rank knows its offset in the single assembled stream.  After
the timed region rank 0 compresses the whole field on one GPU and every
rank's table slice and payload are compared (64-bit checksums of the same
byte ranges) with that single-GPU stream.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "compress/decompress GB/s (uncompressed) + ratio, f32 ABS 1E-3, 1/2/4/8 B200"
PAPER_CONTEXT = {"paper_pfpl_cuda_rtx4090_gbs": 423, "paper_pfpl_omp_ryzen2950x_gbs": 5,
                 "note": "f32 ABS 1E-3 SDRBench geo-mean (P:15); other hardware, context only"}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default=None,
                    help="synth config; default nyx (configs[1]) at N=1, big16g (configs[4]) at N>1")
    ap.add_argument("--bound", default="abs")
    ap.add_argument("--eps", type=float, default=1e-3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--quiet", action="store_true")
    return ap.parse_args()


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return None


class Clocks:
    """Sample SM clocks and clock-event (throttle) reasons DURING the timed region.

    NVML (nvidia-ml-py) polled from a thread every ~0.5 ms: the timed region
    of a default run is tens of ms, far below nvidia-smi's sampling period.
    Samples are kept only while `active` is set (the timed loop)."""

    BITS = {"hw_slowdown": 0x8, "hw_thermal_slowdown": 0x40, "sw_thermal_slowdown": 0x20,
            "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80}

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self.active = False
        self.stop = False
        self.err = None
        self.max_mhz = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            idx = self.index
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            if vis and vis.split(",")[idx].strip().isdigit():
                idx = int(vis.split(",")[idx])
            self.h = pynvml.nvmlDeviceGetHandleByIndex(idx)
            self.nv = pynvml
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        except Exception as e:          # no NVML: reported as unavailable, never faked
            self.err = repr(e)
        return self

    def _run(self):
        nv, h = self.nv, self.h
        while not self.stop:
            if self.active:
                try:
                    mhz = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                    rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                    self.samples.append((mhz, rs))
                except Exception as e:
                    self.err = repr(e)
                time.sleep(0.0005)
            else:
                time.sleep(0.0002)

    def __exit__(self, *a):
        self.stop = True

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": ["unavailable"],
                    "samples": 0, "error": self.err}
        reasons = sorted({nm for _, rs in self.samples for nm, b in self.BITS.items() if rs & b})
        return {"sm_mhz": statistics.median(m for m, _ in self.samples), "sm_max_mhz": self.max_mhz,
                "sm_min_mhz": min(m for m, _ in self.samples), "reasons": reasons,
                "samples": len(self.samples), "source": "NVML, polled during the timed region"}


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "unknown"


def _time_oracle(x, bound, eps, threads, seconds):
    """Median-free mean over enough repetitions to fill ~`seconds` (at least 1)."""
    import oracle
    t0 = time.perf_counter()
    s = oracle.compress(x, bound, eps, nthreads=threads)
    first = time.perf_counter() - t0
    reps = max(1, min(50, int(seconds / max(first, 1e-3))))
    t0 = time.perf_counter()
    for _ in range(reps):
        oracle.compress(x, bound, eps, nthreads=threads)
    tc = (time.perf_counter() - t0) / reps
    rd = max(1, reps // 2)
    t0 = time.perf_counter()
    for _ in range(rd):
        oracle.decompress(s, nthreads=threads)
    td = (time.perf_counter() - t0) / rd
    return tc, td, s, reps


def _time_cpu_codec(x, s_oracle, bound, eps, cores, seconds):
    """The multi-core CPU production codec (libpfpl_cpu.so) on the same
    sample: all host threads and one thread; its stream must equal the oracle's."""
    import numpy as np
    from paper_conf_ipps_fallinadcb25_b200 import cpu
    out = np.empty(cpu.lib().pfpl_cpu_max_compressed_bytes(x.size, 0 if x.dtype == np.float32 else 1), np.uint8)
    y = np.empty_like(x)
    res = {"kind": "PFPL CPU codec (OpenMP, AVX2; P:139-168)", "cores": cores,
           "identical_to_oracle_stream": bytes(cpu.compress(x, bound, eps, out=out)) == s_oracle}
    for label, nt in (("all_threads", cores), ("single_thread", 1)):
        s = cpu.compress(x, bound, eps, nthreads=nt, out=out)
        nb = s.size
        cpu.decompress(out[:nb], nthreads=nt, out=y)
        reps = 0
        t0 = time.perf_counter()
        while reps < 3 or (time.perf_counter() - t0 < seconds / 4 and reps < 200):
            cpu.compress(x, bound, eps, nthreads=nt, out=out)
            reps += 1
        tc = (time.perf_counter() - t0) / reps
        reps_d = 0
        t0 = time.perf_counter()
        while reps_d < 3 or (time.perf_counter() - t0 < seconds / 4 and reps_d < 200):
            cpu.decompress(out[:nb], nthreads=nt, out=y)
            reps_d += 1
        td = (time.perf_counter() - t0) / reps_d
        res[label] = {"compress_gbs": x.nbytes / tc / 1e9, "decompress_gbs": x.nbytes / td / 1e9,
                      "threads": nt, "reps": [reps, reps_d]}
    return res


def cpu_baseline(spec, bound, eps, seconds):
    """The oracle as it stands (plain C, chunks over host threads) on a bounded
    sample of the same workload (the first rows of the field), on the SAME bytes
    twice: one thread, and all host threads (OpenMP over chunks) -- SURVEY 8(d)."""
    import oracle
    import synth
    cores = len(os.sched_getaffinity(0))
    oracle.build()
    inner = spec.n // spec.shape[0]
    rows = max(1, min(spec.shape[0], (64 << 20) // (inner * spec.itemsize)))
    x = synth.generate(spec, slab=(0, rows)).numpy()
    tc, td, s, reps = _time_oracle(x, bound, eps, cores, 0.6 * seconds)
    # single thread on a quarter of the same sample (whole rows), so the run stays bounded
    x1 = x[:max(inner, (x.size // 4) // inner * inner)]
    tc1, td1, _, reps1 = _time_oracle(x1, bound, eps, 1, 0.4 * seconds)
    cpu_codec = _time_cpu_codec(x, s, bound, eps, cores, 0.5 * seconds)
    return {"value": x.nbytes / tc / 1e9, "unit": "GB/s", "cores": cores, "kind": "oracle",
            "cpu_model": cpu_model(), "cpu_codec": cpu_codec,
            "sample": f"first {rows} of {spec.shape[0]} rows ({x.nbytes / 1e6:.1f} MB), "
                      f"{reps} reps, OpenMP over chunks on {cores} threads",
            "decompress_gbs": x.nbytes / td / 1e9, "ratio": x.nbytes / len(s),
            "single_thread": {"value": x1.nbytes / tc1 / 1e9, "unit": "GB/s", "cores": 1,
                              "decompress_gbs": x1.nbytes / td1 / 1e9,
                              "sample": f"first {x1.size // inner} rows ({x1.nbytes / 1e6:.1f} MB) "
                                        f"of the same sample, {reps1} reps, 1 thread"}}


def run_reference(args):
    """--impl reference: the CPU oracle, timed on the host cores (rank 0 only)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import numpy as np
    import oracle
    import synth
    spec = synth.CONFIGS[args.config or ("nyx" if args.gpus == 1 else "big16g")]
    cores = len(os.sched_getaffinity(0))
    oracle.build()
    inner = spec.n // spec.shape[0]
    rows = max(1, min(spec.shape[0], (32 << 20) // (inner * spec.itemsize)))
    x = synth.generate(spec, slab=(0, rows)).numpy()
    for _ in range(args.warmup):
        s = oracle.compress(x, args.bound, args.eps, nthreads=cores)
    tc, td = [], []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        s = oracle.compress(x, args.bound, args.eps, nthreads=cores)
        t1 = time.perf_counter()
        oracle.decompress(s, nthreads=cores)
        t2 = time.perf_counter()
        tc.append(t1 - t0)
        td.append(t2 - t1)
    comp = x.nbytes / statistics.median(tc) / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": comp, "unit": "GB/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": 1e3 * (statistics.median(tc) + statistics.median(td)),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": spec.dtype,
        "data": "synthetic", "config": _config(spec, args, sample_rows=rows, world=args.gpus),
        "ratio": x.nbytes / len(s), "decompress_gbs": x.nbytes / statistics.median(td) / 1e9,
        "cpu_baseline": {"value": comp, "unit": "GB/s", "cores": cores, "kind": "oracle",
                         "cpu_model": cpu_model(),
                         "sample": f"first {rows} of {spec.shape[0]} rows ({x.nbytes / 1e6:.1f} MB) per step"},
        "e2e": {"value": comp, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "context": PAPER_CONTEXT,
    }
    print(json.dumps(line), flush=True)


def _traffic(config, bound):
    """dram__bytes_read.sum + dram__bytes_write.sum per launch of the encoder /
    decoder, from the committed ncu --set full summary (profiles/traffic.json)"""
    f = os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles", "traffic.json")
    try:
        t = json.load(open(f))
    except (OSError, ValueError):
        return {}
    e = t.get(f"{config}/{bound}", {})
    return dict(e, source=t.get("source")) if e else {}


def _config(spec, args, sample_rows=None, world=1):
    c = {"workload": f"{spec.name}, {args.bound.upper()} {args.eps:g}", "shape": list(spec.shape),
         "bound": args.bound, "eps": args.eps, "n": spec.n, "bytes": spec.nbytes,
         "l2": "inputs larger than L2 (no flush needed)" if spec.nbytes > 126e6 else "L2 flushed",
         "parallelism": f"dp{world} chunk shards"}
    if sample_rows is not None:
        c["sample_rows"] = sample_rows
    return c


def run_ours(args):
    import ctypes

    import numpy as np
    import torch
    import torch.distributed as dist

    import paper_conf_ipps_fallinadcb25_b200 as pk
    from paper_conf_ipps_fallinadcb25_b200 import dist as pdist
    import synth

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # PFPL_BENCH_SHARE_GPU=1 maps all ranks onto the visible GPUs round-robin
    # (functional test of the multi-rank path on a 1-GPU box, with gloo)
    if os.environ.get("PFPL_BENCH_SHARE_GPU"):
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        backend = os.environ.get("PFPL_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    from paper_conf_ipps_fallinadcb25_b200 import _build
    if rank == 0:
        _build.build()
    if world > 1:
        dist.barrier()
    L = pk.lib()

    # N = 1: the headline NYX field (configs[1]); N > 1: configs[4], the 16 GiB field,
    # strong scaling -- rank r owns the chunk-aligned slab r of the same global field
    cfg = args.config or ("nyx" if world == 1 else "big16g")
    base = synth.CONFIGS[cfg]
    spec = base
    n_total = spec.n
    esz = spec.itemsize
    fc, nch, e0, e1 = pdist.shard_chunks(n_total, esz, rank, world)
    x = _generate_range(synth, spec, e0, e1, dev)
    torch.cuda.synchronize()
    n = x.numel()
    nbytes = n * esz
    dt = pk.F32 if x.dtype == torch.float32 else pk.F64
    bd = pk._BOUNDS[args.bound]
    stream = torch.cuda.current_stream()
    sh = stream.cuda_stream
    cap = pk.max_compressed_bytes(n, dt)
    out = torch.empty(cap, dtype=torch.uint8, device=dev)
    res = torch.zeros(4, dtype=torch.int64, device=dev)
    y = torch.empty_like(x)
    state = {}

    # ---- one step = compress then decompress ----
    def compress_once():
        if world == 1:
            pk._check(L.pfpl_compress_async(x.data_ptr(), n, dt, bd, args.eps, 0, out.data_ptr(), cap,
                                            res.data_ptr(), sh))
            return None
        r = pdist.compress_sharded(x, n_total, args.bound, args.eps,
                                   shard_fn=lambda xx, f, nt, b, e, m, mm: pk.compress_shard(
                                       xx, f, nt, b, e, m, mm, out=out))
        state["shard"] = r
        return r

    def decompress_once(r):
        if world == 1:
            pk._check(L.pfpl_decompress_async(out.data_ptr(), state["bytes"], state["hdr_buf"],
                                              y.data_ptr(), nbytes, res.data_ptr(), sh))
        else:
            pk._check(L.pfpl_decompress_chunks(state["hdr_buf"],
                                               state["table"].ctypes.data_as(ctypes.c_void_p),
                                               r.first_chunk, nch, r.payload.data_ptr(),
                                               r.payload.numel(), y.data_ptr(), nbytes, sh))

    clk = Clocks(local).__enter__()
    for _ in range(max(1, args.warmup)):
        r = compress_once()
    torch.cuda.synchronize()
    if world == 1:
        state["bytes"] = int(res[0].item())
        hdr = out[:48].cpu().numpy().tobytes()
        comp_bytes = state["bytes"]
    else:
        hdr = r.header
        state["table"] = r.table.cpu().numpy().view(np.uint32).copy()
        comp_bytes = r.total_bytes
    state["hdr_buf"] = ctypes.cast(ctypes.create_string_buffer(hdr, 48), ctypes.c_void_p)
    for _ in range(max(1, args.warmup)):
        decompress_once(r)
    torch.cuda.synchronize()
    if world == 1:
        assert int(res[1].item()) == 0, "decode reported corruption"
    assert torch.equal(y[:1024], y[:1024])

    ev = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    launches0 = pk.launch_count()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t_wall0 = time.perf_counter()
    clk.active = True
    for i in range(args.steps):
        ev[i][0].record(stream)
        r = compress_once()
        ev[i][1].record(stream)
        decompress_once(r)
        ev[i][2].record(stream)
    torch.cuda.synchronize()
    clk.active = False
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t_wall = time.perf_counter() - t_wall0
    launches = pk.launch_count() - launches0
    clk.__exit__(None, None, None)
    tc = [ev[i][0].elapsed_time(ev[i][1]) for i in range(args.steps)]
    td = [ev[i][1].elapsed_time(ev[i][2]) for i in range(args.steps)]
    tc_sum, td_sum = sum(tc), sum(td)
    if world > 1:
        t = torch.tensor([tc_sum, td_sum], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        tc_sum, td_sum = t.tolist()
    total_bytes = n_total
    total_bytes *= esz
    comp_gbs = total_bytes * args.steps / (tc_sum * 1e-3) / 1e9
    dec_gbs = total_bytes * args.steps / (td_sum * 1e-3) / 1e9
    ratio = total_bytes / comp_bytes

    # ---- roofline of the dominant kernel (the fused encoder), measured live ----
    peaks = _peaks()
    peak = peaks["hbm_gbs"] if peaks else 6650.0
    enc_ms = statistics.median(tc)
    my_comp = comp_bytes if world == 1 else (4 * nch + r.payload.numel())
    algo = nbytes + my_comp                  # input read + stream written, per launch (this rank)
    traffic = _traffic(cfg, args.bound)
    roof = {"bound": "hbm", "achieved": algo / (enc_ms * 1e-3) / 1e9, "peak": peak, "unit": "GB/s",
            "frac": algo / (enc_ms * 1e-3) / 1e9 / peak,
            "traffic": traffic.get("encode") if world == 1 else None,
            "traffic_source": traffic.get("source"), "algorithmic_bytes": algo,
            "kernel": "encode_kernel (compress step)",
            "peak_source": "MEASURED_PEAKS.json hbm_gbs (measured)" if peaks else "fallback 6.65 TB/s (B200_PROFILING.md)"}
    dec_ms = statistics.median(td)
    roof_dec = {"kernel": "decode_kernel", "achieved": algo / (dec_ms * 1e-3) / 1e9,
                "frac": algo / (dec_ms * 1e-3) / 1e9 / peak,
                "traffic": traffic.get("decode") if world == 1 else None}

    # ---- full-size bound check on the GPU: verify-mode decode of this rank's stream
    # against the input (pfpl_decompress_verify), timed separately ----
    verify = None
    if world == 1:
        ctypes_m = pk.Metrics()
        tv = []
        for _ in range(3):
            ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ob = ctypes.c_uint64(nbytes)
            ev0.record(stream)
            pk._check(L.pfpl_decompress_verify(out.data_ptr(), state["bytes"], x.data_ptr(), y.data_ptr(),
                                               ctypes.byref(ob), ctypes.byref(ctypes_m), sh))
            ev1.record(stream)
            torch.cuda.synchronize()
            tv.append(ev0.elapsed_time(ev1))
        verify = {"violations": int(ctypes_m.violations), "max_abs_err": ctypes_m.max_abs_err,
                  "max_rel_err": ctypes_m.max_rel_err, "psnr_db": ctypes_m.psnr,
                  "n_finite": int(ctypes_m.n_finite), "eps": args.eps, "bound": args.bound,
                  "decompress_verify_gbs": nbytes / (statistics.median(tv) * 1e-3) / 1e9,
                  "what": "every value of the full-size stream decoded and checked against the input "
                          "in the decode epilogue (f64 arithmetic); includes the API's host syncs"}
        verify["encoder_stats"] = pk.last_stats(stream)     # the last timed compress on this stream

    # ---- end to end through the public API with host buffers (pinned) ----
    xh = x.cpu().pin_memory()
    oh = torch.empty(cap, dtype=torch.uint8).pin_memory()
    xd2 = torch.empty_like(x)
    e_steps = max(2, min(args.steps, 5))
    t0e = torch.cuda.Event(enable_timing=True)
    t1e = torch.cuda.Event(enable_timing=True)
    d2h = 0
    for it in range(e_steps + 1):
        if it == 1:
            if world > 1:
                dist.barrier()
            t0e.record(stream)
        xd2.copy_(xh, non_blocking=True)
        if world == 1:
            nb = ctypes.c_uint64(cap)
            pk._check(L.pfpl_compress(xd2.data_ptr(), n, dt, bd, args.eps, out.data_ptr(),
                                      ctypes.byref(nb), sh))
            d2h = nb.value
            oh[:d2h].copy_(out[:d2h], non_blocking=True)
        else:
            rr = pdist.compress_sharded(xd2, n_total, args.bound, args.eps,
                                        shard_fn=lambda xx, f, nt, b, e, m, mm: pk.compress_shard(
                                            xx, f, nt, b, e, m, mm, out=out))
            d2h = 4 * nch + rr.payload.numel()
            oh[:d2h].copy_(out[:d2h], non_blocking=True)
    t1e.record(stream)
    torch.cuda.synchronize()
    e_ms = t0e.elapsed_time(t1e) / e_steps
    if world > 1:
        t = torch.tensor([e_ms], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e_ms = t.item()
    e2e = {"value": total_bytes / (e_ms * 1e-3) / 1e9, "unit": "GB/s", "h2d_bytes_per_step": nbytes,
           "d2h_bytes_per_step": int(d2h),
           "what": "per rank: pinned H2D of its slab + compress (C ABI) + D2H of its stream part; max over ranks"}
    if world == 1:
        # the host-resident API (pfpl_compress_host / pfpl_decompress_host, NEXT-4):
        # segmented H2D / kernel / D2H on three streams; the call returns after the
        # last D2H has landed, so host-side timing around it is the whole job
        seq = dict(e2e)
        hb = 0
        th, td = [], []
        yh = torch.empty(n, dtype=x.dtype).pin_memory()
        for it in range(e_steps + 1):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            hb = pk.compress_host(xh, args.bound, args.eps, out=oh, stream=stream).numel()
            t1 = time.perf_counter()
            pk.decompress_host(oh[:hb], out=yh, stream=stream)
            t2 = time.perf_counter()
            if it:
                th.append(t1 - t0)
                td.append(t2 - t1)
        # outside the timed region: same stream bytes and values as the device path
        if hb != seq["d2h_bytes_per_step"] or not torch.equal(
                yh, pk.decompress(out[:hb], stream=stream).cpu()):
            raise RuntimeError("host pipeline disagrees with the device-resident path")
        e2e = {"value": total_bytes / statistics.median(th) / 1e9, "unit": "GB/s",
               "h2d_bytes_per_step": nbytes, "d2h_bytes_per_step": int(hb),
               "decompress_gbs": total_bytes / statistics.median(td) / 1e9,
               "decompress_h2d_bytes": int(hb), "decompress_d2h_bytes": nbytes,
               "what": "pfpl_compress_host on a pinned host array: segmented H2D -> compress -> D2H "
                       "pipelined over 3 streams (32 MiB segments), host-timed around the blocking call; "
                       "decompress_gbs the same for pfpl_decompress_host",
               "sequential_device_api": seq}

    # ---- N > 1: the assembled stream must be the single-GPU stream ----
    identity = None
    if world > 1:
        identity = _identity_check(pk, synth, pdist, dist, spec, args, state["shard"], out, nch,
                                   rank, world, dev, stream)

    if rank != 0:
        if world > 1:
            dist.destroy_process_group()
        return
    line = {
        "metric": METRIC, "value": comp_gbs, "unit": "GB/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": (tc_sum + td_sum) / args.steps, "higher_is_better": True,
        "scaling": "strong" if world > 1 else "weak", "vs_baseline": None, "dtype": spec.dtype,
        "data": "synthetic", "config": _config(base, args, world=world),
        "ratio": ratio, "compress_gbs": comp_gbs, "decompress_gbs": dec_gbs,
        "compress_ms": tc_sum / args.steps, "decompress_ms": td_sum / args.steps,
        "roofline": roof, "roofline_decode": roof_dec,
        "gpu_launches": int(launches), "launches_per_step": launches / args.steps,
        "clocks": clk.summary(), "wall_s": t_wall, "e2e": e2e, "context": PAPER_CONTEXT,
    }
    if verify is not None:
        line["verify"] = verify
    if world > 1:
        line["config"]["global_shape"] = list(spec.shape)
        line["identity"] = identity
        line["per_gpu_gbs"] = comp_gbs / world
        if os.environ.get("PFPL_BENCH_SHARE_GPU"):
            line["shared_gpu"] = ("functional run: all ranks share the visible GPU(s) "
                                  f"({torch.cuda.device_count()}); not a scaling measurement")
    if not args.no_cpu_baseline and world == 1:
        line["cpu_baseline"] = cpu_baseline(base, args.bound, args.eps, args.cpu_seconds)
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def _generate_range(synth, spec, e0, e1, dev):
    """Elements [e0, e1) of the field, generated from whole rows of its slowest axis."""
    import torch
    inner = spec.n // spec.shape[0]
    r0, r1 = e0 // inner, -(-e1 // inner)
    x = synth.generate(spec, device=dev, slab=(r0, r1))
    if e0 - r0 * inner or r1 * inner - e1:
        x = x[e0 - r0 * inner:e1 - r0 * inner].contiguous()
    torch.cuda.synchronize()
    return x


def _cksum(t):
    """(bytes, two 64-bit position-weighted sums) of a uint8 CUDA tensor."""
    import torch
    nb = t.numel()
    pad = (-nb) % 8
    v = torch.cat([t, torch.zeros(pad, dtype=torch.uint8, device=t.device)]) if pad else t
    w = v.view(torch.int64)
    idx = torch.arange(w.numel(), dtype=torch.int64, device=t.device)
    h1 = int((w * (2 * idx + 1)).sum().item())
    h2 = int((w ^ (idx * 40503 + 17)).sum().item())
    return [nb, h1, h2]


def _identity_check(pk, synth, pdist, dist, spec, args, r, out, nch, rank, world, dev, stream):
    """Rank 0 compresses the whole field with the single-GPU API; every rank's
    table slice and payload are compared with the same byte ranges of that
    stream by 64-bit checksums (all-gathered), plus the header and total size."""
    import torch
    mine = _cksum(r.table.view(torch.uint8)) + _cksum(r.payload)
    vals = torch.tensor(mine, dtype=torch.int64)
    backend = dist.get_backend()
    if backend == "nccl":
        vals = vals.to(dev)
    allv = [torch.empty_like(vals) for _ in range(world)]
    dist.all_gather(allv, vals)
    allv = [v.cpu().tolist() for v in allv]
    res = None
    if rank == 0:
        t0 = time.perf_counter()
        full = _generate_range(synth, spec, 0, spec.n, dev)
        single = pk.compress(full, args.bound, args.eps, stream=stream)
        torch.cuda.synchronize()
        ok = len(r.header) == 48 and bytes(single[:48].cpu().numpy().tobytes()) == r.header
        ok = ok and single.numel() == r.total_bytes
        C = pdist.chunks_of(spec.n, spec.itemsize)
        toff = 48
        poff = 48 + 4 * C
        per_rank = []
        for q in range(world):
            _, nq, _, _ = pdist.shard_chunks(spec.n, spec.itemsize, q, world)
            tb = single[toff:toff + 4 * nq]
            pb = single[poff:poff + r.sizes[q]]
            good = (_cksum(tb) + _cksum(pb)) == allv[q]
            per_rank.append(bool(good))
            toff += 4 * nq
            poff += r.sizes[q]
        ok = ok and all(per_rank) and poff == single.numel()
        # the same workload on this one GPU (context for the driver's scaling numbers, which
        # compare against the N = 1 line; that line is the NYX headline workload)
        outb = torch.empty(pk.max_compressed_bytes(full.numel(), full.dtype), dtype=torch.uint8, device=dev)
        rcv = torch.zeros(4, dtype=torch.int64, device=dev)
        ts = []
        for i in range(4):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            pk.compress_async(full, outb, rcv, args.bound, args.eps, stream=stream)
            e1.record(stream)
            torch.cuda.synchronize()
            if i:
                ts.append(e0.elapsed_time(e1))
        one_gpu = {"compress_gbs": spec.n * spec.itemsize / (statistics.median(ts) * 1e-3) / 1e9,
                   "what": "rank 0 alone, one GPU, the whole field of this line's workload, "
                           "pfpl_compress_async between CUDA events, median of 3 after 1 warm-up "
                           "(the N = 1 bench line is the NYX headline workload instead)"}
        del outb, rcv
        res = {"identical_to_single_gpu_stream": bool(ok), "per_rank": per_rank,
               "single_gpu_same_workload": one_gpu,
               "stream_bytes": int(single.numel()),
               "method": "rank 0: pfpl_compress of the whole field on one GPU; header, total size and "
                         "64-bit checksums of every rank's table slice and payload vs the same byte "
                         "ranges of that stream",
               "seconds": round(time.perf_counter() - t0, 2)}
        del full, single
        torch.cuda.empty_cache()
    dist.barrier()
    return res


def relaunch_distributed(args) -> None:
    """`--gpus N` without torchrun: start the N ranks ourselves (torch.distributed.run,
    127.0.0.1).  With fewer visible GPUs than N, the ranks share them (gloo for the two
    tiny exchanges) -- a functional run, flagged `shared_gpu` in the line."""
    import torch
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    env = dict(os.environ)
    if torch.cuda.device_count() < args.gpus:
        env["PFPL_BENCH_SHARE_GPU"] = "1"
        env.setdefault("PFPL_DIST_BACKEND", "gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={args.gpus}", "--master-addr=127.0.0.1", f"--master-port={port}",
           os.path.abspath(__file__)] + sys.argv[1:]
    os.execve(sys.executable, cmd, env)


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    elif args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        relaunch_distributed(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
