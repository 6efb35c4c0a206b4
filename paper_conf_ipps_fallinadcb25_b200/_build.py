"""Build libpfpl.so in-tree for sm_100a (nvcc cross-compiles without a GPU).

Flags that matter for CPU/GPU bit-identity: -fmad=false (no FMA
contraction), IEEE division/sqrt, no flush-to-zero; host code with
-ffp-contract=off.
"""
from __future__ import annotations

import glob
import os
import shutil
import subprocess

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
LIB = os.path.join(PKG, "libpfpl.so")
SRCS = sorted(f for f in glob.glob(os.path.join(PKG, "csrc", "*.cu")) if not f.endswith("pfpl_inst.cu"))
INST = os.path.join(PKG, "csrc", "pfpl_inst.cu")
# (kind, dtype, mode): encoder f32/f64 x ABS/REL/RAW/NOA, decoder f32/f64 x ABS/REL/RAW
INST_JOBS = [(0, d, m) for d in (0, 1) for m in range(4)] + [(1, d, m) for d in (0, 1) for m in range(3)]
DEPS = SRCS + [INST] + glob.glob(os.path.join(PKG, "csrc", "*.h")) + glob.glob(os.path.join(PKG, "csrc", "*.cuh")) \
    + [os.path.join(ROOT, "include", "pfpl.h")]

NVCC_FLAGS = [
    "-gencode", "arch=compute_100a,code=sm_100a",
    "-O3", "-lineinfo", "-std=c++17",
    "-fmad=false", "-prec-div=true", "-prec-sqrt=true", "-ftz=false",
    "-Xcompiler", "-fPIC,-ffp-contract=off,-fno-fast-math,-O2",
    "-Xptxas", "-v",
    "--expt-relaxed-constexpr",
]


def nvcc() -> str:
    for c in (os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")):
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found")


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in DEPS)


def build(force: bool = False, verbose: bool = False, jobs: int = os.cpu_count() or 8,
          out: str | None = None, extra: list | None = None) -> str:
    """Compile libpfpl.so (or, for tuning experiments, a variant library `out`
    built with `extra` nvcc flags, e.g. -DPFPL_ENC_NIN=1)."""
    lib = out or LIB
    extra = list(extra or [])
    if not force and not extra and out is None and not needs_build():
        return LIB
    bdir = os.path.join(ROOT, "build" if not extra else "build_" + os.path.basename(lib).replace(".so", ""))
    os.makedirs(bdir, exist_ok=True)
    jobs_ = []
    for src in SRCS:
        jobs_.append((src, os.path.join(bdir, os.path.basename(src) + ".o"), []))
    for k, d, m in INST_JOBS:
        jobs_.append((INST, os.path.join(bdir, f"{'enc' if k == 0 else 'dec'}_{d}_{m}.o"),
                      [f"-DPFPL_KIND={k}", f"-DPFPL_DT={d}", f"-DPFPL_MODE={m}"]))
    jobs_.sort(key=lambda j: 0 if j[2] else 1)      # long instantiation TUs first
    objs = [j[1] for j in jobs_]
    # tuning variants: PFPL_VARIANT_ONLY="enc_0_0,dec_0_0" recompiles only those
    # instantiations (plus the host files); the rest are linked from build/
    only = os.environ.get("PFPL_VARIANT_ONLY")
    if extra and only:
        keep = set(only.split(","))
        base = os.path.join(ROOT, "build")
        objs = [o if (not j[2] or os.path.basename(o)[:-2] in keep) else os.path.join(base, os.path.basename(o))
                for j, o in zip(jobs_, objs)]
        jobs_ = [j for j in jobs_ if not j[2] or os.path.basename(j[1])[:-2] in keep]
    running, pending = [], list(jobs_)
    while pending or running:
        while pending and len(running) < max(1, jobs):
            src, obj, defs = pending.pop(0)
            cmd = [nvcc(), *NVCC_FLAGS, *extra, *defs, "-I", os.path.join(ROOT, "include"), "-c", src, "-o", obj]
            log = open(obj + ".log", "w")
            running.append((subprocess.Popen(cmd, stdout=log, stderr=subprocess.STDOUT), cmd, obj))
        p, cmd, obj = running.pop(0)
        if p.wait() != 0:
            for q, _, _ in running:
                q.kill()
            raise RuntimeError("nvcc failed: " + " ".join(cmd) + "\n" + open(obj + ".log").read())
        if verbose:
            print(open(obj + ".log").read())
    tmp = lib + ".tmp"
    subprocess.run([nvcc(), "-shared", "-gencode", "arch=compute_100a,code=sm_100a", *objs,
                    "-o", tmp], check=True)
    os.replace(tmp, lib)
    return lib


CPU_SRC = os.path.join(PKG, "cpu", "pfpl_cpu.c")
CPU_LIB = os.path.join(PKG, "libpfpl_cpu.so")
# the multi-core CPU codec: x86-64-v3 (AVX2, BMI2) + OpenMP; IEEE-strict
# floating point (no contraction) so its streams are bit-identical to the GPU's
CPU_FLAGS = ["-O3", "-march=x86-64-v3", "-std=c11", "-fPIC", "-shared", "-fopenmp",
             "-ffp-contract=off", "-fno-fast-math", "-Wall", "-Wno-unused-parameter"]


def build_cpu(force: bool = False) -> str:
    deps = [CPU_SRC, os.path.join(ROOT, "include", "pfpl_cpu.h")]
    if force or not os.path.exists(CPU_LIB) or any(os.path.getmtime(d) > os.path.getmtime(CPU_LIB) for d in deps):
        tmp = CPU_LIB + ".tmp"
        subprocess.run(["gcc", *CPU_FLAGS, CPU_SRC, "-o", tmp, "-lm"], check=True)
        os.replace(tmp, CPU_LIB)
    return CPU_LIB


if __name__ == "__main__":
    import sys
    if len(sys.argv) > 2:      # _build.py OUT.so -DFLAG ...   (tuning variants)
        print(build(force=True, out=os.path.join(PKG, sys.argv[1]), extra=sys.argv[2:]))
    else:
        build(force=True, verbose=True)
        print(LIB)
