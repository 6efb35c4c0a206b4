#!/bin/bash
# on the GPU box: f32 ABS NYX table for each variant library given (twice, interleaved)
mkdir -p gpurun_out
for rep in 1 2; do
for v in "$@"; do
  echo "== $v"; PFPL_LIB=$v timeout 300 python tools/bench_all.py ${VAR_CASES:-nyx_abs nyx_rough_abs cesm_abs} 2>&1 | grep "^| [A-Z]"
done; done
