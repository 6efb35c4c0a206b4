#!/bin/bash
# ncu --set full of the NYX f32 ABS encoder (and decoder), source counters for the per-stage budget
mkdir -p gpurun_out
TAG=${TAG:-r02}
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/${TAG}_nyx python tools/prof_run.py --iters 1 > gpurun_out/${TAG}_nyx.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_b_ncu.log 2>&1
ls -la gpurun_out/${TAG}*
