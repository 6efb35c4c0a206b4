#!/bin/bash
# round 2, on the GPU box: gpu tests, smoke, bench, sanitizers.
# racecheck / synccheck run on libpfpl_race.so (built with -DPFPL_LANE_ARRIVE=1: every
# compute lane arrives on the IO-queue barrier itself, the form racecheck can follow;
# the production build arrives once per warp after __syncwarp, which orders the lanes'
# writes under the CUDA memory model but is not modelled by racecheck)
mkdir -p gpurun_out
(timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t.log)
tail -3 gpurun_out/t.log
timeout 120 python __graft_entry__.py smoke 2>&1 | tail -1
timeout 300 python bench.py > gpurun_out/bench.log 2>&1; tail -1 gpurun_out/bench.log | cut -c1-300
if [ "${SAN:-1}" = "1" ]; then
  CS=/usr/local/cuda/bin/compute-sanitizer
  for tool in racecheck synccheck memcheck; do
    LIB=libpfpl.so; [ $tool != memcheck ] && LIB=libpfpl_race.so
    (PFPL_LIB=$LIB PFPL_GRID_LIMIT=8 timeout 1200 $CS --tool $tool --print-limit 20 python tools/sanitize_cases.py --small > gpurun_out/san_$tool.log 2>&1; echo "rc=$? lib=$LIB" >> gpurun_out/san_$tool.log)
    tail -3 gpurun_out/san_$tool.log
  done
  (timeout 1800 $CS --tool memcheck --print-limit 20 python tools/sanitize_cases.py --fuzz 200 --mb 100 > gpurun_out/san_fuzz.log 2>&1; echo "rc=$?" >> gpurun_out/san_fuzz.log)
  tail -3 gpurun_out/san_fuzz.log
fi
