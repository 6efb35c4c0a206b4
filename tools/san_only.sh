#!/bin/bash
# compute-sanitizer pass only (see tools/r2_check.sh)
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in ${TOOLS:-racecheck synccheck memcheck}; do
  LIB=libpfpl.so; [ $tool != memcheck ] && LIB=libpfpl_race.so
  (PFPL_LIB=$LIB PFPL_GRID_LIMIT=8 timeout 1200 $CS --tool $tool --print-limit 20 python tools/sanitize_cases.py --small > gpurun_out/san_$tool.log 2>&1; echo "rc=$? lib=$LIB" >> gpurun_out/san_$tool.log)
  tail -3 gpurun_out/san_$tool.log
done
