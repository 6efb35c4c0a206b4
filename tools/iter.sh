#!/bin/bash
# fast iteration on the GPU box: key parity tests, all-config table, racecheck on the encoder
mkdir -p gpurun_out
T=${TESTS:-"tests/test_gpu_parity.py tests/test_gpu_hardening.py"}
(timeout 900 python -m pytest $T -x -q > gpurun_out/it_t.log 2>&1; echo "pytest rc=$?" >> gpurun_out/it_t.log)
tail -2 gpurun_out/it_t.log
timeout 600 python tools/bench_all.py ${CASES:-} 2>&1 | tail -12
if [ "${RACE:-0}" = "1" ]; then
  (PFPL_GRID_LIMIT=8 timeout 1200 /usr/local/cuda/bin/compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_cases.py --small > gpurun_out/it_race.log 2>&1; echo "rc=$?" >> gpurun_out/it_race.log)
  tail -3 gpurun_out/it_race.log
fi
if [ "${PROF:-0}" = "1" ]; then
  ncu --set full --import-source on --clock-control none -k regex:"encode_kernel" -c 1 -f -o gpurun_out/it_nyx python tools/prof_run.py --iters 1 --what enc > /dev/null 2>&1
  ncu --metrics smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum,sm__warps_active.avg.pct_of_peak_sustained_active --cache-control none --clock-control none -k regex:"encode_kernel" -s 3 -c 2 python tools/prof_run.py --iters 6 --what enc 2>&1 | grep -E "inst_executed|issue_active|duration|warps_active" 
fi
