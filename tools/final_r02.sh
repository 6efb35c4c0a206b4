#!/bin/bash
# round-2 final pass on the GPU box: full GPU tests, smoke, bench line, all-config table,
# ncu captures (NYX encoder/decoder, Hurricane REL encoder, bench launch list), memcheck
mkdir -p gpurun_out
(timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/fin_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/fin_tests.log)
tail -2 gpurun_out/fin_tests.log
(timeout 300 python __graft_entry__.py smoke > gpurun_out/fin_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/fin_smoke.log)
tail -1 gpurun_out/fin_smoke.log
timeout 600 python bench.py > gpurun_out/fin_bench.log 2>&1; echo "bench rc=$?"
timeout 600 python tools/bench_all.py > gpurun_out/fin_bench_all.log 2>&1; cat gpurun_out/fin_bench_all.log | grep "^|"
bash tools/prof_r02.sh > /dev/null 2>&1
(PFPL_GRID_LIMIT=8 timeout 1200 /usr/local/cuda/bin/compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_cases.py --small > gpurun_out/fin_memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/fin_memcheck.log)
tail -3 gpurun_out/fin_memcheck.log
