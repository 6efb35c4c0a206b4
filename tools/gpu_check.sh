#!/bin/bash
# on the GPU box: gpu tests, smoke, bench line and the all-config table
mkdir -p gpurun_out
(timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t.log)
tail -3 gpurun_out/t.log
timeout 120 python __graft_entry__.py smoke 2>&1 | tail -1
timeout 300 python bench.py > gpurun_out/bench.log 2>&1; tail -1 gpurun_out/bench.log
timeout 600 python tools/bench_all.py > gpurun_out/bench_all.log 2>&1; cat gpurun_out/bench_all.log
