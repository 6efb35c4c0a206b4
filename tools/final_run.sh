#!/bin/bash
# on the GPU box: gpu tests, smoke, bench line, all-config table, eval grid, ncu captures and launch list
mkdir -p gpurun_out
(timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/tf.log 2>&1; echo "pytest rc=$?" >> gpurun_out/tf.log)
timeout 120 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1
timeout 300 python bench.py > gpurun_out/benchf.log 2>&1
timeout 600 python tools/bench_all.py > gpurun_out/bench_allf.log 2>&1
timeout 900 python tools/eval_grid.py > gpurun_out/gridf.log 2>&1; cp profiles/r01_eval_grid.* gpurun_out/ 2>/dev/null
bash tools/prof2.sh
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"encode|decode|scan|minmax|derive|header" --csv --log-file gpurun_out/cesm_launches.csv python tools/prof_run.py --config cesm --iters 3 > gpurun_out/cesm.log 2>&1
