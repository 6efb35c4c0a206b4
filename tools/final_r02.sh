#!/bin/bash
# round-2 final pass on the GPU box: full GPU tests, smoke, bench line (N=1 and the 2-rank
# shared-GPU run), all-config table incl. the 16 GiB field, ncu captures (NYX encoder/decoder,
# Hurricane REL encoder, 16 GiB encoder in its split form, bench launch list)
mkdir -p gpurun_out
(timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/fin_tests.log 2>&1; echo "pytest rc=$?" >> gpurun_out/fin_tests.log)
tail -2 gpurun_out/fin_tests.log
(timeout 300 python __graft_entry__.py smoke > gpurun_out/fin_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/fin_smoke.log)
tail -1 gpurun_out/fin_smoke.log
timeout 600 python bench.py > gpurun_out/fin_bench.log 2>&1; echo "bench rc=$?"
timeout 900 python bench.py --gpus 2 --steps 3 --warmup 3 > gpurun_out/fin_bench2.log 2>&1; echo "bench2 rc=$?"
timeout 600 python tools/bench_all.py > gpurun_out/fin_bench_all.log 2>&1; grep "^|" gpurun_out/fin_bench_all.log
timeout 600 python tools/bench_all.py big > gpurun_out/fin_bench_big.log 2>&1; grep "^| [0-9A-Z]" gpurun_out/fin_bench_big.log
bash tools/prof_r02.sh > /dev/null 2>&1
ncu --set full --import-source on --clock-control none --cache-control none -k regex:"encode_kernel" -s 3 -c 1 -f -o gpurun_out/r02_enc_big python tools/prof_run.py --config big16g --iters 5 --what enc > gpurun_out/r02_enc_big.log 2>&1
ls gpurun_out | head -40
