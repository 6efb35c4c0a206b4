#!/bin/bash
# round-2 profiles: warm (4th launch, caches not flushed) full-set capture of the NYX
# encoder and decoder for the per-stage budget, the REL encoder, and the launch list
mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none --cache-control none -k regex:"encode_kernel" -s 3 -c 1 -f -o gpurun_out/r02_enc_nyx python tools/prof_run.py --iters 5 --what enc > gpurun_out/r02_enc_nyx.log 2>&1
ncu --set full --import-source on --clock-control none --cache-control none -k regex:"decode_kernel" -s 3 -c 1 -f -o gpurun_out/r02_dec_nyx python tools/prof_run.py --iters 5 > gpurun_out/r02_dec_nyx.log 2>&1
ncu --set full --import-source on --clock-control none --cache-control none -k regex:"encode_kernel" -s 3 -c 1 -f -o gpurun_out/r02_enc_rel python tools/prof_run.py --config hurricane --bound rel --iters 5 --what enc > gpurun_out/r02_enc_rel.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/r02_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/r02_b_ncu.log 2>&1
ls -la gpurun_out/r02_*
