#!/bin/bash
# ncu --set full (source counters) of the encoder+decoder on NYX ABS, Hurricane REL, Miranda f64 REL
mkdir -p gpurun_out
TAG=${TAG:-cur}
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/${TAG}_nyx python tools/prof_run.py --iters 1 > gpurun_out/${TAG}_nyx.log 2>&1
if [ "${REL:-1}" = "1" ]; then
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/${TAG}_hur python tools/prof_run.py --config hurricane --bound rel --iters 1 > gpurun_out/${TAG}_hur.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/${TAG}_mir python tools/prof_run.py --config miranda --bound rel --eps 1e-4 --iters 1 > gpurun_out/${TAG}_mir.log 2>&1
fi
ls -la gpurun_out/${TAG}_*
