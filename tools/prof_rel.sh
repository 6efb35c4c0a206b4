mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/rel_hur python tools/prof_run.py --config hurricane --bound rel --iters 1 > gpurun_out/rel_hur.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/rel_mir python tools/prof_run.py --config miranda --bound rel --eps 1e-4 --iters 1 > gpurun_out/rel_mir.log 2>&1
ls -la gpurun_out/rel_*
