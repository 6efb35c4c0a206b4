mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/p_nyx python tools/prof_run.py --iters 1 > gpurun_out/p_nyx.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/p_rel python tools/prof_run.py --config hurricane --bound rel --iters 1 > gpurun_out/p_rel.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel|minmax" -c 4 -f -o gpurun_out/p_noa python tools/prof_run.py --bound noa --iters 1 > gpurun_out/p_noa.log 2>&1
ls -la gpurun_out
