mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel" -c 1 -f -o gpurun_out/c1_rough python tools/prof_run.py --config nyx_rough --iters 1 --what enc > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel" -c 1 -f -o gpurun_out/c1_hurabs python tools/prof_run.py --config hurricane --bound abs --iters 1 --what enc > /dev/null 2>&1
ls -la gpurun_out/c1_*
