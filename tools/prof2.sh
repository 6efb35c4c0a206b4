mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/p2_nyx python tools/prof_run.py --iters 1 > gpurun_out/p2_nyx.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/p2_rel python tools/prof_run.py --config hurricane --bound rel --iters 1 > gpurun_out/p2_rel.log 2>&1
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel|decode_kernel" -c 2 -f -o gpurun_out/p2_mir python tools/prof_run.py --config miranda --bound abs --eps 1e-4 --iters 1 > gpurun_out/p2_mir.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/b_ncu.log 2>&1
ls -la gpurun_out
