VARS="libpfpl_t16.so libpfpl_t32.so" CASES="hurricane miranda_rel" bash tools/ab.sh
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel" -c 1 -f -o gpurun_out/c3_hur python tools/prof_run.py --config hurricane --bound rel --iters 1 --what enc > /dev/null 2>&1
ncu --set full --import-source on --clock-control none -k regex:"encode_kernel" -c 1 -f -o gpurun_out/c3_mir python tools/prof_run.py --config miranda --bound rel --eps 1e-4 --iters 1 --what enc > /dev/null 2>&1
