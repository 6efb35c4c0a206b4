mkdir -p gpurun_out
for v in libpfpl.so libpfpl_t4.so; do
PFPL_LIB=$v ncu --set full --import-source on --clock-control none --cache-control none -k regex:"encode_kernel" -s 3 -c 1 -f -o gpurun_out/v_${v%.so} python tools/prof_run.py --iters 5 --what enc > /dev/null 2>&1
done
ls gpurun_out/v_*
