mkdir -p gpurun_out
for v in pf2 ex1 ex2 ex3; do
  DEDUP_LIB=build/variants/libdedup_$v.so SIZES=256 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/var_$v.csv python tools/scan_sizes.py > /dev/null 2>&1
done
