mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
SIZES=64,256 python tools/scan_sizes.py > gpurun_out/scan_ilp2.log 2>&1
DEDUP_LIB=build/variants/libdedup_ilp1.so SIZES=64,256 python tools/scan_sizes.py > gpurun_out/scan_ilp1.log 2>&1
for v in ilp2 ilp1; do
  if [ $v = ilp2 ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_$v.so; fi
  DEDUP_LIB=$L SIZES=256 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/var_$v.csv python tools/scan_sizes.py > /dev/null 2>&1
done
python tools/trace.py 2> gpurun_out/trace_c32.log > /dev/null
