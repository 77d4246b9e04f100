mkdir -p gpurun_out
DEDUP_LIB=build/variants/libdedup_t1024.so timeout 300 python -m pytest tests -m gpu -x -q -k "C1" > gpurun_out/pytest_t1024.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for v in t512m2 main; do
  if [ $v = main ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_$v.so; fi
  DEDUP_LIB=$L timeout 300 python bench.py --steps 300 --warmup 8 --no-cpu-baseline --e2e-steps 4 > gpurun_out/bench_$v.log 2>&1
done
