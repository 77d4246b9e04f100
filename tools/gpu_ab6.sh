mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
DEDUP_LIB=build/variants/libdedup_tma.so timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_tma.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_tma.log
timeout 600 python bench.py > gpurun_out/bench_full.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_full.log
for v in $VARIANTS; do
  L=build/variants/libdedup_$v.so
  DEDUP_LIB=$L SIZES=64,256 timeout 120 python tools/scan_sizes.py > gpurun_out/ab_scan_$v.log 2>&1
  DEDUP_LIB=$L timeout 300 python bench.py --steps 400 --warmup 8 --no-cpu-baseline --e2e-steps 4 > gpurun_out/ab_bench_$v.log 2>&1
done
SIZES=64,256 timeout 120 python tools/scan_sizes.py > gpurun_out/ab_scan_default.log 2>&1
echo done
