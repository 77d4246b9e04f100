mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/bench_full.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_full.log
for v in $VARIANTS; do
  L=build/variants/libdedup_$v.so
  DEDUP_LIB=$L timeout 300 python bench.py --steps 400 --warmup 8 --no-cpu-baseline --e2e-steps 4 > gpurun_out/ab_bench_$v.log 2>&1
done
for sl in 16 32; do
  timeout 300 python bench.py --steps 400 --warmup 8 --no-cpu-baseline --e2e-steps 4 --slots $sl > gpurun_out/ab_bench_slots$sl.log 2>&1
done
echo done
