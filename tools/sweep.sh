mkdir -p gpurun_out
set -x
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
for cfg in "32 16" "32 32" "16 32" "64 16" "8 48"; do
  set -- $cfg
  timeout 300 python bench.py --steps 400 --warmup 8 --batch-mb $1 --slots $2 --no-cpu-baseline --e2e-steps 40 > gpurun_out/bench_b$1_s$2.log 2>&1
done
