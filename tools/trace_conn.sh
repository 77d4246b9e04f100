mkdir -p gpurun_out
CUDA_DEVICE_MAX_CONNECTIONS=32 python tools/trace.py 2> gpurun_out/trace_c32.log > /dev/null
CUDA_DEVICE_MAX_CONNECTIONS=32 SLOTS=32 BATCH_MB=32 python tools/trace.py 2> gpurun_out/trace_c32_b32.log > /dev/null
for cfg in "64 16" "32 32" "16 48"; do
  set -- $cfg
  CUDA_DEVICE_MAX_CONNECTIONS=32 timeout 300 python bench.py --steps 400 --warmup 8 --batch-mb $1 --slots $2 --no-cpu-baseline --e2e-steps 40 > gpurun_out/benchc_b$1_s$2.log 2>&1
done
