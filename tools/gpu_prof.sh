mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python tools/one_batch.py > gpurun_out/one_batch.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"rabin_scan|select_agg|select_emit|table_insert|pack" -s 8 -c 5 -o gpurun_out/prof_full -f python tools/one_batch.py > gpurun_out/ncu_full.log 2>&1
CUDA_DEVICE_MAX_CONNECTIONS=32 python tools/trace.py 2> gpurun_out/trace_c32.log > /dev/null
CUDA_DEVICE_MAX_CONNECTIONS=32 timeout 300 python bench.py --steps 400 --warmup 8 --batch-mb 64 --slots 16 --no-cpu-baseline --e2e-steps 40 > gpurun_out/benchc_b64_s16.log 2>&1
