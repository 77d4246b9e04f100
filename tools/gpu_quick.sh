mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python tools/one_batch.py > gpurun_out/one_batch.log 2>&1
python tools/trace.py 2> gpurun_out/trace_c32.log > /dev/null
timeout 300 python bench.py --steps 400 --warmup 8 --no-cpu-baseline --e2e-steps 40 > gpurun_out/bench_b64_s24.log 2>&1
