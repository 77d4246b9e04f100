mkdir -p gpurun_out
python tools/probe_host.py > gpurun_out/probe_host.log 2>&1
DEDUP_STAGE_EVENTS=0 python tools/probe_host.py > gpurun_out/probe_host_noev.log 2>&1
DEDUP_TIME_EVERY=8 timeout 300 python bench.py --steps 400 --warmup 8 --batch-mb 64 --slots 24 --no-cpu-baseline --e2e-steps 40 > gpurun_out/bench_te8.log 2>&1
DEDUP_STAGE_EVENTS=0 timeout 300 python bench.py --steps 400 --warmup 8 --batch-mb 64 --slots 24 --no-cpu-baseline --e2e-steps 40 > gpurun_out/bench_noev.log 2>&1
