timeout 1500 python -m pytest tests/ -m gpu -x -q > gpurun_out/pytest_all.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_all.log
timeout 300 python bench.py --steps 20 --warmup 5 > gpurun_out/bench20.json 2> gpurun_out/bench20.err
timeout 300 python bench.py --steps 300 --warmup 5 --step-only > gpurun_out/bench300.json 2>&1
echo fin
