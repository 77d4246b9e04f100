mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_findmatch.py -x -q > gpurun_out/pytest_fm.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_fm.log
timeout 300 python tools/fm_sizes.py > gpurun_out/fm_sizes.log 2>&1
timeout 300 python bench.py --steps 400 --warmup 8 --no-cpu-baseline --e2e-steps 4 > gpurun_out/bench.log 2>&1
echo done
