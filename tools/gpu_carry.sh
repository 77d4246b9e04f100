# GPU call: carry-over mode tests + throughput, regression tests of the engine.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_stream.py tests/test_gpu_parity.py tests/test_gpu_mg.py -x -q > gpurun_out/pytest_carry.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_carry.log
timeout 300 python -c "
import bench, synthgen, json
d = synthgen.config_stream('C3')
print(json.dumps(bench.carry_throughput(d)))
print(json.dumps(bench.carry_throughput(d, piece=16 * 1024 * 1024 + 16)))
" > gpurun_out/carry_tp.log 2>&1
echo done
