timeout 1200 python -m pytest tests/test_gpu_mg.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_p2p.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_p2p.log
echo fin
