mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
CS=/usr/local/cuda/bin/compute-sanitizer
DEDUP_LIB=build/ab/bitmap_old.so timeout 900 $CS --tool memcheck --leak-check no --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -x -q -k "not_a_tile_multiple and single" > gpurun_out/memchk_old.log 2>&1; echo "rc=$?" >> gpurun_out/memchk_old.log
timeout 900 $CS --tool memcheck --leak-check no --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -x -q -k "not_a_tile_multiple" > gpurun_out/memchk_new.log 2>&1; echo "rc=$?" >> gpurun_out/memchk_new.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_mg.py tests/test_gpu_dist_loopback.py -x -q > gpurun_out/pytest_par.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_par.log
