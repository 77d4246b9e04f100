timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stream.py tests/test_gpu_maxchunk.py -x -q > gpurun_out/pytest_sel.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_sel.log
LIBS="build/ab/seltiles_old.so" STEPS=300 REPS=2 ISOLATED="python tools/kern_rates.py" bash tools/gpu_ab.sh
timeout 300 python bench.py --steps 20 --warmup 5 --step-only >> gpurun_out/ab.log 2>&1
NBATCH=3 timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"select_tiles|rabin_roll" --csv python tools/one_batch.py > gpurun_out/sel_ncu.csv 2>&1
echo fin
