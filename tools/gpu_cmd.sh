mkdir -p gpurun_out
nvcc -o /tmp/psb tools/probe_smem_base.cu && /tmp/psb > gpurun_out/probe_smem.txt 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stream.py tests/test_gpu_maxchunk.py tests/test_gpu_fullsize.py -x -q > gpurun_out/pytest_new.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_new.log
for rep in 1 2; do for lib in paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so build/ab/fused.so; do
  echo "== $lib" >> gpurun_out/ab.log
  DEDUP_LIB=$lib timeout 300 python bench.py --steps 300 --warmup 5 --step-only 2>&1 | cut -c1-200 >> gpurun_out/ab.log
  if [ $rep = 1 ]; then DEDUP_LIB=$lib timeout 300 python tools/kern_rates.py >> gpurun_out/ab.log 2>&1; fi
done; done
echo fin
