# GPU call: SHA-1 pipe-balance variants in the pipeline (C3, 300 steps, x2) and isolated.
mkdir -p gpurun_out
rm -f gpurun_out/ab3.log
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "op_sha1" > gpurun_out/pytest_sha.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_sha.log
for rep in 1 2; do for lib in paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so build/ab/sha_nofmasel.so build/ab/sha_rot30.so build/ab/sha_rot1.so; do
  echo "== $lib" >> gpurun_out/ab3.log
  DEDUP_LIB=$lib timeout 300 python bench.py --steps 300 --warmup 5 --step-only 2>&1 | cut -c100-180 >> gpurun_out/ab3.log
  if [ $rep = 1 ]; then DEDUP_LIB=$lib MB=672 CASES=uniform,real REPS=5 timeout 300 python tools/sha_sizes.py >> gpurun_out/ab3.log 2>&1; fi
done; done
echo done
