# GPU call: SHA-1 kernel A/B (old build vs current) on isolated launches, GPU tests, bench.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for lib in build/ab/libdedup_oldsha.so paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; do
  echo "== $lib" >> gpurun_out/sha_ab.log
  DEDUP_LIB=$lib MB=672 CASES=uniform,jitter,real REPS=5 timeout 300 python tools/sha_sizes.py >> gpurun_out/sha_ab.log 2>&1
done
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python bench.py --steps 20 --warmup 5 --step-only > gpurun_out/bench_20.log 2>&1
timeout 300 python bench.py --steps 300 --warmup 5 --step-only > gpurun_out/bench_300.log 2>&1
echo done
