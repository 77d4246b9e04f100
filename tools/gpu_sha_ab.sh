# GPU call: SHA-1 staging variants and pipeline sizing (slots x SHA-1 lane bytes).
mkdir -p gpurun_out
rm -f gpurun_out/sha_ab2.log
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for lib in paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so build/ab/sha_smem4.so build/ab/sha_smem5.so; do
  echo "== $lib" >> gpurun_out/sha_ab2.log
  DEDUP_LIB=$lib MB=672 CASES=uniform,real REPS=5 timeout 300 python tools/sha_sizes.py >> gpurun_out/sha_ab2.log 2>&1
  DEDUP_LIB=$lib timeout 300 python bench.py --steps 200 --warmup 5 --step-only 2>&1 | cut -c1-160 >> gpurun_out/sha_ab2.log
done
for sl in 24 40 56; do for ln in 16384 32768 65536; do
  echo "== slots $sl lane $ln" >> gpurun_out/sha_ab2.log
  timeout 300 python bench.py --steps 200 --warmup 5 --step-only --slots $sl --sha-lane $ln 2>&1 | cut -c1-160 >> gpurun_out/sha_ab2.log
done; done
echo done
