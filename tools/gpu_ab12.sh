mkdir -p gpurun_out
DEDUP_LIB=build/variants/libdedup_$V.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "sha1 or c1 or adversarial or full_size" > gpurun_out/pytest_$V.log 2>&1; echo rc=$? >> gpurun_out/pytest_$V.log
for rep in 1 2; do
for v in default $V; do
  if [ $v = default ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_$v.so; fi
  DEDUP_LIB=$L MB=1000 CASES=uniform,jitter,real timeout 300 python tools/sha_sizes.py > gpurun_out/ab12_sha_${v}_$rep.log 2>&1
  DEDUP_LIB=$L timeout 300 python bench.py --steps 600 --warmup 8 --step-only > gpurun_out/ab12_${v}_$rep.log 2>&1
done
done
echo done
