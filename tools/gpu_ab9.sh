mkdir -p gpurun_out
for v in default $VARIANTS; do
  if [ $v = default ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_$v.so; fi
  DEDUP_LIB=$L MB=1000 CASES=uniform,jitter,real timeout 300 python tools/sha_sizes.py > gpurun_out/ab_sha_$v.log 2>&1
  DEDUP_LIB=$L timeout 300 python bench.py --steps 400 --warmup 8 --no-cpu-baseline --e2e-steps 4 > gpurun_out/ab_bench_$v.log 2>&1
done

echo done
