mkdir -p gpurun_out
for rep in 1 2; do
for v in default $VARIANTS; do
  if [ $v = default ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_$v.so; fi
  DEDUP_LIB=$L timeout 300 python bench.py --steps 600 --warmup 8 --step-only > gpurun_out/ab15_${v}_$rep.log 2>&1
done
done
DEDUP_LIB=build/variants/libdedup_mb2.so MB=1000 CASES=uniform,real timeout 300 python tools/sha_sizes.py > gpurun_out/ab15_sha_mb2.log 2>&1
echo done
