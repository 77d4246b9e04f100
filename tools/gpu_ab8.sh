# bench A/B over library variants and slot counts
mkdir -p gpurun_out
for v in ${BASE-default} $VARIANTS; do
  if [ $v = default ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_$v.so; fi
  for sl in $SLOTSET; do
    DEDUP_LIB=$L timeout 300 python bench.py --steps 400 --warmup 8 --no-cpu-baseline --e2e-steps 4 --slots $sl > gpurun_out/ab_bench_${v}_s$sl.log 2>&1
  done
done
echo done
