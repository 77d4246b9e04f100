mkdir -p gpurun_out
for rep in 1 2; do
for v in default $VARIANTS; do
  if [ $v = default ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_$v.so; fi
  DEDUP_LIB=$L timeout 300 python bench.py --steps 600 --warmup 8 --step-only > gpurun_out/ab11_${v}_$rep.log 2>&1
done
done
for sl in 32 48 64; do timeout 300 python bench.py --steps 600 --warmup 8 --step-only --slots $sl > gpurun_out/ab11_slots$sl.log 2>&1; done
echo done
