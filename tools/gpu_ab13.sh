mkdir -p gpurun_out
for v in default $VARIANTS; do
  if [ $v = default ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_$v.so; fi
  DEDUP_LIB=$L timeout 300 python tools/sweep_only.py > gpurun_out/ab13_$v.log 2>&1
done
echo done
