mkdir -p gpurun_out
DEDUP_LIB=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "op_chunk or c1 or adversarial" > gpurun_out/pytest_l1.log 2>&1; echo rc=$? >> gpurun_out/pytest_l1.log
for rep in 1 2; do
for v in default $VARIANTS; do
  if [ $v = default ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_$v.so; fi
  DEDUP_LIB=$L SIZES=256 timeout 120 python tools/scan_sizes.py > gpurun_out/ab14_scan_${v}_$rep.log 2>&1
  DEDUP_LIB=$L timeout 300 python bench.py --steps 600 --warmup 8 --step-only > gpurun_out/ab14_${v}_$rep.log 2>&1
done
done
echo done
