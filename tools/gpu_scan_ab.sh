# GPU call: scan kernel A/B (r1 kernel cleaned vs + IMAD anchor test), parity, bench.
mkdir -p gpurun_out
rm -f gpurun_out/scan_ab.log
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_maxchunk.py -x -q > gpurun_out/pytest_scan.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_scan.log
for lib in paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so build/ab/scan_mul.so; do
  echo "== $lib" >> gpurun_out/scan_ab.log
  DEDUP_LIB=$lib SIZES=64,672 timeout 300 python tools/scan_sizes.py >> gpurun_out/scan_ab.log 2>&1
  DEDUP_LIB=$lib timeout 300 python bench.py --steps 20 --warmup 5 --step-only 2>&1 | cut -c1-200 >> gpurun_out/scan_ab.log
  DEDUP_LIB=$lib timeout 300 python bench.py --steps 200 --warmup 5 --step-only 2>&1 | cut -c1-200 >> gpurun_out/scan_ab.log
done
echo done
