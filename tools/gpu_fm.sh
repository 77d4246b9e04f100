mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_findmatch.py -x -q > gpurun_out/pytest_fm.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_fm.log
timeout 300 python tools/fm_sizes.py > gpurun_out/fm_sizes.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:findmatch -s 1 -c 1 -o gpurun_out/prof_fm -f python tools/fm_sizes.py > gpurun_out/ncu_fm.log 2>&1
for v in default $VARIANTS; do
  if [ $v = default ]; then L=paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so; else L=build/variants/libdedup_$v.so; fi
  DEDUP_LIB=$L timeout 300 python bench.py --steps 400 --warmup 8 --no-cpu-baseline --e2e-steps 4 > gpurun_out/ab_bench_$v.log 2>&1
done
echo done
