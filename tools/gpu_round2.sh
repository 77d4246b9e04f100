# GPU call: full bench (driver command) x2, step-only 600, overlap trace, FMASEL repeat A/B.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
timeout 300 python bench.py --steps 600 --warmup 5 --step-only > gpurun_out/bench_600.log 2>&1
timeout 300 python tools/overlap_trace.py > gpurun_out/overlap.txt 2>&1
rm -f gpurun_out/ab2.log
for rep in 1 2 3; do for lib in paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so build/ab/sha_fmasel.so; do
  echo "== $lib" >> gpurun_out/ab2.log
  DEDUP_LIB=$lib timeout 300 python bench.py --steps 20 --warmup 5 --step-only 2>&1 | cut -c100-200 >> gpurun_out/ab2.log
  DEDUP_LIB=$lib timeout 300 python bench.py --steps 300 --warmup 5 --step-only 2>&1 | cut -c100-200 >> gpurun_out/ab2.log
done; done
echo done
