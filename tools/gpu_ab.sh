# GPU call: A/B of library variants in the pipeline.  Build the variants first
# (python tools/build_variant.py NAME -DX=1 ... -> build/ab/NAME.so), then
#   LIBS="build/ab/a.so build/ab/b.so" STEPS=300 REPS=2 bash tools/gpu_ab.sh
# Each rep runs the C3 step-only bench for the default library and every
# variant back to back (interleaved, so clock drift hits all alike);
# ISOLATED="cmd" runs once per library in the first rep (e.g. tools/scan_sizes.py).
mkdir -p gpurun_out
rm -f gpurun_out/ab.log
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/pytest_ab.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ab.log
for rep in $(seq 1 ${REPS:-2}); do
  for lib in paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so ${LIBS:-}; do
    echo "== $lib" >> gpurun_out/ab.log
    DEDUP_LIB=$lib timeout 300 python bench.py --steps ${STEPS:-300} --warmup 5 --step-only 2>&1 | cut -c1-200 >> gpurun_out/ab.log
    if [ $rep = 1 ] && [ -n "${ISOLATED:-}" ]; then DEDUP_LIB=$lib timeout 300 bash -c "$ISOLATED" >> gpurun_out/ab.log 2>&1; fi
  done
done
echo done
