# GPU call: A/B of environment settings in the pipeline, interleaved reps:
#   ENVS="DEDUP_X=0 DEDUP_X=1" STEPS=300 REPS=3 bash tools/gpu_envab.sh
mkdir -p gpurun_out
rm -f gpurun_out/envab.log
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for rep in $(seq 1 ${REPS:-3}); do
  for e in ${ENVS}; do
    for st in ${STEPS:-300} 20; do
      echo "$e steps $st $(env $e timeout 300 python bench.py --steps $st --warmup 5 --step-only 2>&1 | grep -o '"value": [0-9.]*')" >> gpurun_out/envab.log
    done
  done
done
echo done
