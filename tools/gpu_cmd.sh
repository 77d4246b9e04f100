rm -f gpurun_out/knobs.log
for rep in 1 2 3; do
  for cfg in "--sha-lane 32768" "--sha-lane 16384" "--sha-lane 8192" "--sha-lane 16384 --slots 56"; do
  echo "== $cfg" >> gpurun_out/knobs.log; timeout 300 python bench.py --steps 20 --warmup 5 --step-only $cfg 2>&1 | cut -c1-150 >> gpurun_out/knobs.log
  done
done
for cfg in "--sha-lane 32768" "--sha-lane 16384"; do echo "== 300 $cfg" >> gpurun_out/knobs.log; timeout 300 python bench.py --steps 300 --warmup 5 --step-only $cfg 2>&1 | cut -c1-150 >> gpurun_out/knobs.log; done
echo fin
