# GPU call: SHA-1 FMA-select variant A/B + sanitizers over the round-2 code.
mkdir -p gpurun_out
rm -f gpurun_out/ab.log
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for lib in paper_conf_ipps_rockenbachsgmtd19_b200/libdedup_b200.so build/ab/sha_fmasel.so; do
  echo "== $lib" >> gpurun_out/ab.log
  DEDUP_LIB=$lib MB=672 CASES=uniform,real REPS=5 timeout 300 python tools/sha_sizes.py >> gpurun_out/ab.log 2>&1
  DEDUP_LIB=$lib timeout 300 python bench.py --steps 200 --warmup 5 --step-only 2>&1 | cut -c1-160 >> gpurun_out/ab.log
  DEDUP_LIB=$lib timeout 300 python -c "
import bench, synthgen, numpy as np, json
d = synthgen.config_stream('C3'); off = synthgen.split_items(d)
import torch
r = bench.int_rates(); dd = torch.from_numpy(d).cuda()
k = bench.isolated_kernels(dd, off, bench.sha1_peak(r), r['lop3'])
print(json.dumps({'sha1': k['sha1']['input_gbs'], 'frac': k['sha1']['frac']}))" >> gpurun_out/ab.log 2>&1
done
bash tools/gpu_sanitize.sh
echo done
