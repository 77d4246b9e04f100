# Profiles committed under profiles/ (summaries): launch list of the bench
# step command and one ncu --set full capture of the hot kernels (64 MiB
# batches of C3), plus the isolated SHA-1 launch (tools/sha_sizes.py).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/bench_launches.csv python bench.py --steps 3 --warmup 3 --step-only > gpurun_out/bench_under_ncu.log 2>&1
NBATCH=3 timeout 900 ncu --set full --clock-control none --import-source on -k regex:"rabin_roll|select_tiles|select_emit_ev|sha1_kernel|table_insert|sha_scatter|pack_kernel" -s 6 -c 6 -o gpurun_out/prof_full -f python tools/one_batch.py > gpurun_out/ncu_full.log 2>&1
MB=672 CASES=real REPS=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"sha1_kernel" -s 1 -c 1 -o gpurun_out/prof_sha -f python tools/sha_sizes.py > gpurun_out/ncu_sha.log 2>&1
for r in prof_full prof_sha; do ncu -i gpurun_out/$r.ncu-rep --page raw --csv > gpurun_out/$r.raw.csv 2>/dev/null; done
echo done
