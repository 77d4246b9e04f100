# Profiles committed under profiles/ (summaries): launch list of the bench
# step command and one ncu --set full capture of the hot kernels (64 MiB
# batches of C3), plus the isolated SHA-1 launch (tools/sha_sizes.py) and the
# roll kernel over the whole stream (tools/scan_sizes.py).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
PM=sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fmaheavy.sum,sm__inst_executed_pipe_lsu.sum
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 800 --csv --log-file gpurun_out/bench_launches.csv python bench.py --steps 3 --warmup 3 --step-only > gpurun_out/bench_under_ncu.log 2>&1
NBATCH=3 timeout 900 ncu --set full --metrics $PM --clock-control none --import-source on -k regex:"rabin_roll|select_tiles|select_emit_ev|sha1_kernel|table_insert|sha_scatter|pack_kernel" -s 7 -c 7 -o gpurun_out/prof_full -f python tools/one_batch.py > gpurun_out/ncu_full.log 2>&1
MB=672 CASES=real REPS=1 timeout 600 ncu --set full --metrics $PM --clock-control none --import-source on -k regex:"sha1_kernel" -s 1 -c 1 -o gpurun_out/prof_sha -f python tools/sha_sizes.py > gpurun_out/ncu_sha.log 2>&1
SIZES=672 timeout 600 ncu --set full --metrics $PM --clock-control none --import-source on -k regex:"rabin_roll|select_tiles" -s 6 -c 2 -o gpurun_out/prof_roll -f python tools/scan_sizes.py > gpurun_out/ncu_roll.log 2>&1
for r in prof_full prof_sha prof_roll; do ncu -i gpurun_out/$r.ncu-rep --page raw --csv > gpurun_out/$r.raw.csv 2>/dev/null; done
echo done
