# Profiles committed under profiles/: launch list of the bench command and one
# ncu --set full capture of the hot kernels (one 64 MiB batch of C2).
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/bench_launches.csv python bench.py --steps 6 --warmup 3 --step-only > gpurun_out/bench_under_ncu.log 2>&1
BATCH_MB=64 NBATCH=3 timeout 900 ncu --set full --clock-control none --import-source on -k regex:"rabin_scan_agg2|select_emit_ev|sha1_kernel|table_insert" -s 4 -c 4 -o gpurun_out/prof_full -f python tools/one_batch.py > gpurun_out/ncu_full.log 2>&1

timeout 300 ncu --set full --clock-control none --import-source on -k regex:findmatch -s 1 -c 1 -o gpurun_out/prof_fm -f python tools/fm_sizes.py > gpurun_out/ncu_fm.log 2>&1
echo done
