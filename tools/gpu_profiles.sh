mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/bench_launches.csv python bench.py --steps 4 --warmup 3 --e2e-steps 4 --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:"rabin_scan_agg|sha1_kernel|select_emit|table_insert" -s 9 -c 4 -o gpurun_out/prof_r01 -f python tools/one_batch.py > gpurun_out/ncu_r01.log 2>&1
