mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:"rabin_scan_agg" -s 2 -c 1 -o gpurun_out/prof_scan2 -f python tools/one_batch.py > gpurun_out/ncu_scan2.log 2>&1
