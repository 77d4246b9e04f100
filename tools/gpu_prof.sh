mkdir -p gpurun_out
python tools/probe_host.py > gpurun_out/probe_host.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python tools/one_batch.py > gpurun_out/one_batch.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:rabin_scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan -f python tools/one_batch.py > gpurun_out/ncu_scan.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:select_ -s 3 -c 3 -o gpurun_out/prof_select -f python tools/one_batch.py > gpurun_out/ncu_select.log 2>&1
