mkdir -p gpurun_out
python tools/probe.py > gpurun_out/probe.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python tools/one_batch.py > gpurun_out/one_batch.log 2>&1
