mkdir -p gpurun_out
for mb in 4 16 64; do
BATCH_MB=$mb NBATCH=3 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$mb.csv python tools/one_batch.py > /dev/null 2>&1
done
