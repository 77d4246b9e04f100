# Pipe attribution of the integer opcodes (microbench) and of the SHA-1 / scan
# kernels, the isolated SHA-1 rate vs grid size, and the driver's bench command.
mkdir -p gpurun_out
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o /tmp/mbp tools/microbench_pipes.cu
/tmp/mbp > gpurun_out/pipes.txt 2>&1
M=sm__inst_executed_pipe_alu.sum,sm__inst_executed_pipe_fma.sum,sm__inst_executed_pipe_fmaheavy.sum,sm__inst_executed_pipe_fmalite.sum,sm__inst_executed.sum,sm__cycles_active.avg,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active,sm__pipe_fmalite_cycles_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum
timeout 300 ncu --metrics $M --csv /tmp/mbp > gpurun_out/pipes_ncu.csv 2>&1
for L in 32768 8192 4096; do MB=672 CASES=real REPS=3 LANE=$L timeout 300 python tools/sha_sizes.py >> gpurun_out/sha_lane.txt 2>&1; done
MB=672 CASES=real REPS=1 LANE=4096 timeout 300 ncu --metrics $M --csv -k regex:sha1_kernel -s 1 -c 1 python tools/sha_sizes.py > gpurun_out/sha_ncu.csv 2>&1
NBATCH=2 timeout 300 ncu --metrics $M --csv -k regex:"rabin_roll|sha1_kernel" -s 2 -c 2 python tools/one_batch.py > gpurun_out/batch_ncu.csv 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench20.json 2> gpurun_out/bench20.err
echo done
