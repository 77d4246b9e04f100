# GPU call: the per-process multi-GPU path at world size 1 with the host
# profile of the wave path (DEDUP_MG_PROFILE=1: per-section host time, one
# table per drained run), plus the multi-GPU GPU tests.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_mg.py tests/test_gpu_dist_loopback.py -x -q > gpurun_out/pytest_mg.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_mg.log
DEDUP_MG_PROFILE=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps ${STEPS:-20} --warmup 5 --no-cpu-baseline > gpurun_out/distprof.log 2>&1; echo "rc=$?" >> gpurun_out/distprof.log
