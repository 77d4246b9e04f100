mkdir -p gpurun_out
for v in $PVARIANTS; do
  DEDUP_LIB=build/variants/libdedup_$v.so timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist_loopback.py -x -q > gpurun_out/pytest_$v.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_$v.log
done
VARIANTS="$VARIANTS" bash tools/gpu_ab9.sh
