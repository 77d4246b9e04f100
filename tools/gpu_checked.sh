# Checked build (DEDUP_CHECK: device-side bounds checks in the roll, selection,
# SHA-1 and p2p table kernels, a trap with the failed condition printed) over
# the GPU test suites -- compute-sanitizer is closed on the GPU pool.
#   python tools/build_variant.py checked -DDEDUP_CHECK; bash tools/gpu_checked.sh
mkdir -p gpurun_out
DEDUP_LIB=build/ab/checked.so timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stream.py tests/test_gpu_mg.py tests/test_gpu_maxchunk.py tests/test_gpu_fullsize.py tests/test_gpu_dist_loopback.py -q > gpurun_out/checked.log 2>&1; echo "checked rc=$?" >> gpurun_out/checked.log
echo done
