# compute-sanitizer over the GPU parity tests (SURVEY 4.3 "Sanitizers"):
# memcheck on op-level, engine (single + multi-GPU copy transport), carry-over
# and NEXT-row tests; racecheck / synccheck on the shared-memory kernels.
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
export CUDA_DEVICE_MAX_CONNECTIONS=8
timeout 1500 $CS --tool memcheck --leak-check no --error-exitcode 9 python -m pytest tests/test_gpu_parity.py -x -q -k "op_sha1 or op_chunk_edge or not_a_tile_multiple or (all_zero and single) or (c1_bit_exact_device and (single or copy2)) or (tiny_and_empty and (single or copy2)) or (adversarial and single)" > gpurun_out/san_memcheck.log 2>&1; echo "memcheck rc=$?" >> gpurun_out/san_memcheck.log
timeout 1500 $CS --tool memcheck --leak-check no --error-exitcode 9 python -m pytest tests/test_gpu_stream.py tests/test_gpu_mg.py -x -q -k "host_fed or device_streams or join or all_duplicate" > gpurun_out/san_memcheck3.log 2>&1; echo "memcheck3 rc=$?" >> gpurun_out/san_memcheck3.log
timeout 900 $CS --tool memcheck --error-exitcode 9 python -m pytest tests/test_gpu_findmatch.py tests/test_gpu_mandel.py -x -q -k "random_starts or runs_and_dense or skip or rows_whole_image or image_pipeline" > gpurun_out/san_memcheck2.log 2>&1; echo "memcheck2 rc=$?" >> gpurun_out/san_memcheck2.log
timeout 1200 $CS --tool racecheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py tests/test_gpu_findmatch.py -x -q -k "op_chunk_edge or op_sha1_single or runs_and_dense" > gpurun_out/san_racecheck.log 2>&1; echo "racecheck rc=$?" >> gpurun_out/san_racecheck.log
timeout 900 $CS --tool synccheck --error-exitcode 9 python -m pytest tests/test_gpu_parity.py tests/test_gpu_findmatch.py -x -q -k "op_chunk_edge or op_sha1_single or runs_and_dense" > gpurun_out/san_synccheck.log 2>&1; echo "synccheck rc=$?" >> gpurun_out/san_synccheck.log
echo done
