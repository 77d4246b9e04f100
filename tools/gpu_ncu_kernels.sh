# ncu --set full (source-level) of the scan and SHA-1 kernels in isolation.
mkdir -p gpurun_out
SIZES=64 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"rabin_roll" -s 2 -c 1 -o gpurun_out/prof_scan -f python tools/scan_sizes.py > gpurun_out/ncu_scan.log 2>&1
MB=1024 CASES=uniform REPS=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"sha1_kernel" -s 1 -c 1 -o gpurun_out/prof_sha -f python tools/sha_sizes.py > gpurun_out/ncu_sha.log 2>&1
echo done
