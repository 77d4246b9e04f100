mkdir -p gpurun_out
DEDUP_LIB=build/variants/libdedup_e12.so SIZES=256 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"rabin_scan_agg2" -s 2 -c 1 -o gpurun_out/prof_scan_e12 -f python tools/scan_sizes.py > gpurun_out/ncu_scan_e12.log 2>&1
SIZES=256 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"rabin_scan_agg2" -s 2 -c 1 -o gpurun_out/prof_scan256 -f python tools/scan_sizes.py > gpurun_out/ncu_scan256.log 2>&1
echo done
