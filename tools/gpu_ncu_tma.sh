mkdir -p gpurun_out
DEDUP_LIB=build/variants/libdedup_tma.so SIZES=256 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"rabin_scan_agg2" -s 2 -c 1 -o gpurun_out/prof_scan_tma -f python tools/scan_sizes.py > gpurun_out/ncu_scan_tma.log 2>&1
SIZES=256 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"rabin_scan_agg2|select_emit_ev" -s 4 -c 2 -o gpurun_out/prof_scan_cur -f python tools/scan_sizes.py > gpurun_out/ncu_scan_cur.log 2>&1
echo done
