# ncu capture of the SCAN kernel at the c5 shape (one launch), plus a summary
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan -c 1 -f -o gpurun_out/scan_c5 \
  python scripts/prof_one.py 16384 16384 f64 0 6 - 1 > gpurun_out/ncu_scan_c5.log 2>&1
python scripts/ncu_summary.py gpurun_out/scan_c5.ncu-rep gpurun_out/ncu_scan_c5.txt >> gpurun_out/ncu_scan_c5.log 2>&1
