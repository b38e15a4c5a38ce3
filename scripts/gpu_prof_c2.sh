mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan_il3 -c 1 -f -o gpurun_out/c2_il3 python scripts/prof_one.py 1024 1024 f64 1 0 - 2 > gpurun_out/ncu_c2.log 2>&1
python scripts/ncu_summary.py gpurun_out/c2_il3.ncu-rep gpurun_out/ncu_c2_il3.txt >> gpurun_out/ncu_c2.log 2>&1
ncu -i gpurun_out/c2_il3.ncu-rep --page source --csv --print-source sass > gpurun_out/c2_il3_sass.csv 2>/dev/null
