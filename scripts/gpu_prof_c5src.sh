# ncu of the c5 SCAN kernel with source-line attribution (stall samples / instructions per line)
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan -c 1 -f -o gpurun_out/c5_scan python scripts/prof_one.py 16384 16384 f64 0 0 - 1 > gpurun_out/ncu_c5.log 2>&1
python scripts/ncu_summary.py gpurun_out/c5_scan.ncu-rep gpurun_out/ncu_c5_scan.txt >> gpurun_out/ncu_c5.log 2>&1
ncu -i gpurun_out/c5_scan.ncu-rep --page source --csv --print-source sass,cuda > gpurun_out/c5_scan_sc.csv 2>/dev/null
