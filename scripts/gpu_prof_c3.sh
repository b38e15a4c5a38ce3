# c3 SCAN_MC: ncu full of the look-back kernel (+ source-level stalls)
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k k_scan_mc_lb -c 1 -f -o gpurun_out/c3_lb_full python scripts/prof_one.py 16777216 1 f64 0 7 - 2 > gpurun_out/ncu_c3.log 2>&1
python scripts/ncu_summary.py gpurun_out/c3_lb_full.ncu-rep gpurun_out/ncu_c3_lb.txt >> gpurun_out/ncu_c3.log 2>&1
ncu -i gpurun_out/c3_lb_full.ncu-rep --page source --csv > gpurun_out/c3_lb_source.csv 2>/dev/null
