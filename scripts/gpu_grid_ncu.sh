mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan_grid -c 1 -f -o gpurun_out/c2_grid python scripts/prof_one.py 1024 1024 f64 1 0 - 2 > gpurun_out/ncu_c2.log 2>&1
python scripts/ncu_summary.py gpurun_out/c2_grid.ncu-rep gpurun_out/ncu_c2_grid.txt >> gpurun_out/ncu_c2.log 2>&1
ncu -i gpurun_out/c2_grid.ncu-rep --page source --csv --print-source sass > gpurun_out/c2_grid_sass.csv 2>/dev/null
ncu -i gpurun_out/c2_grid.ncu-rep --page source --csv --print-source cuda > gpurun_out/c2_grid_cuda.csv 2>/dev/null
