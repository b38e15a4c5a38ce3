mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan1_r16 -c 1 -f -o gpurun_out/c4_r16 python scripts/prof_one.py 256 1048576 f32 0 0 - 1 > gpurun_out/ncu_c4.log 2>&1
python scripts/ncu_summary.py gpurun_out/c4_r16.ncu-rep gpurun_out/ncu_c4_r16.txt >> gpurun_out/ncu_c4.log 2>&1
ncu -i gpurun_out/c4_r16.ncu-rep --page source --csv --print-source sass > gpurun_out/c4_r16_sass.csv 2>/dev/null
ncu -i gpurun_out/c4_r16.ncu-rep --page raw --csv > gpurun_out/c4_r16_raw.csv 2>/dev/null
