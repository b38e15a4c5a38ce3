mkdir -p gpurun_out
( for dl in 1 2 4 8; do echo "== delta $dl"; for args in "1024 1024 f64 1 0" "2048 2048 f64 1 0" "1024 4096 f64 1 0" "16384 2048 f64 0 0"; do TRI_SCAN_DELTA=$dl timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done; done ) > gpurun_out/scan_times.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan_mc -c 3 -f -o gpurun_out/c3_scanmc_full python scripts/prof_one.py 16777216 1 f64 0 0 - 1 > gpurun_out/ncu_c3.log 2>&1
python scripts/ncu_summary.py gpurun_out/c3_scanmc_full.ncu-rep gpurun_out/ncu_c3_scanmc.txt >> gpurun_out/ncu_c3.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan -c 1 -f -o gpurun_out/c2_scanil_full python scripts/prof_one.py 1024 1024 f64 1 0 - 1 > gpurun_out/ncu_c2.log 2>&1
python scripts/ncu_summary.py gpurun_out/c2_scanil_full.ncu-rep gpurun_out/ncu_c2_scanil.txt >> gpurun_out/ncu_c2.log 2>&1
