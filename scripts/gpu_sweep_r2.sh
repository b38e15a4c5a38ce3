# r02 planner sweeps (SCAN_MC included) + ncu of the c4 kernel after the fp64-scan change
mkdir -p gpurun_out
for dt in f64 f32; do for lay in 0 1; do
  timeout 1200 python scripts/sweep_scan.py $dt $lay > gpurun_out/r02_sweep_scan_${dt}_${lay}.jsonl 2> gpurun_out/sweep_${dt}_${lay}.err
done; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan -c 1 -f -o gpurun_out/c4_scan_full python scripts/prof_one.py 256 1048576 f32 0 0 - 1 > gpurun_out/ncu_c4.log 2>&1
python scripts/ncu_summary.py gpurun_out/c4_scan_full.ncu-rep gpurun_out/ncu_c4_scan.txt >> gpurun_out/ncu_c4.log 2>&1
