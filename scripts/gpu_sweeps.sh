mkdir -p gpurun_out/sweeps
for dt in f64 f32; do for lay in 0 1; do
  timeout 1500 python scripts/sweep_scan.py $dt $lay > gpurun_out/sweeps/r02b_sweep_scan_${dt}_${lay}.jsonl 2> gpurun_out/sweeps/${dt}_${lay}.err
done; done
