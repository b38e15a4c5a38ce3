mkdir -p gpurun_out
timeout 1500 python scripts/sweep_scan.py f64 > gpurun_out/sweep_scan_f64.jsonl 2> gpurun_out/sweep_scan_f64.err
timeout 1500 python scripts/sweep_scan.py f32 > gpurun_out/sweep_scan_f32.jsonl 2> gpurun_out/sweep_scan_f32.err
