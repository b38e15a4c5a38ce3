# re-measure the interleaved planner sweeps (and the contiguous ones) with the round-2 kernels
mkdir -p gpurun_out/sw
timeout 1500 python scripts/sweep_scan.py f64 1 > gpurun_out/sw/r02_sweep_scan_f64_1.jsonl 2> gpurun_out/sw/f64_1.err
timeout 1500 python scripts/sweep_scan.py f32 1 > gpurun_out/sw/r02_sweep_scan_f32_1.jsonl 2> gpurun_out/sw/f32_1.err
timeout 1500 python scripts/sweep_scan.py f64 0 > gpurun_out/sw/r02_sweep_scan_f64_0.jsonl 2> gpurun_out/sw/f64_0.err
timeout 1500 python scripts/sweep_scan.py f32 0 > gpurun_out/sw/r02_sweep_scan_f32_0.jsonl 2> gpurun_out/sw/f32_0.err
