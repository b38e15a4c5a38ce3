mkdir -p gpurun_out
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 1500 python scripts/sweep_scan.py f64 1 > gpurun_out/sweep_scan_il_f64.jsonl 2> gpurun_out/sweep_scan_il_f64.err
timeout 1500 python scripts/sweep_scan.py f32 1 > gpurun_out/sweep_scan_il_f32.jsonl 2> gpurun_out/sweep_scan_il_f32.err
