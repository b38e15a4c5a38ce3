mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -q -k "scan" > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
( for args in "256 1048576 f32 0 0" "16384 16384 f64 0 0" "16384 9472 f32 0 0"; do timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done ) > gpurun_out/scan_times.log 2>&1
