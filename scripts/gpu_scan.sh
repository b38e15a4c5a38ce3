mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "scan or stream" > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
( for sv in 2 4 8; do echo "== S $sv"; for args in "1024 1024 f64 1 6" "16384 16384 f64 1 6" "256 1048576 f32 1 6" "2048 16384 f64 1 6" "4096 4096 f64 1 6" "512 65536 f32 1 6"; do TRI_SCAN_S=$sv timeout 120 python scripts/prof_one.py $args - 2 | grep -v "^time"; done; done
for args in "16384 16384 f64 0 0" "256 1048576 f32 0 0" "16777216 1 f64 0 0"; do timeout 120 python scripts/prof_one.py $args - 2 | grep -v "^time"; done
) > gpurun_out/scan_times.log 2>&1
