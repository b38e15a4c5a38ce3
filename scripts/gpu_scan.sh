mkdir -p gpurun_out
TRI_SCAN_S=16 timeout 600 python -m pytest tests/test_parity_gpu.py -q -k "interleaved or batched" --timeout 120 -x > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
( for sv in 8 16; do echo "== S $sv"; for args in "1024 1024 f32 1 6" "1024 1024 f64 1 6" "256 16384 f32 1 6" "4096 4096 f32 1 6" "4096 4096 f64 1 6" "2048 16384 f64 1 6"; do TRI_SCAN_S=$sv timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done; done ) > gpurun_out/scan_times.log 2>&1
