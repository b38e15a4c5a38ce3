mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "scan" > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
TRI_SCAN_DELTA=3 timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "scan_parity" >> gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
( for dl in 1 4 8 16 24; do echo "=== delta $dl"; for args in "16384 16384 f64 0 6" "2048 16384 f64 0 6" "512 65536 f64 0 6" "1024 32768 f64 0 6" "1024 65536 f32 0 6"; do TRI_SCAN_DELTA=$dl timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done; done
) > gpurun_out/scan_times.log 2>&1
