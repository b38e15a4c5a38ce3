mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_parity_gpu.py -q -k "scan and not mc and not interleaved and not batched" --timeout 120 -x > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
( for rep in 1 2; do for pr in 1 0; do echo "== pair $pr"; for args in "256 1048576 f32 0 0" "200 1048576 f32 0 0" "256 65535 f32 0 0"; do TRI_SCAN_PAIR=$pr timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done; done; done ) > gpurun_out/scan_times.log 2>&1
