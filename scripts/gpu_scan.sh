mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_parity_gpu.py -q -k "scan_mc or sliced" --timeout 120 -x > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
( for rep in 1 2; do for w in 3 0; do echo "== w128 $w"; for args in "16777216 1 f64 0 0" "16777216 1 f32 0 0" "65536 16 f64 0 0"; do TRI_SCAN_W128=$w timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done; done; done ) > gpurun_out/scan_times.log 2>&1
