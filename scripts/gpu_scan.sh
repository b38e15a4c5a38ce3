mkdir -p gpurun_out
timeout 1500 python -m pytest tests -q -m gpu --timeout 120 > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
( for args in "16384 16384 f64 0 0" "256 1048576 f32 0 0" "1024 1024 f64 1 0" "16777216 1 f64 0 0"; do timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done ) > gpurun_out/scan_times.log 2>&1
