mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "stream" > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
for nm in "16384 2048" "16384 16384"; do timeout 120 python scripts/prof_one.py $nm f64 0 5 - 2; done > gpurun_out/stream_times.log 2>&1
( echo "== mode 0"; timeout 120 python scripts/prof_stream.py 16384 2048 ) > gpurun_out/prof_stream.log 2>&1
