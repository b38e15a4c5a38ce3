mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
for nm in "16384 2048" "16384 16384"; do timeout 120 python scripts/prof_one.py $nm f64 0 5 - 2; done > gpurun_out/stream_times.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_stream -c 1 -o gpurun_out/stream_full5 python scripts/prof_one.py 16384 2048 f64 0 5 - 1 > gpurun_out/ncu_stream.log 2>&1
