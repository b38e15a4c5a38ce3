mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_dist_sliced_gpu.py -q --timeout 300 > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
