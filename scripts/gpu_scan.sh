mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -q -k "autotune" > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
