mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_parity_gpu.py -q -k "role_split" --timeout 300 > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
