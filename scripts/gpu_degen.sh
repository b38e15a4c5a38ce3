mkdir -p gpurun_out/degen
timeout 1200 python -m pytest tests/test_parity_gpu.py -q -m gpu -p no:cacheprovider --timeout 900 -k degenerate > gpurun_out/degen/pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/degen/pytest.log
