mkdir -p gpurun_out/large
timeout 1500 python -m pytest tests/test_large_gpu.py tests/test_bench_contract.py -q -m gpu -p no:cacheprovider --timeout 1200 -x > gpurun_out/large/pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/large/pytest.log
