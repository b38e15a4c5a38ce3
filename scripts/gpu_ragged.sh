mkdir -p gpurun_out/ragged
timeout 2000 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > gpurun_out/ragged/pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/ragged/pytest.log
