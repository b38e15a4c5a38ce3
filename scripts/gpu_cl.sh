mkdir -p gpurun_out/cl
timeout 1200 python -m pytest tests -q -x -m gpu -p no:cacheprovider --timeout 900 -k "cluster_option or interleaved or c2" > gpurun_out/cl/pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/cl/pytest.log
