mkdir -p gpurun_out
timeout 300 python -m pytest tests -q -x -m gpu -p no:cacheprovider -k "scan_grid or scan_interleaved or row_scale_range or batched_layout" > gpurun_out/pytest_quick.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_quick.log
timeout 60 python scripts/prof_grid.py 1024 1024 f64 > gpurun_out/prof_grid.txt 2>&1
timeout 120 python bench.py --config c2 --no-e2e --no-cpu > gpurun_out/qbench_c2.json 2> gpurun_out/qbench_c2.err
