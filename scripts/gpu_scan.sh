mkdir -p gpurun_out
( timeout 120 python scripts/prof_scan.py 1024 1024 f64 1 ) > gpurun_out/prof_scan.log 2>&1
