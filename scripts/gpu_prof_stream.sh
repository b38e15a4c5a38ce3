mkdir -p gpurun_out
( echo "== mode 0"; timeout 120 python scripts/prof_stream.py 16384 2048 ) > gpurun_out/prof_stream.log 2>&1
