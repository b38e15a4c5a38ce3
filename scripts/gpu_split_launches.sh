mkdir -p gpurun_out
for k in 14 10 6; do
timeout 300 python scripts/launch_times.py python scripts/prof_one.py 16777216 1 f64 0 2 $k 2 > gpurun_out/split_c3_k$k.txt 2>&1
done
timeout 300 python scripts/launch_times.py python scripts/prof_one.py 1000003 16 f64 0 2 - 2 > gpurun_out/split_ragged.txt 2>&1
timeout 300 python scripts/launch_times.py python scripts/prof_one.py 65536 37 f64 1 2 - 2 > gpurun_out/split_il37.txt 2>&1
