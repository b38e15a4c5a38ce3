# SPLIT bench lines with the register-tile passes: c3 k=14 (+ launch list), the ragged
# and few-long-interleaved shapes the planner sends to SPLIT, over a few k
mkdir -p gpurun_out/split2
B="timeout 300 python bench.py --no-e2e --no-cpu --steps 20 --variant 2"
$B --config c3 --k 14 > gpurun_out/split2/c3_k14.json 2> gpurun_out/split2/c3_k14.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/split2/launches_c3_k14.csv \
  python bench.py --config c3 --variant 2 --k 14 --no-e2e --no-cpu --no-check --steps 3 --warmup 3 > /dev/null 2>&1
for k in 10 12 14 16; do $B --config c3 --n 1048579 --m 1 --k $k > gpurun_out/split2/ragged_k$k.json 2> gpurun_out/split2/ragged_k$k.err; done
for k in 5 6 8 10; do $B --config c5 --n 65536 --m 37 --layout 1 --k $k > gpurun_out/split2/il37_k$k.json 2> gpurun_out/split2/il37_k$k.err; done
for k in 3 6 9; do $B --config c2 --k $k > gpurun_out/split2/c2_k$k.json 2> gpurun_out/split2/c2_k$k.err; done
