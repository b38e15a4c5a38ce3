mkdir -p gpurun_out/split3
B="timeout 300 python bench.py --no-e2e --no-cpu --steps 20 --variant 2"
for k in 12 14; do $B --config c3 --n 1048579 --m 1 --k $k > gpurun_out/split3/ragged_k$k.json 2> gpurun_out/split3/ragged_k$k.err; done
for k in 8 10; do $B --config c5 --n 65536 --m 37 --layout 1 --k $k > gpurun_out/split3/il37_k$k.json 2> gpurun_out/split3/il37_k$k.err; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file gpurun_out/split3/launches_ragged_k14.csv \
  python bench.py --config c3 --n 1048579 --m 1 --variant 2 --k 14 --no-e2e --no-cpu --no-check --steps 3 --warmup 3 > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 30 --csv --log-file gpurun_out/split3/launches_il37_k8.csv \
  python bench.py --config c5 --n 65536 --m 37 --layout 1 --variant 2 --k 8 --no-e2e --no-cpu --no-check --steps 3 --warmup 3 > /dev/null 2>&1
