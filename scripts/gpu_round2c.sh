# full validation after the register-tile SPLIT passes and the cluster option:
# all GPU tests, smoke, bench lines of every config, SPLIT c3 ncu traffic
set -u
O=gpurun_out/r2c
mkdir -p $O
timeout 2400 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
for c in c5 c4 c3 c2 c1; do timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; done
timeout 600 python bench.py --config c3 --variant 2 --k 14 > $O/bench_c3_split.json 2> $O/bench_c3_split.err
timeout 900 ncu --set full --clock-control none -k regex:"k_pcr|k_pthomas" -c 5 -f -o $O/c3_split \
  python bench.py --config c3 --variant 2 --k 14 --no-e2e --no-cpu --no-check --steps 1 --warmup 0 > $O/ncu_c3_split.log 2>&1
python scripts/ncu_summary.py $O/c3_split.ncu-rep $O/ncu_c3_split.txt $O/traffic_c3_split.json 16777216 1 14 2 0 >> $O/ncu_c3_split.log 2>&1
