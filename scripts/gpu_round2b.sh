# after restoring the SCAN lag 8: tests, smoke, sanitizers, c5 / c2 lines and ncu
set -u
O=gpurun_out/r2b
mkdir -p $O
timeout 1800 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
for c in c5 c2 c1; do timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; done
prof() {
  PROF_GRAPH=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:$9 -s $8 -c $8 -f -o $O/$1 python scripts/prof_one.py $2 $3 $4 $5 $6 $7 2 > $O/ncu_$1.log 2>&1
  python scripts/ncu_summary.py $O/$1.ncu-rep $O/ncu_$1.txt $O/traffic_$1.json $2 $3 ${7/-/0} $6 $5 >> $O/ncu_$1.log 2>&1
}
prof c5_scan 16384 16384 f64 0 6 - 1 k_scan
prof c2_scanil 1024 1024 f64 1 6 - 1 k_scan
timeout 600 python scripts/launch_times.py python bench.py --config c5 --steps 2 --warmup 1 --no-e2e --no-cpu --no-check > $O/launches_c5.txt 2>&1
mv gpurun_out/san gpurun_out/san_prev 2>/dev/null
bash scripts/gpu_sanitize.sh
