# round-2 final validation: every -m gpu test, smoke, bench lines of c1..c5 (+ the
# reference arm and a 2-rank code-path run), ncu of the c5 kernel, launch lists
set -u
O=gpurun_out/final9
mkdir -p $O
timeout 2400 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 900 python bench.py > $O/bench_c5.json 2> $O/bench_c5.err
for c in c4 c3 c2 c1; do timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; done
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_ref.json 2> $O/bench_ref.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --steps 10 --warmup 3 > $O/bench_2ranks.json 2> $O/bench_2ranks.err
timeout 600 ncu --set full --clock-control none -k regex:k_scan_w512 -c 1 -f -o $O/c5_w512 python scripts/prof_one.py 16384 16384 f64 0 0 - 1 > $O/ncu_c5.log 2>&1
python scripts/ncu_summary.py $O/c5_w512.ncu-rep $O/ncu_c5_w512.txt >> $O/ncu_c5.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_c5.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > $O/ncu_launch_c5.log 2>&1
rm -f $O/*.ncu-rep
timeout 300 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum -k regex:k_scan_mc --launch-skip 3 -c 3 python scripts/prof_one.py 16777216 1 f64 0 0 - 2 > $O/ncu_c3_nocache.log 2>&1
for c in c4 c5; do timeout 600 python bench.py --config $c --layout 1 --no-e2e --no-cpu > $O/bench_${c}_il.json 2> $O/bench_${c}_il.err; done
