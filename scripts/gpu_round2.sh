# Round-2 evidence on one B200: GPU tests, smoke, bench lines of every config and of the
# paper's method (forced STREAM / SPLIT), launch lists, ncu --set full of the hot kernels
# with traffic files, and a 2-rank code-path check of the strong-scaling bench.
set -u
mkdir -p gpurun_out/r2
O=gpurun_out/r2
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/smi.txt
timeout 1800 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
for c in c5 c1 c2 c3 c4; do timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; done
timeout 600 python bench.py --config c5 --layout 1 --no-e2e > $O/bench_c5_il.json 2> $O/bench_c5_il.err
timeout 600 python bench.py --config c4 --layout 1 --no-e2e > $O/bench_c4_il.json 2> $O/bench_c4_il.err
timeout 600 python bench.py --config c5 --variant 5 --no-e2e --no-cpu > $O/bench_c5_stream.json 2> $O/bench_c5_stream.err
timeout 600 python bench.py --config c3 --variant 2 --no-e2e --no-cpu > $O/bench_c3_split.json 2> $O/bench_c3_split.err
timeout 600 python bench.py --config c5 --k 3 --no-e2e --no-cpu > $O/bench_c5_k3.json 2> $O/bench_c5_k3.err
timeout 600 python bench.py --config c5 --no-graph --no-e2e --no-cpu > $O/bench_c5_nograph.json 2> $O/bench_c5_nograph.err
timeout 600 python bench.py --impl reference --config c5 > $O/bench_ref_c5.json 2> $O/bench_ref_c5.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu > $O/bench_c5_2ranks_1gpu.json 2> $O/bench_c5_2ranks_1gpu.err
timeout 600 python scripts/launch_times.py python bench.py --config c5 --steps 2 --warmup 1 --no-e2e --no-cpu --no-check > $O/launches_c5.txt 2>&1
timeout 600 python scripts/launch_times.py python scripts/prof_one.py 16777216 1 f64 0 2 - 2 > $O/launches_split_c3.txt 2>&1
# ncu --set full of each config's solve (all its launches), traffic files
prof() {  # name n m dt layout variant k launches regex
  PROF_GRAPH=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:$9 -s $8 -c $8 -f -o $O/$1 python scripts/prof_one.py $2 $3 $4 $5 $6 $7 2 > $O/ncu_$1.log 2>&1
  python scripts/ncu_summary.py $O/$1.ncu-rep $O/ncu_$1.txt $O/traffic_$1.json $2 $3 ${7/-/0} $6 $5 >> $O/ncu_$1.log 2>&1
}
prof c5_scan 16384 16384 f64 0 6 - 1 k_scan
prof c4_scan 256 1048576 f32 0 6 - 1 k_scan
prof c3_scanmc 16777216 1 f64 0 7 - 3 k_scan_mc
prof c2_scanil 1024 1024 f64 1 6 - 1 k_scan
prof c3_split_k14 16777216 1 f64 0 2 14 3 "k_tiled|k_pthomas"
