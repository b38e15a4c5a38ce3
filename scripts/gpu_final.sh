# final validation: every -m gpu test, smoke, the default bench line, the reference
# arm, a 2-rank strong-scaling code-path run on the one GPU, c1..c5 lines
set -u
O=gpurun_out/final
mkdir -p $O
timeout 2400 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_ref.json 2> $O/bench_ref.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --steps 10 --warmup 3 > $O/bench_2ranks.json 2> $O/bench_2ranks.err
for c in c4 c3 c2 c1; do timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; done
