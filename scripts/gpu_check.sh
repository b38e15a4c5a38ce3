# Round-2 check on one B200: GPU tests, smoke, racecheck probe, short bench lines.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 1500 python -m pytest tests -q -m gpu -p no:cacheprovider --timeout 900 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -o /tmp/san_probe scripts/san/probe.cu > /dev/null 2>&1
for md in 0 1 2 3 4; do timeout 120 /usr/local/cuda/bin/compute-sanitizer --tool racecheck /tmp/san_probe $md > gpurun_out/probe_race_$md.log 2>&1; done
for c in c5 c1 c2 c3 c4; do timeout 600 python bench.py --config $c > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; done
