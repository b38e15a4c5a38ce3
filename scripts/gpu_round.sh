# Round evidence on one B200: GPU tests, smoke, bench lines of every config,
# launch list of the c5 bench command, ncu --set full of the c5 and c4 kernels.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
for c in c5 c1 c2 c3 c4; do timeout 600 python bench.py --config $c > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; done
timeout 600 python scripts/launch_times.py python bench.py --config c5 --steps 2 --warmup 1 --no-e2e --no-cpu --no-check > gpurun_out/launches_c5.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan -c 1 -f -o gpurun_out/c5_scan_full python scripts/prof_one.py 16384 16384 f64 0 0 - 1 > gpurun_out/ncu_c5.log 2>&1
python scripts/ncu_summary.py gpurun_out/c5_scan_full.ncu-rep gpurun_out/ncu_c5_scan.txt >> gpurun_out/ncu_c5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan -c 1 -f -o gpurun_out/c4_scan_full python scripts/prof_one.py 256 1048576 f32 0 0 - 1 > gpurun_out/ncu_c4.log 2>&1
python scripts/ncu_summary.py gpurun_out/c4_scan_full.ncu-rep gpurun_out/ncu_c4_scan.txt >> gpurun_out/ncu_c4.log 2>&1
# the paper's PCR method on the configs where the planner now prefers SCAN / SCAN_MC
timeout 600 python bench.py --config c3 --variant 2 --no-e2e --no-cpu > gpurun_out/bench_c3_split.json 2> gpurun_out/bench_c3_split.err
timeout 600 python bench.py --config c5 --variant 5 --no-e2e --no-cpu > gpurun_out/bench_c5_stream.json 2> gpurun_out/bench_c5_stream.err
timeout 600 python bench.py --config c4 --variant 2 --k 0 --no-e2e --no-cpu > gpurun_out/bench_c4_split.json 2> gpurun_out/bench_c4_split.err
