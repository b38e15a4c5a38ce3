# SCAN_MC look-back path (TRI_SCAN_MC_LB=1): parity of the SCAN_MC suite, c3 bench A/B
mkdir -p gpurun_out
TRI_SCAN_MC_LB=1 timeout 300 python -m pytest tests/test_parity_gpu.py -x -q -m gpu -k "scan_mc or baseline or sliced" > gpurun_out/mclb_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/mclb_pytest.log
timeout 200 python bench.py --config c3 --no-e2e --no-cpu > gpurun_out/mclb_c3_base.json 2> gpurun_out/mclb_c3_base.err
for w in 24 32 48 64; do
  TRI_SCAN_MC_LB=1 TRI_SCAN_MC_LBW=$w timeout 200 python bench.py --config c3 --no-e2e --no-cpu > gpurun_out/mclb_c3_$w.json 2> gpurun_out/mclb_c3_$w.err
done
TRI_SCAN_MC_LB=1 timeout 200 python scripts/prof_one.py 16777216 1 f32 0 7 - 3 > gpurun_out/mclb_f32.txt 2>&1
timeout 200 python scripts/prof_one.py 16777216 1 f32 0 7 - 3 >> gpurun_out/mclb_f32.txt 2>&1
TRI_SCAN_MC_LB=1 timeout 200 python scripts/launch_times.py python bench.py --config c3 --steps 2 --warmup 1 --no-e2e --no-cpu --no-check > gpurun_out/mclb_launches_c3.txt 2>&1
