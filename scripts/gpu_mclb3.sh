# SCAN_MC look-back (lag-1 pipelined): parity + c3 A/B over chunk sizes
mkdir -p gpurun_out
TRI_SCAN_MC_LB=1 timeout 300 python -m pytest tests/test_parity_gpu.py -x -q -m gpu -k "scan_mc or baseline or sliced" > gpurun_out/mclb5_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/mclb5_pytest.log
timeout 200 python bench.py --config c3 --no-e2e --no-cpu > gpurun_out/mclb5_c3_base.json 2> gpurun_out/mclb5_c3_base.err
for w in 24 32 48 64; do
  TRI_SCAN_MC_LB=1 TRI_SCAN_MC_LBW=$w timeout 200 python bench.py --config c3 --no-e2e --no-cpu > gpurun_out/mclb5_c3_$w.json 2> gpurun_out/mclb5_c3_$w.err
done
for w in 24 48; do
TRI_SCAN_MC_LB=1 TRI_SCAN_MC_LBW=$w timeout 200 python scripts/prof_one.py 16777216 1 f32 0 7 - 3 > gpurun_out/mclb5_f32_$w.txt 2>&1
done
timeout 200 python scripts/prof_one.py 16777216 1 f32 0 7 - 3 > gpurun_out/mclb5_f32_base.txt 2>&1
TRI_SCAN_MC_LB=1 TRI_SCAN_MC_LBW=32 timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan_mc_lb -c 2 -f -o gpurun_out/mclb5_full python scripts/prof_one.py 16777216 1 f64 0 7 - 1 > gpurun_out/mclb5_ncu.log 2>&1
python scripts/ncu_summary.py gpurun_out/mclb5_full.ncu-rep gpurun_out/ncu_mclb3.txt >> gpurun_out/mclb5_ncu.log 2>&1
