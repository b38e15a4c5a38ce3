# SCAN_MC look-back: bench A/B over chunk sizes + ncu DRAM bytes of the look-back kernel
mkdir -p gpurun_out
TRI_SCAN_MC_LB=1 timeout 300 python -m pytest tests/test_parity_gpu.py -x -q -m gpu -k "scan_mc or baseline or sliced" > gpurun_out/mclb_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/mclb_pytest.log
for w in 48 64 80; do
  TRI_SCAN_MC_LB=1 TRI_SCAN_MC_LBW=$w timeout 200 python bench.py --config c3 --no-e2e --no-cpu > gpurun_out/mclb_c3_$w.json 2> gpurun_out/mclb_c3_$w.err
done
TRI_SCAN_MC_LB=1 TRI_SCAN_MC_LBW=64 timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_scan_mc_lb -c 2 -f -o gpurun_out/mclb_full python scripts/prof_one.py 16777216 1 f64 0 7 - 1 > gpurun_out/mclb_ncu.log 2>&1
python scripts/ncu_summary.py gpurun_out/mclb_full.ncu-rep gpurun_out/ncu_mclb.txt >> gpurun_out/mclb_ncu.log 2>&1
