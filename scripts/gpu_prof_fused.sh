mkdir -p gpurun_out
for mode in 0 1 3 4 5; do echo "== mode $mode"; TRI_FUSED_DBG_MODE=$mode timeout 120 python scripts/prof_fused.py 16384 2048; done > gpurun_out/prof_fused.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_fused -c 1 -o gpurun_out/fused_full python scripts/prof_one.py 16384 2048 f64 0 3 - 1 > gpurun_out/ncu_fused.log 2>&1
