mkdir -p gpurun_out
( timeout 120 python scripts/prof_scan.py 16384 16384; TRI_FUSED_DBG_MODE=2 timeout 120 python scripts/prof_scan.py 16384 16384; TRI_FUSED_DBG_MODE=1 timeout 120 python scripts/prof_scan.py 16384 16384 ) > gpurun_out/prof_scan.log 2>&1
