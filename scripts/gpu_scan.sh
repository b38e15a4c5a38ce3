mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "scan" > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
( for lib in "" build_var/libtri_nw8.so; do
  echo "=== lib $lib"
  for args in "16384 16384 f64 0 6" "2048 16384 f64 0 6"; do TRI_LIB_PATH=${lib:-paper_conf_icpp_kimwch11_b200/libtri.so} timeout 120 python scripts/prof_one.py $args - 2; done
done
timeout 120 python scripts/prof_scan.py 16384 16384; TRI_FUSED_DBG_MODE=2 timeout 120 python scripts/prof_scan.py 16384 16384
) > gpurun_out/scan_times.log 2>&1
