mkdir -p gpurun_out
TRI_SCAN_RS=1 timeout 600 python -m pytest tests/test_parity_gpu.py -q -k "scan and not mc and not interleaved and not batched" --timeout 120 -x > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
( for rep in 1 2; do for lib in paper_conf_icpp_kimwch11_b200/libtri.so build_var/libtri_rs11_4.so build_var/libtri_rs9_5.so; do echo "== $lib RS"; for args in "16384 16384 f64 0 0" "2048 16384 f64 0 0" "16384 9472 f32 0 0"; do TRI_SCAN_RS=1 TRI_LIB_PATH=$lib timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done; done
echo "== baseline"; for args in "16384 16384 f64 0 0" "2048 16384 f64 0 0" "16384 9472 f32 0 0"; do timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done; done ) > gpurun_out/scan_times.log 2>&1
