mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -k "scan and not mc" > gpurun_out/pytest_scan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_scan.log
( for rep in 1 2; do for lib in paper_conf_icpp_kimwch11_b200/libtri.so build_var/libtri_db0.so; do echo "== $lib"; for args in "256 1048576 f32 0 0" "256 1048576 f64 0 0" "128 2097152 f32 0 0"; do TRI_LIB_PATH=$lib timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done; done;
echo "== old path"; for args in "256 1048576 f32 0 0" "256 1048576 f64 0 0" "128 2097152 f32 0 0"; do TRI_SCAN1_OFF=1 timeout 120 python scripts/prof_one.py $args - 2 | grep graph; done; done ) > gpurun_out/scan_times.log 2>&1
