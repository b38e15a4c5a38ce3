mkdir -p gpurun_out
for W in 8 10 14; do echo "== W=$W"; TRI_LIB_PATH=$PWD/paper_conf_icpp_kimwch11_b200/libtri_w$W.so timeout 120 python scripts/prof_one.py 16384 16384 f64 0 5 - 2 | grep graph; TRI_LIB_PATH=$PWD/paper_conf_icpp_kimwch11_b200/libtri_w$W.so timeout 120 python scripts/prof_one.py 16384 2048 f64 0 5 - 2 | grep graph; done > gpurun_out/stream_w.log 2>&1
echo "== W=12"; timeout 120 python scripts/prof_one.py 16384 16384 f64 0 5 - 2 | grep graph >> gpurun_out/stream_w.log
