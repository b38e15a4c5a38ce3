# A/B of L2-blocked SCAN_MC super-chunks (SMC_L2_MB) at c3, alternating runs; parity tests
mkdir -p gpurun_out/abl2
for r in 1 2 3; do
  for v in base l2mb24 l2mb64 l2off; do
    lib=""; [ $v != base ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
    env $lib timeout 300 python bench.py --config c3 --no-e2e --no-cpu --steps 20 > gpurun_out/abl2/${v}_c3_$r.json 2> gpurun_out/abl2/${v}_c3_$r.err
  done
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 40 --csv --log-file gpurun_out/abl2/launches_c3.csv \
  python bench.py --config c3 --no-e2e --no-cpu --no-check --steps 1 --warmup 1 > /dev/null 2>&1
timeout 1500 python -m pytest tests -q -x -m gpu -p no:cacheprovider --timeout 900 -k "scan_mc or sliced or c3 or ragged or set_k_every or full_size" > gpurun_out/abl2/pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/abl2/pytest.log
