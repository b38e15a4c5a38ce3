mkdir -p gpurun_out/cl
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan -c 1 -o gpurun_out/cl/c2_cl -f \
  python bench.py --config c2 --no-e2e --no-cpu --no-check --steps 1 --warmup 0 > gpurun_out/cl/ncu.log 2>&1
TRI_LIB_PATH=build_var/nocl/libtri.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_scan -c 1 -o gpurun_out/cl/c2_chain -f \
  python bench.py --config c2 --no-e2e --no-cpu --no-check --steps 1 --warmup 0 > gpurun_out/cl/ncu2.log 2>&1
