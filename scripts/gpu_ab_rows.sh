# A/B of k_pcr_rows builds (build_var/*): c3 SPLIT k = 14, alternating runs
mkdir -p gpurun_out/abrows
for r in 1 2; do
  for v in base r16pf0 r16pf1 r8pf0; do
    lib=""; [ $v != base ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
    env $lib timeout 300 python bench.py --config c3 --variant 2 --k 14 --no-e2e --no-cpu --steps 20 > gpurun_out/abrows/${v}_$r.json 2> gpurun_out/abrows/${v}_$r.err
  done
done
