# A/B of k_scan builds (build_var/*) on c5 and c2, alternating runs
mkdir -p gpurun_out/abscan
for r in 1 2 3; do
  for v in base bwdlast nw14 nw15; do
    lib=""; [ $v != base ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
    for c in c5 c2; do env $lib timeout 300 python bench.py --config $c --no-e2e --no-cpu --steps 20 > gpurun_out/abscan/${v}_${c}_$r.json 2> gpurun_out/abscan/${v}_${c}_$r.err; done
  done
done
timeout 1200 python -m pytest tests -q -x -m gpu -p no:cacheprovider --timeout 900 -k "scan" > gpurun_out/abscan/pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/abscan/pytest.log
