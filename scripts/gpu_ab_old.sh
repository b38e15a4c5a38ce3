# A/B: in-tree build vs build_var/old (the previous commit), alternating runs
mkdir -p gpurun_out/ab2
for r in 1 2 3; do
  for v in base old; do
    lib=""; [ $v != base ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
    for c in $AB_CONFIGS; do env $lib timeout 300 python bench.py --config $c --no-e2e --no-cpu --steps 20 > gpurun_out/ab2/${v}_${c}_$r.json 2>gpurun_out/ab2/${v}_${c}_$r.err; done
  done
done
