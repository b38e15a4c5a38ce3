# A/B of the SCAN warps per CTA (SC_NW_DEF) on c5 / c2 / c4: default build vs build_var/nw14, nw15
mkdir -p gpurun_out/ab
for v in base nw14 nw15; do
  lib=""; [ $v != base ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
  for c in c5 c2; do
    for r in 1 2; do env $lib timeout 300 python bench.py --config $c --no-e2e --no-cpu --steps 20 > gpurun_out/ab/${v}_${c}_$r.json 2>gpurun_out/ab/${v}_${c}_$r.err; done
  done
done
