# A/B of the SCAN back-substitution lag (TRI_SCAN_DELTA) on the chained configs
mkdir -p gpurun_out
for dl in 8 1 2 4 0; do
  for c in c1 c2 c5; do
    TRI_SCAN_DELTA=$dl timeout 300 python bench.py --config $c --no-e2e --no-cpu --steps 50 > gpurun_out/delta_${dl}_$c.json 2> gpurun_out/delta_${dl}_$c.err
  done
done
