# A/B of k_scan_w512 compile-time parameters on c5 (alternating runs, same box), with
# the bench's sampled parity check on: $@ = build_var names (or "cur")
mkdir -p gpurun_out/ab5
for r in 1 2 3; do
  for v in "$@"; do
    lib=""; [ $v != cur ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
    env $lib timeout 120 python bench.py --config c5 --no-e2e --no-cpu 2>>gpurun_out/ab5/err_$v.log | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$v', d['ms_per_step'], d.get('parity', d.get('check')))"
  done
done
