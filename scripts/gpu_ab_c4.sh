# A/B of builds on c4 (alternating runs, same box): $@ = build_var names (or "cur")
mkdir -p gpurun_out/ab
for r in ${ROUNDS:-1 2 3}; do
  for v in "$@"; do
    lib=""; [ $v != cur ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
    env $lib timeout 120 python bench.py --config c4 --no-e2e --no-cpu --no-check 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$v', d['ms_per_step'])"
  done
done
