timeout 300 python -m pytest tests -q -x -m gpu -p no:cacheprovider -k "32_systems or scan_interleaved or ignored_entries_nan_scan or 16_byte" 2>&1 | tail -2
for r in 1 2; do
for v in cur s8; do
  lib=""; [ $v != cur ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
  env $lib timeout 120 python bench.py --config c4 --layout 1 --variant 6 --no-e2e --no-cpu --no-check 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c4il-scan $v', d['ms_per_step'], d['config']['plan'][-60:])"
done
done
timeout 120 python bench.py --config c4 --layout 1 --no-e2e --no-cpu --no-check 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c4il-auto', d['ms_per_step'], d['config']['plan'][:120])"
