timeout 600 python -m pytest tests -q -x -m gpu -p no:cacheprovider -k "f32 or interleaved or row_scale or 32_systems or ignored or 16_byte or scan_mc or batched or strided" 2>&1 | tail -1
for r in 1 2 3; do
for v in prev cur; do
  lib=""; [ $v != cur ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
  env $lib timeout 120 python bench.py --config c4 --layout 1 --no-e2e --no-cpu --no-check 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c4il $v', d['ms_per_step'], d['roofline']['frac'])"
done
done
