timeout 300 python -m pytest tests -q -x -m gpu -p no:cacheprovider -k "32_systems or scan_interleaved or ignored_entries_nan_scan or 16_byte or c4_auto or full_size" 2>&1 | tail -2
for r in 1 2; do
for v in cur nw12; do
  lib=""; [ $v != cur ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
  env $lib timeout 120 python bench.py --config c4 --layout 1 --no-e2e --no-cpu --no-check 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c4il $v', d['ms_per_step'], d['roofline']['frac'])"
done
done
timeout 600 python scripts/sweep_s32.py f32,f64 64,128,256 > gpurun_out/sweep_s32c.jsonl 2>&1
