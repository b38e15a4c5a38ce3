timeout 600 python -m pytest tests -q -m gpu -p no:cacheprovider -k "scan or w512 or degenerate or ignored or auto_plan or set_k or solve_host" > gpurun_out/pt_c1.log 2>&1; tail -1 gpurun_out/pt_c1.log; grep FAILED gpurun_out/pt_c1.log | head -5
for r in 1 2 3; do
for v in prev cur; do
  lib=""; [ $v != cur ] && lib="TRI_LIB_PATH=build_var/$v/libtri.so"
  env $lib timeout 120 python bench.py --config c1 --no-e2e --no-cpu --no-check 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('c1 $v', d['ms_per_step'], d['b2b']['ms_per_step'])"
done
done
