# A/B of the k_scan build against build_var/old on c5 (alternating runs, same box)
mkdir -p gpurun_out/ab
timeout 300 python -m pytest tests -q -x -m gpu -p no:cacheprovider -k "scan and not full_size and not large" > gpurun_out/ab/pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/ab/pytest.log
for r in 1 2 3; do
  for v in new old; do
    lib=""; [ $v = old ] && lib="TRI_LIB_PATH=build_var/old/libtri.so"
    env $lib timeout 120 python bench.py --config c5 --no-e2e --no-cpu --no-check 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$v', d['ms_per_step'])"
  done
done
