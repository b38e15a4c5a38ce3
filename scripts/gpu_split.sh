# SPLIT register-tile passes: bench lines at c3 for several k, the launch list at
# k = 14, then the SPLIT parity selection
mkdir -p gpurun_out/split
for k in ${SPLIT_KS:-5 8 11 14}; do
  timeout 300 python bench.py --config c3 --variant 2 --k $k --no-e2e --no-cpu --steps 20 > gpurun_out/split/c3_k$k.json 2> gpurun_out/split/c3_k$k.err
done
timeout 300 python bench.py --config c3 --variant 2 --k 14 --no-e2e --no-cpu --steps 20 --layout 0 > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/split/launches_c3_k14.csv \
  python bench.py --config c3 --variant 2 --k 14 --no-e2e --no-cpu --no-check --steps 3 --warmup 3 > /dev/null 2>&1
timeout 1800 python -m pytest tests/test_parity_gpu.py -q -x -p no:cacheprovider --timeout 900 \
  -k "${SPLIT_SEL:-split_every or pcr_stage_matches or chain_interleaved or set_k_every or split_on_small}" > gpurun_out/split/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/split/pytest.log
