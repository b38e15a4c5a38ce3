mkdir -p gpurun_out/split
python scripts/split_pcr_check.py 16777216 1 2 3 5 > gpurun_out/split/pcr_c3.txt 2>&1
python scripts/split_pcr_check.py 1000003 1 2 3 5 >> gpurun_out/split/pcr_c3.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pcr_rows -c 1 -o gpurun_out/split/c3_k14_rows2 -f \
  python bench.py --config c3 --variant 2 --k 14 --no-e2e --no-cpu --no-check --steps 1 --warmup 0 > gpurun_out/split/ncu.log 2>&1
SPLIT_KS="14" SPLIT_SEL="cp_async or split_every or pcr_stage_matches or chain_interleaved or set_k_every or split_on_small" bash scripts/gpu_split.sh
