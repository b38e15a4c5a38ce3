mkdir -p gpurun_out/split
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pcr_rows -c 1 -o gpurun_out/split/c3_k14_rows -f \
  python bench.py --config c3 --variant 2 --k 14 --no-e2e --no-cpu --no-check --steps 1 --warmup 0 > gpurun_out/split/ncu.log 2>&1
SPLIT_KS="14 13 15" bash scripts/gpu_split.sh
