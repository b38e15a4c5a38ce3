mkdir -p gpurun_out/split
SPLIT_KS="14" SPLIT_SEL="cp_async or split_every or pcr_stage_matches or chain_interleaved or set_k_every or split_on_small" bash scripts/gpu_split.sh
