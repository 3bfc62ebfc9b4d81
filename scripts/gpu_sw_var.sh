bash scripts/gpu_sw.sh
bash scripts/gpu_variants.sh
