rm -f gpurun_out/variants.log
DP_NUSS5_N=200000 STEPS=2 bash scripts/gpu_variants.sh --config nuss5
STEPS=5 bash scripts/gpu_variants.sh --config nuss4
