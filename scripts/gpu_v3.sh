rm -f gpurun_out/variants.log
STEPS=20 bash scripts/gpu_variants.sh --config hmm
STEPS=20 bash scripts/gpu_variants.sh --config diag
