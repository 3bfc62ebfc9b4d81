python -m pytest tests -m gpu -q -x -k "nussinov or smoke" 2>&1 | tail -2 > gpurun_out/n1t.log
rm -f gpurun_out/variants.log
STEPS=200 bash scripts/gpu_variants.sh --config nuss1
