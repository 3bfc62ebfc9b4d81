python -m pytest tests -m gpu -q -x -k "nussinov" 2>&1 | tail -3 > gpurun_out/gpu_tests_nuss.log
DP_NUSS_ROUNDS=1 python bench.py --config nuss4 --steps 1 --warmup 0 --no-cpu 2>&1 | grep -v '^round' | grep 'traceback' | head -2 >> gpurun_out/gpu_tests_nuss.log
rm -f gpurun_out/variants.log; bash scripts/gpu_variants.sh --config nuss4
