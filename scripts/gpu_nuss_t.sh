DP_NUSS_TIMING=1 DP_NUSS5_N=20000 python bench.py --config nuss5 --steps 1 --warmup 0 --no-cpu 2>&1 | grep "^nuss " | tail -7 > gpurun_out/nuss_timing.txt
