DP_SW_TIMING=1 python bench.py --steps 1 --warmup 0 --no-cpu 2>&1 | grep "^tb " | tail -8 > gpurun_out/tb_timing.txt
DP_NUSS_TIMING=1 DP_NUSS5_N=20000 python bench.py --config nuss5 --steps 1 --warmup 0 --no-cpu 2>&1 | grep "^nuss " | tail -7 > gpurun_out/nuss_timing.txt
bash scripts/gpu_sw.sh
