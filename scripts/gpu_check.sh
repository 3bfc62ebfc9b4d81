# parity + quick bench lines (run under gpurun)
python -m pytest tests -m gpu -q -x 2>&1 | tail -15
python bench.py --steps 10 --warmup 3 --no-cpu 2>&1 | tail -1
python bench.py --config nuss4 --steps 3 --warmup 3 --no-cpu 2>&1 | tail -1
DP_NUSS5_N=100000 python bench.py --config nuss5 --steps 2 --warmup 3 --no-cpu 2>&1 | tail -1
