python -m pytest tests -m gpu -q -x 2>&1 | tail -4
python bench.py --steps 10 --warmup 3 --no-cpu 2>&1 | tail -1
python bench.py --config hmm --steps 5 --warmup 3 --no-cpu 2>&1 | tail -1
python bench.py --config nuss4 --steps 3 --warmup 3 --no-cpu 2>&1 | tail -1
DP_NUSS5_N=100000 python bench.py --config nuss5 --steps 2 --warmup 3 --no-cpu 2>&1 | tail -1
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_sw_r01b.csv python bench.py --steps 2 --warmup 1 --no-cpu > /dev/null 2>&1
