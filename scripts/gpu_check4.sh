timeout 300 python scripts/nuss_tb_probe.py 20000
python -m pytest tests -m gpu -q -x -k "forward or hmm" 2>&1 | tail -4
python bench.py --config hmm --steps 5 --warmup 3 --no-cpu 2>&1 | tail -1 | cut -c1-300
