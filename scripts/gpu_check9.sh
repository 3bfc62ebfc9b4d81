python -m pytest tests -m gpu -q -x 2>&1 | tail -4
python bench.py --steps 10 --warmup 3 --no-cpu 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sw', d['ms_per_step'], d['phases_ms'], d['roofline']['frac'], d['e2e']['ms_per_step'], d['clocks'])"
python bench.py --config nuss1 --steps 20 --warmup 5 --no-cpu 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('nuss1', d['ms_per_step'], d['phases_ms'], d['e2e']['ms_per_step'])"
