python -m pytest tests -m gpu -q -x -k "sw or align or host or edit" 2>&1 | tail -15
python bench.py --steps 10 --warmup 3 --no-cpu 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sw', d['ms_per_step'], d['phases_ms'], d['roofline']['frac'], d['e2e']['ms_per_step'], d['clocks'])"
