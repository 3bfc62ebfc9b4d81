python -m pytest tests -m gpu -q -x -k "forward or hmm or viterbi" 2>&1 | tail -4
python bench.py --config hmm --steps 5 --warmup 3 --no-cpu 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('hmm', d['value'], d['ms_per_step'], d['phases_ms'], d['roofline']['frac'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"
