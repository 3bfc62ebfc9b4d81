python -m pytest tests -m gpu -q -x 2>&1 | tail -4
for c in sw hmm nuss1 nuss4; do
python bench.py --config $c --steps 5 --warmup 3 --no-cpu 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$c', d['value'], d['ms_per_step'], d['phases_ms'], d['roofline']['frac'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"
done
