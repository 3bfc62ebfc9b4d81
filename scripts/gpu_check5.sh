timeout 300 python scripts/nuss_tb_probe.py 20000 nuss4
python -m pytest tests -m gpu -q -x 2>&1 | tail -3
python bench.py --config hmm --steps 5 --warmup 3 --no-cpu 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('hmm', d['ms_per_step'], d['kernel_ms'], d['roofline']['frac'])"
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_hmm_r01b.csv python bench.py --config hmm --steps 1 --warmup 1 --no-cpu > /dev/null 2>&1
