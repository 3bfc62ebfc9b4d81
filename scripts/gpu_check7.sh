timeout 300 python scripts/nuss_tb_probe.py 20000 nuss4
python -m pytest tests -m gpu -q -x -k "nussinov or sw or align or host" 2>&1 | tail -2
python bench.py --steps 10 --warmup 3 --no-cpu 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sw', d['ms_per_step'], d['kernel_ms'], d['roofline']['frac'])"
DP_SW_TB_UNPACKED=1 python bench.py --steps 10 --warmup 3 --no-cpu 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sw unpacked tb', d['ms_per_step'], d['kernel_ms'])"
