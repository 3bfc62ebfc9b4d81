python -m pytest tests -m gpu -q -x 2>&1 | grep -E "FAILED|passed|failed|^E " | head -20
timeout 900 compute-sanitizer --tool memcheck --show-backtrace no python -m pytest tests -m gpu -q -x -k "ragged or degenerate or odd or smem or random" 2>&1 | grep -E "ERROR SUMMARY|Invalid|at |passed|failed" | head -20
python bench.py --steps 10 --warmup 3 --no-cpu 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sw', d['ms_per_step'], d['kernel_ms'], d['roofline']['frac'], d['e2e']['ms_per_step'])"
