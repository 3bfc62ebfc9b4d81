python -m pytest tests -m gpu -q -x -k "nussinov" 2>&1 | tail -3 > gpurun_out/gpu_tests_nuss.log
DP_NUSS_TIMING=1 DP_NUSS5_N=20000 python bench.py --config nuss5 --steps 1 --warmup 0 --no-cpu 2>&1 | grep "^nuss " | tail -7 >> gpurun_out/gpu_tests_nuss.log
python bench.py --config nuss4 --steps 3 --warmup 3 --no-cpu 2>/dev/null | tail -1 > gpurun_out/bench_nuss4.json
python bench.py --config nuss5 --steps 2 --warmup 3 --no-cpu 2>gpurun_out/bench_nuss5.err | tail -1 > gpurun_out/bench_nuss5.json
for c in nuss4 nuss5; do python -c "import json; d=json.load(open('gpurun_out/bench_$c.json')); print('$c', d['value'], d['ms_per_step'], d['phases_ms'], d['roofline']['frac'])" >> gpurun_out/gpu_tests_nuss.log 2>&1; done
