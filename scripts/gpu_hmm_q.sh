python -m pytest tests -m gpu -q -x -k "viterbi or hmm or forward" 2>&1 | tail -3 > gpurun_out/gpu_tests_hmm.log
python bench.py --config hmm --steps 5 --warmup 3 --no-cpu 2>/dev/null | tail -1 > gpurun_out/bench_hmm.json
python -c "import json; d=json.load(open('gpurun_out/bench_hmm.json')); print(d['value'], d['ms_per_step'], d.get('phases_ms'), d['e2e']['value'])" >> gpurun_out/gpu_tests_hmm.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 8 --csv --log-file gpurun_out/launches_hmm_q.csv python bench.py --config hmm --steps 1 --warmup 1 --no-cpu > /dev/null 2>&1
python scripts/ncu_summary.py --launches gpurun_out/launches_hmm_q.csv >> gpurun_out/gpu_tests_hmm.log 2>&1
