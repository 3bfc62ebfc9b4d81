python -m pytest tests -m gpu -q -x -k "sw or align or host or smoke" 2>&1 | tail -15 > gpurun_out/gpu_tests_sw.log
python bench.py --steps 10 --warmup 3 --no-cpu 2>gpurun_out/bench_sw.err | tail -1 > gpurun_out/bench_sw.json
python -c "import json; d=json.load(open('gpurun_out/bench_sw.json')); print(d['value'], d['ms_per_step'], d.get('phases_ms'), d['e2e']['value'], d['roofline']['kernel_ms'])" >> gpurun_out/gpu_tests_sw.log 2>&1
DP_SW_TIMING=1 python bench.py --steps 1 --warmup 0 --no-cpu 2>&1 | grep '^tb' >> gpurun_out/gpu_tests_sw.log
