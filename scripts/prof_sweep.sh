python -m pytest tests -m gpu -q -x -k "sw or align or host or smoke" 2>&1 | tail -3 > gpurun_out/gpu_tests_sw.log
python bench.py --steps 10 --warmup 3 --no-cpu 2>/dev/null | tail -1 > gpurun_out/bench_sw.json
python -c "import json; d=json.load(open('gpurun_out/bench_sw.json')); print(d['value'], d['ms_per_step'], d.get('phases_ms'), d['e2e']['value'])" >> gpurun_out/gpu_tests_sw.log 2>&1
ncu --set full --clock-control none --import-source on -k k_sw16 -c 1 -o gpurun_out/prof_sweep python bench.py --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu -i gpurun_out/prof_sweep.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_sweep_src.csv 2>/dev/null
