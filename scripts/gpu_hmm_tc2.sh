python -m pytest tests -m gpu -q -x -k "forward or hmm or smoke" 2>&1 | tail -3 > gpurun_out/tc2.log
python bench.py --config hmm --no-cpu 2>/dev/null | tail -1 > gpurun_out/tc2a.json
DP_HMM_TC1=1 python bench.py --config hmm --no-cpu 2>/dev/null | tail -1 > gpurun_out/tc2b.json
python -c "
import json
for f in ['gpurun_out/tc2a.json','gpurun_out/tc2b.json']:
    d=json.load(open(f)); print(f, d['value'], d['ms_per_step'], d['phases_ms'], d['roofline']['frac'], d['e2e']['value'])
" >> gpurun_out/tc2.log
ncu --metrics gpu__time_duration.sum --clock-control none -c 6 --csv --log-file gpurun_out/launches_tc2.csv python bench.py --config hmm --steps 1 --warmup 1 --no-cpu > /dev/null 2>&1
python scripts/ncu_summary.py --launches gpurun_out/launches_tc2.csv >> gpurun_out/tc2.log 2>&1
