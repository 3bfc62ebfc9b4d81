python -m pytest tests -m gpu -q -x -k "forward or hmm" 2>&1 | tail -2 > gpurun_out/hs.log
python bench.py --config hmm --no-cpu 2>/dev/null | tail -1 > gpurun_out/hs1.json
DP_HMM_TC_SHARE=1 python bench.py --config hmm --no-cpu 2>/dev/null | tail -1 > gpurun_out/hs2.json
python -c "
import json
for f in ['gpurun_out/hs1.json','gpurun_out/hs2.json']:
    d=json.load(open(f)); print(f, d['value'], d['ms_per_step'], d['phases_ms'], d['e2e']['value'])
" >> gpurun_out/hs.log
