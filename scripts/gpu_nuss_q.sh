python -m pytest tests -m gpu -q -x -k "nussinov" 2>&1 | tail -3 > gpurun_out/gpu_tests_nuss.log
python bench.py --config nuss4 --steps 3 --warmup 2 --no-cpu 2>/dev/null | tail -1 > gpurun_out/bn4.json
DP_NUSS5_N=200000 python bench.py --config nuss5 --steps 2 --warmup 1 --no-cpu 2>/dev/null | tail -1 > gpurun_out/bn5.json
python -c "
import json
for f in ['gpurun_out/bn4.json','gpurun_out/bn5.json']:
    d=json.load(open(f)); print(f, d['value'], d['ms_per_step'], d['roofline']['frac'])
" >> gpurun_out/gpu_tests_nuss.log 2>&1
