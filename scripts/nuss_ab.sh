#!/bin/bash
# Nussinov A/B: GPU parity tests for the Nussinov kernels, then bench lines for configs 5, 4, nussmid.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "nuss" 2>&1 | tail -2
for c in nuss5 nuss4 nussmid; do
  timeout 600 python bench.py --config $c --only --steps 3 --warmup 3 --no-cpu > gpurun_out/ab_$c.json 2>gpurun_out/ab_$c.err
  python -c "import json; d=json.load(open('gpurun_out/ab_$c.json')); print('$c', d['value'], d['ms_per_step'], d['roofline']['frac'], d.get('result_sha256','')[:16])"
done
