#!/bin/bash
# e2e (dp_solve_batch_host) of one bench config at several host chunk counts: $1 = config, rest = counts
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
c=$1; shift
for n in "$@"; do
  DP_HOST_CHUNKS=$n timeout 300 python bench.py --config $c --only --steps 5 --warmup 3 --no-cpu > gpurun_out/e2e_${c}_$n.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/e2e_${c}_$n.json')); print('$c chunks=$n', d['ms_per_step'], d['e2e']['value'], d['e2e']['ms_per_step'])"
done
