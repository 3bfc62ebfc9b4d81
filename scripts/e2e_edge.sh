#!/bin/bash
# e2e of a config at several (host chunks, edge fraction) settings: $1 = config, then "chunks:edge" pairs
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
c=$1; shift
for ce in "$@"; do
  n=${ce%%:*}; f=${ce##*:}
  DP_HOST_CHUNKS=$n DP_HOST_EDGE=$f timeout 300 python bench.py --config $c --only --steps 10 --warmup 3 --no-cpu > gpurun_out/edge_${c}_${n}_$f.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/edge_${c}_${n}_$f.json')); print('$c chunks=$n edge=$f', d['ms_per_step'], d['e2e']['value'], d['e2e']['ms_per_step'], d.get('result_sha256'))"
done
