#!/bin/bash
# N = 1 vs N = 2 ranks on one GPU (DP_BENCH_BACKEND=gloo test hook): the sharded path's gathered
# outputs must hash the same as N = 1 for every batched config.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
for c in sw swa swshort hmm phmm diag nuss5; do
  h1=$(DP_NUSS5_N=20000 timeout 300 python bench.py --config $c --only --steps 2 --warmup 3 --no-cpu 2>/dev/null | tail -1 | python -c "import json,sys; print(json.loads(sys.stdin.read()).get('result_sha256'))")
  h2=$(DP_NUSS5_N=20000 DP_BENCH_BACKEND=gloo timeout 600 python bench.py --gpus 2 --config $c --only --steps 2 --warmup 3 --no-cpu 2>/dev/null | tail -1 | python -c "import json,sys; print(json.loads(sys.stdin.read()).get('result_sha256'))")
  echo "$c N1=$h1 N2=$h2 $([ "$h1" = "$h2" ] && echo same || echo DIFFERENT)"
done
