#!/bin/bash
# usage: scripts/gpu_variants.sh "<bench args>" name1 name2 ...  (exp/libdp_<name>.so; "main" = in-tree)
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
args="$1"; shift
for v in "$@"; do
  if [ "$v" = main ]; then lib=""; else lib="$PWD/exp/libdp_$v.so"; fi
  DP_LIB=$lib timeout 600 python bench.py $args --no-cpu > gpurun_out/var_$v.json 2> gpurun_out/var_$v.err
  python -c "import json,sys; d=json.load(open('gpurun_out/var_$v.json')); print('$v', d['ms_per_step'], d['phases_ms'], d.get('intra_task_ms'))" >> gpurun_out/variants.txt 2>&1
done
