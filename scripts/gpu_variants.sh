# usage: bash scripts/gpu_variants.sh [bench args...]  — one bench line per exp/libdp_*.so plus the in-tree build
for lib in paper_conf_pldi_carteylm12_b200/libdp.so exp/libdp_*.so; do
  DP_LIB=$PWD/$lib python bench.py --steps ${STEPS:-10} --warmup 3 --no-cpu "$@" 2>/dev/null | tail -1 > gpurun_out/v.json
  python -c "import json,sys; d=json.load(open('gpurun_out/v.json')); print(sys.argv[1], d['value'], d['ms_per_step'], d.get('phases_ms'))" $lib >> gpurun_out/variants.log
done
