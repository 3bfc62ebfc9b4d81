for k in 16 12 10 8; do
  DP_NUSS_BATCH_PER_SM=$k DP_NUSS5_N=200000 python bench.py --config nuss5 --steps 2 --warmup 1 --no-cpu 2>/dev/null | tail -1 > gpurun_out/nb_$k.json
  python -c "import json; d=json.load(open('gpurun_out/nb_$k.json')); print($k, d['value'], d['ms_per_step'])" >> gpurun_out/nb.log
done
