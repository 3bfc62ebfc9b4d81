for k in 1 2 3 4 6; do
  DP_HMM_NS=$k ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_viterbi -c 2 --csv --log-file gpurun_out/ns_$k.csv python bench.py --config hmm --steps 1 --warmup 1 --no-cpu > /dev/null 2>&1
  echo "NS=$k" >> gpurun_out/ns.log; python scripts/ncu_summary.py --launches gpurun_out/ns_$k.csv | head -3 >> gpurun_out/ns.log
done
