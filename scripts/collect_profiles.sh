#!/bin/bash
# Copy a scripts/round_measure.sh pass from gpurun_out/ into profiles/ (suffix $1, e.g. r02)
R=${1:-r02}
cp gpurun_out/bench.json profiles/bench_$R.json
cp gpurun_out/bench_ref.json profiles/bench_ref_$R.json
cp gpurun_out/gpu_tests.log profiles/gpu_tests_$R.log
[ -s gpurun_out/traffic.json ] && cp gpurun_out/traffic.json profiles/traffic_$R.json
[ -s gpurun_out/ubench.jsonl ] && cp gpurun_out/ubench.jsonl profiles/ubench_$R.jsonl
for c in sw hmm nuss1 nuss4 nuss5 swa swshort nussmid diag phmm; do  # summaries written on the box
  [ -s gpurun_out/sum/launches_$c.txt ] && cp gpurun_out/sum/launches_$c.txt profiles/launches_${c}_$R.txt
  [ -s gpurun_out/sum/ncu_$c.txt ] && cp gpurun_out/sum/ncu_$c.txt profiles/ncu_${c}_$R.txt
done
if ls gpurun_out/san/*.log > /dev/null 2>&1; then
  mkdir -p profiles/sanitizer_$R
  for f in gpurun_out/san/*.log; do tail -25 "$f" > profiles/sanitizer_$R/$(basename "$f"); done
fi
