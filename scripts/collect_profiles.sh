#!/bin/bash
# Copy a scripts/round_measure.sh pass from gpurun_out/ into profiles/ (suffix $1, e.g. r02)
R=${1:-r02}
cp gpurun_out/bench.json profiles/bench_$R.json
cp gpurun_out/bench_ref.json profiles/bench_ref_$R.json
cp gpurun_out/gpu_tests.log profiles/gpu_tests_$R.log
[ -s gpurun_out/traffic.json ] && cp gpurun_out/traffic.json profiles/traffic_$R.json
[ -s gpurun_out/ubench.jsonl ] && cp gpurun_out/ubench.jsonl profiles/ubench_$R.jsonl
for c in sw hmm nuss1 nuss4 nuss5 swa swshort nussmid diag phmm; do
  [ -s gpurun_out/launches_$c.csv ] && python scripts/ncu_summary.py --launches gpurun_out/launches_$c.csv > profiles/launches_${c}_$R.txt
  [ -s gpurun_out/ncu_$c.ncu-rep ] && python scripts/ncu_summary.py gpurun_out/ncu_$c.ncu-rep > profiles/ncu_${c}_$R.txt
done
mkdir -p profiles/sanitizer_$R
for f in gpurun_out/san/*.log; do tail -25 "$f" > profiles/sanitizer_$R/$(basename "$f"); done
