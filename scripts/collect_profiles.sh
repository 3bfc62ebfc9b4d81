# Copy a round_measure.sh pass from gpurun_out/ into profiles/ (suffix $1, e.g. r01)
R=${1:-r01}
for c in sw ref hmm nuss1 nuss4 nuss5; do cp gpurun_out/bench_$c.json profiles/bench_${c}_$R.json; done
cp gpurun_out/gpu_tests.log profiles/gpu_tests_$R.log
for c in sw hmm nuss4 nuss5; do
  python scripts/ncu_summary.py --launches gpurun_out/launches_$c.csv > profiles/launches_${c}_$R.txt
  python scripts/ncu_summary.py gpurun_out/ncu_$c.ncu-rep > profiles/ncu_${c}_$R.txt
done
