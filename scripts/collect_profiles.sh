# Copy a round_measure.sh pass from gpurun_out/ into profiles/ (suffix $1, e.g. r01)
R=${1:-r01}
for c in sw ref swa hmm nuss1 nuss4 nuss5 diag; do
  [ -s gpurun_out/bench_$c.json ] && cp gpurun_out/bench_$c.json profiles/bench_${c}_$R.json
done
cp gpurun_out/gpu_tests.log profiles/gpu_tests_$R.log
for c in sw hmm nuss4 nuss5 diag; do
  [ -s gpurun_out/launches_$c.csv ] && python scripts/ncu_summary.py --launches gpurun_out/launches_$c.csv > profiles/launches_${c}_$R.txt
done
for c in sw hmm nuss4 nuss5 diag swa; do
  [ -s gpurun_out/ncu_$c.ncu-rep ] && python scripts/ncu_summary.py gpurun_out/ncu_$c.ncu-rep > profiles/ncu_${c}_$R.txt
done
# instruction mix of the SW kernels (sweep + traceback), from the source page
ncu -i gpurun_out/ncu_sw.ncu-rep --page source --csv --print-source sass > /tmp/ncu_sw_src.csv 2>/dev/null && \
  python scripts/ncu_mix.py /tmp/ncu_sw_src.csv > profiles/ncu_sw_mix_$R.txt
