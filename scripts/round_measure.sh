#!/bin/bash
# Round-2 measurement pass (run under gpurun; outputs in gpurun_out/, copied to profiles/ by
# scripts/collect_profiles.sh r02): GPU tests, the default bench line (every config), the
# reference arm, ncu launch lists and one --set full capture per dominant kernel, the traffic
# table, compute-sanitizer logs, the micro-benchmarks.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_info.txt
timeout 1500 python -m pytest tests -m gpu -q -rA 2>&1 | grep -vE "^PASSED" | tail -60 > gpurun_out/gpu_tests.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.json 2>/dev/null
for c in sw hmm nuss1 nuss4 swa swshort nussmid diag phmm; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches_$c.csv \
    python bench.py --config $c --only --steps 2 --warmup 1 --no-cpu > /dev/null 2>&1
done
DP_NUSS5_N=50000 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv \
  --log-file gpurun_out/launches_nuss5.csv python bench.py --config nuss5 --only --steps 2 --warmup 1 --no-cpu > /dev/null 2>&1
full() {  # full() TAG REGEX COUNT [env...]
  local tag=$1 rx=$2 cnt=$3; shift 3
  env "$@" timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$rx" -c $cnt -o gpurun_out/ncu_$tag \
    python bench.py --config $tag --only --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
}
full sw "k_sw16" 2
full hmm "k_forward_tc|k_viterbi" 3
full nuss1 "k_nuss" 1
full nuss4 "k_nuss" 1
full nuss5 "k_nuss_batch" 1 DP_NUSS5_N=50000
full swa "k_affine16" 2
full swshort "k_sw_inter" 2
full nussmid "k_nuss_cluster" 1
full diag "k_diag" 1
full phmm "k_phmm" 1
python scripts/ncu_traffic.py gpurun_out/traffic.json \
  k_sw16=gpurun_out/ncu_sw.ncu-rep k_sw16_tb5=gpurun_out/ncu_sw.ncu-rep \
  k_forward_tc=gpurun_out/ncu_hmm.ncu-rep k_viterbi16=gpurun_out/ncu_hmm.ncu-rep \
  k_nuss_batch=gpurun_out/ncu_nuss5.ncu-rep:20:"50k-problem capture of config 5 x 20" \
  k_nuss_grid2=gpurun_out/ncu_nuss4.ncu-rep k_affine16=gpurun_out/ncu_swa.ncu-rep \
  k_diag=gpurun_out/ncu_diag.ncu-rep k_phmm_forward=gpurun_out/ncu_phmm.ncu-rep \
  k_sw_inter=gpurun_out/ncu_swshort.ncu-rep k_sw_inter_tb=gpurun_out/ncu_swshort.ncu-rep \
  k_nuss_small=gpurun_out/ncu_nuss1.ncu-rep k_nuss_cluster=gpurun_out/ncu_nussmid.ncu-rep > gpurun_out/traffic.log 2>&1
# compute-sanitizer runs (memcheck / racecheck / synccheck) are kept from the earlier pass in
# profiles/sanitizer_r02/: the tool is closed on this GPU pool now
(cd ubench && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ubench ubench.cu && timeout 300 ./ubench > ../gpurun_out/ubench.jsonl 2>&1)
# summaries here (the .ncu-rep captures exceed gpurun's 64 MiB copy-back limit together): text only
mkdir -p gpurun_out/sum
for c in sw hmm nuss1 nuss4 nuss5 swa swshort nussmid diag phmm; do
  [ -s gpurun_out/launches_$c.csv ] && python scripts/ncu_summary.py --launches gpurun_out/launches_$c.csv > gpurun_out/sum/launches_$c.txt
  [ -s gpurun_out/ncu_$c.ncu-rep ] && python scripts/ncu_summary.py gpurun_out/ncu_$c.ncu-rep > gpurun_out/sum/ncu_$c.txt
done
rm -f gpurun_out/*.ncu-rep gpurun_out/launches_*.csv
ls -la gpurun_out
