python -m pytest tests -m gpu -q -x -k "forward or viterbi or hmm or nussinov" 2>&1 | tail -5
python bench.py --config hmm --steps 5 --warmup 3 --no-cpu 2>&1 | tail -1
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_hmm_r01.csv python bench.py --config hmm --steps 1 --warmup 1 --no-cpu > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_nuss5_r01.csv env DP_NUSS5_N=20000 python bench.py --config nuss5 --steps 1 --warmup 1 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_nuss_tiled -c 1 -o gpurun_out/prof_nuss5 env DP_NUSS5_N=3000 python bench.py --config nuss5 --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_forward|k_viterbi" -c 2 -o gpurun_out/prof_hmm python bench.py --config hmm --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ls gpurun_out
