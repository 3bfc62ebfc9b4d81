python -m pytest tests -m gpu -q -x 2>&1 | tail -4
python bench.py --steps 10 --warmup 3 --no-cpu 2>&1 | tail -1 | cut -c1-400
python bench.py --config nuss4 --steps 3 --warmup 3 --no-cpu 2>&1 | tail -1 | cut -c1-300
DP_NUSS5_N=100000 python bench.py --config nuss5 --steps 2 --warmup 3 --no-cpu 2>&1 | tail -1 | cut -c1-300
ncu --set full --clock-control none --import-source on -k regex:"k_sw16_tb" -c 1 -o gpurun_out/prof_sw16tb python bench.py --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_forward" -c 1 -o gpurun_out/prof_fwd python bench.py --config hmm --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_nuss_tiled_grid" -c 1 -o gpurun_out/prof_nuss4 python bench.py --config nuss4 --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ls gpurun_out
