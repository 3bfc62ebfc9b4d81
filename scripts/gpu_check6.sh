timeout 300 python scripts/nuss_tb_probe.py 20000
python -m pytest tests -m gpu -q -x -k "nussinov" 2>&1 | tail -2
ncu --set full --clock-control none --import-source on -k regex:"k_nuss_tiled_cta" -c 1 -o gpurun_out/prof_nuss5b env DP_NUSS5_N=3000 python bench.py --config nuss5 --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_sw16_tb|k_viterbi<" -c 2 -o gpurun_out/prof_tb2 python bench.py --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ls gpurun_out
