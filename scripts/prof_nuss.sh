DP_NUSS5_N=3000 ncu --set full --clock-control none --import-source on -k regex:"k_nuss_batch" -c 1 -o gpurun_out/prof_nuss5 python bench.py --config nuss5 --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu -i gpurun_out/prof_nuss5.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_nuss5_src.csv 2>/dev/null
ls gpurun_out | grep nuss5
