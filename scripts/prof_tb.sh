ncu --set full --clock-control none --import-source on -k regex:"k_sw16_tb" -c 1 -o gpurun_out/prof_tb4 python bench.py --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu -i gpurun_out/prof_tb4.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_tb4_src.csv 2>/dev/null
ls gpurun_out | grep tb4
