ncu --set full --clock-control none --import-source on -k regex:"k_sw16_tb" -c 1 -o gpurun_out/prof_tb6 python bench.py --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ls gpurun_out | grep tb6
