ncu --set full --clock-control none --import-source on -k regex:"k_sw16" -c 2 -o gpurun_out/prof_sw2 python bench.py --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ls gpurun_out
