set -x
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_sw_r01.csv python bench.py --steps 2 --warmup 1 --no-cpu > gpurun_out/b_ncu.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_sw16 -c 3 -o gpurun_out/prof_sw16 python bench.py --steps 1 --warmup 0 --no-cpu > gpurun_out/prof.log 2>&1
tail -3 gpurun_out/prof.log
