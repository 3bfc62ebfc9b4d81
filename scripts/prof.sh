#!/bin/bash
# One `ncu --set full` capture of the first launch of kernel regex $1 in `bench.py $2`, tagged $3:
# gpurun_out/prof_$3.ncu-rep plus its summary and top SASS lines by stall samples.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$1" -c 1 -o gpurun_out/prof_$3 \
  python bench.py $2 --no-cpu --only > gpurun_out/prof_$3.log 2>&1
python scripts/ncu_summary.py gpurun_out/prof_$3.ncu-rep > gpurun_out/prof_$3_summary.txt 2>&1
ncu -i gpurun_out/prof_$3.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_$3_src.csv 2>/dev/null
python scripts/ncu_src_top.py gpurun_out/prof_$3_src.csv 60 > gpurun_out/prof_$3_top.txt 2>&1
rm -f gpurun_out/prof_$3_src.csv
echo done
