ncu --set full --clock-control none --import-source on -k regex:"k_viterbi" -c 1 -o gpurun_out/prof_vit python bench.py --config hmm --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ls gpurun_out | grep vit
