bash scripts/gpu_sw.sh
bash scripts/prof_tb.sh
