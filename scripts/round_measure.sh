# Full measurement pass (run under gpurun): tests, bench lines for every config,
# launch lists and ncu captures of the dominant kernels. Outputs in gpurun_out/.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_info.txt
python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/gpu_tests.log
python bench.py 2>gpurun_out/bench_sw.err | tail -1 > gpurun_out/bench_sw.json
python bench.py --impl reference --steps 3 --warmup 1 2>/dev/null | tail -1 > gpurun_out/bench_ref.json
python bench.py --config swa --warmup 3 2>/dev/null | tail -1 > gpurun_out/bench_swa.json
python bench.py --config hmm --warmup 3 2>/dev/null | tail -1 > gpurun_out/bench_hmm.json
python bench.py --config nuss1 --warmup 5 2>/dev/null | tail -1 > gpurun_out/bench_nuss1.json
python bench.py --config nuss4 --warmup 3 2>/dev/null | tail -1 > gpurun_out/bench_nuss4.json
python bench.py --config nuss5 --steps 2 --warmup 3 2>gpurun_out/bench_nuss5.err | tail -1 > gpurun_out/bench_nuss5.json
python bench.py --config diag --warmup 3 2>/dev/null | tail -1 > gpurun_out/bench_diag.json
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_sw.csv python bench.py --steps 2 --warmup 1 --no-cpu > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_hmm.csv python bench.py --config hmm --steps 2 --warmup 1 --no-cpu > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_nuss4.csv python bench.py --config nuss4 --steps 2 --warmup 1 --no-cpu > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_nuss5.csv env DP_NUSS5_N=50000 python bench.py --config nuss5 --steps 2 --warmup 1 --no-cpu > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 12 --csv --log-file gpurun_out/launches_diag.csv python bench.py --config diag --steps 2 --warmup 1 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_sw16" -c 2 -o gpurun_out/ncu_sw python bench.py --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_forward_tc|k_viterbi" -c 3 -o gpurun_out/ncu_hmm python bench.py --config hmm --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_nuss" -c 1 -o gpurun_out/ncu_nuss4 python bench.py --config nuss4 --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_nuss" -c 1 -o gpurun_out/ncu_nuss5 env DP_NUSS5_N=50000 python bench.py --config nuss5 --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_diag|k_align_affine" -c 2 -o gpurun_out/ncu_diag python bench.py --config diag --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"k_align_affine" -c 2 -o gpurun_out/ncu_swa python bench.py --config swa --steps 1 --warmup 0 --no-cpu > /dev/null 2>&1
ls -la gpurun_out
