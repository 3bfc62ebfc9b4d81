python -m pytest tests -m gpu -q -x -k "diag or host or errors" 2>&1 | tail -15 > gpurun_out/gpu_tests_diag.log
python bench.py --config diag --steps 5 --warmup 3 2>gpurun_out/bench_diag.err | tail -1 > gpurun_out/bench_diag.json
