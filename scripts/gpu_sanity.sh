# Quick sanity pass: GPU tests + default bench line (+ affine SW line).
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_info.txt
python -m pytest tests -m gpu -q -x 2>&1 | tail -15 > gpurun_out/gpu_tests.log
python bench.py 2>gpurun_out/bench_sw.err | tail -1 > gpurun_out/bench_sw.json
python bench.py --config swa --steps 5 --warmup 3 2>/dev/null | tail -1 > gpurun_out/bench_swa.json
