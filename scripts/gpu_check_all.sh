#!/bin/bash
# Full GPU test suite + default bench line (every config); outputs in gpurun_out/.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -rA 2>&1 | grep -vE "^PASSED" | tail -60 > gpurun_out/gpu_tests.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
echo done
