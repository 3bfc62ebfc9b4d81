#!/bin/bash
# Quick GPU check of selected tests (-k expression in $1) and optional bench args ($2).
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -k "$1" -rA 2>&1 | grep -vE "^(PASSED|\.)" | tail -60 > gpurun_out/quick_pytest.log
if [ -n "$2" ]; then timeout 900 python bench.py $2 > gpurun_out/quick_bench.json 2> gpurun_out/quick_bench.err; fi
echo done
