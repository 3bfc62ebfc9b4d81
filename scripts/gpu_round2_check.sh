#!/bin/bash
# GPU check: the -m gpu suite (config-4 golden deselected until it exists), smoke, the default bench line.
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
DESEL=""
[ -f tests/golden/config4.json ] || DESEL="--deselect tests/test_gpu_parity.py::test_nussinov_config4_golden"
timeout 1200 python -m pytest tests -m gpu -q $DESEL -rA 2>&1 | tail -80 > gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
echo done
