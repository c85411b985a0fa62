#!/bin/bash
# GPU-box check: smoke, GPU parity tests, a short bench run. Logs land in gpurun_out/.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu_info.txt
nproc >> gpurun_out/gpu_info.txt; free -g >> gpurun_out/gpu_info.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout ${TESTS_TIMEOUT:-1500} python -m pytest tests -m gpu -q --timeout 600 ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"
tail -30 gpurun_out/gpu_tests.log
if [ -n "$BENCH" ]; then
  timeout 900 python bench.py $BENCH --out gpurun_out/bench.json > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
  tail -c 3000 gpurun_out/bench.log
fi
