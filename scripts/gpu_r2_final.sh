#!/bin/bash
# Round-2 closing session (one GPU box): smoke, the GPU test suite, then the measurement session at HEAD
# (scripts/gpu_r2_measure.sh: bench lines, per-policy ncu captures, launch list, reference arm).
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"
tail -3 gpurun_out/gpu_tests.log
CONFIGS="${CONFIGS:-c5 c3 c2 c3sh c5sh}" bash scripts/gpu_r2_measure.sh
