#!/bin/bash
# A/B over environment settings: ENVS="SPMM_KERNEL=1|SPMM_KERNEL=3,SPMM_AFF_V=2" CONFIGS="c3 c2"
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
if [ -n "$PYTEST_K" ]; then
  timeout 1800 python -m pytest tests -m gpu -q -x --timeout 900 -k "$PYTEST_K" > gpurun_out/gpu_tests_k.log 2>&1; echo "tests($PYTEST_K) rc=$?"; tail -3 gpurun_out/gpu_tests_k.log
fi
IFS='|' read -ra LIST <<< "$ENVS"
for c in $CONFIGS; do
  i=0
  for e in "${LIST[@]}"; do
    i=$((i+1))
    env $(echo $e | tr ',' ' ') timeout 1500 python bench.py --config $c --steps 10 --warmup 3 --policy-steps 5 --no-cpu-baseline --no-cusparse --no-ceiling --policies ${POLS:-identity,cta_aware} --out gpurun_out/env_${c}_$i.json > gpurun_out/env_${c}_$i.log 2>&1; echo "== $c [$e] rc=$?"
    python scripts/summ.py gpurun_out/env_${c}_$i.json 2>&1 | grep -E "^(value|identity|cta|nnz|hybrid|plain)"
  done
done
