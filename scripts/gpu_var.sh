#!/bin/bash
# A/B of run-time kernel variants: VARS="0 1 2 3" CONFIGS="c3 c2"
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for c in $CONFIGS; do
  for v in $VARS; do
    SPMM_VARIANT=$v timeout 1500 python bench.py --config $c --steps 10 --warmup 3 --policy-steps 5 --no-cpu-baseline --no-cusparse --no-ceiling --policies ${POLS:-identity,cta_aware} --out gpurun_out/var_${c}_$v.json > gpurun_out/var_${c}_$v.log 2>&1; echo "== $c var=$v rc=$?"
    python scripts/summ.py gpurun_out/var_${c}_$v.json 2>&1 | grep -E "^(value|identity|cta|nnz)"
  done
done
