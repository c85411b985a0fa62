#!/bin/bash
# Round measurement: bench lines (default C5 + C3 + C2), ncu --set full of k_spmm (raw CSV), launch list.
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for c in ${BENCH_CONFIGS:-c5 c3 c2}; do
  timeout 1500 python bench.py --config $c --out gpurun_out/bench_$c.json > gpurun_out/bench_$c.log 2>&1; echo "bench $c rc=$?"
  python scripts/summ.py gpurun_out/bench_$c.json 2>&1 | head -12
done
for cp in ${PROFILES:-c5:cta_aware c3:cta_aware c3:identity c2:identity}; do
  c=${cp%%:*}; pol=${cp##*:}
  PENVS="def:PROF=1" CONFIG=$c POLICY=$pol bash scripts/gpu_prof_env.sh
done
if [ -z "$NO_LAUNCHES" ]; then
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
     python bench.py --steps 3 --warmup 3 --policy-steps 3 --e2e-steps 3 --no-cpu-baseline > gpurun_out/launches_bench.log 2>&1
  echo "launch list rc=$?"
fi
