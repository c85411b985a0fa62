#!/bin/bash
# run several bench configs + profiles: CONFIGS="c2 c5" PROFILES="c2:identity c2:nnz_sort"
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for c in $CONFIGS; do
  timeout 1500 python bench.py --config $c ${BENCH_ARGS:---steps 10 --warmup 3 --policy-steps 5} --out gpurun_out/bench_$c.json > gpurun_out/bench_$c.log 2>&1; echo "bench $c rc=$?"
  python scripts/summ.py gpurun_out/bench_$c.json 2>&1 | head -12
done
for cp in $PROFILES; do
  c=${cp%%:*}; pol=${cp##*:}
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 1 -c 1 -f -o gpurun_out/prof_${c}_$pol \
     python scripts/profile_spmm.py --config $c --policy $pol --runs 2 > gpurun_out/prof_${c}_$pol.log 2>&1; echo "prof $c $pol rc=$?"
done
