#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
if [ -z "$SKIP_TESTS" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -x --timeout 600 > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/gpu_tests.log
fi
for c in $CONFIGS; do
  for sch in ${SCHEDS:-1}; do
    SPMM_SCHED=$sch timeout 1500 python bench.py --config $c ${BENCH_ARGS:---steps 10 --warmup 3 --policy-steps 5 --no-cpu-baseline} --out gpurun_out/bench_${c}_s$sch.json > gpurun_out/bench_${c}_s$sch.log 2>&1; echo "bench $c sched=$sch rc=$?"
    python scripts/summ.py gpurun_out/bench_${c}_s$sch.json 2>&1 | head -12
  done
done
for cp in $PROFILES; do
  c=${cp%%:*}; pol=${cp##*:}
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 1 -c 1 -f -o gpurun_out/prof_${c}_$pol \
     python scripts/profile_spmm.py --config $c --policy $pol --runs 2 > gpurun_out/prof_${c}_$pol.log 2>&1; echo "prof $c $pol rc=$?"
done
if [ -n "$CORPUS" ]; then
  timeout 3000 python scripts/corpus.py $CORPUS --out gpurun_out/corpus.jsonl > gpurun_out/corpus.log 2>&1; echo "corpus rc=$?"; tail -3 gpurun_out/corpus.log
fi
