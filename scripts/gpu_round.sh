#!/bin/bash
# One GPU-box session: tests, bench, launch list and ncu captures. Everything lands in gpurun_out/.
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
if [ -z "$SKIP_TESTS" ]; then
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
  timeout ${TESTS_TIMEOUT:-1500} python -m pytest tests -m gpu -q --timeout 600 ${PYTEST_K:+-k "$PYTEST_K"} > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"
  tail -15 gpurun_out/gpu_tests.log
fi
if [ -n "$BENCH" ]; then
  timeout 1200 python bench.py $BENCH --out gpurun_out/bench.json > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
  tail -c 1500 gpurun_out/bench.log
fi
if [ -n "$LAUNCHES" ]; then
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/launches.csv \
     python bench.py $LAUNCHES > gpurun_out/launches_bench.log 2>&1; echo "launches rc=$?"
fi
for pol in $PROFILE; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 1 -c 1 -f -o gpurun_out/prof_${PCONFIG:-c3}_$pol \
     python scripts/profile_spmm.py --config ${PCONFIG:-c3} --policy $pol --runs 2 > gpurun_out/prof_$pol.log 2>&1; echo "prof $pol rc=$?"
done
