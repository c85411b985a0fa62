#!/bin/bash
# Round-end style session: smoke, all GPU tests (incl. full-size), sanitizers, default bench, launch list,
# ncu capture of the selected policy.
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"; tail -4 gpurun_out/gpu_tests.log
[ -n "$SANITIZE" ] && bash scripts/sanitize.sh
timeout 1500 python bench.py ${BENCH_ARGS} --out gpurun_out/bench.json > gpurun_out/bench.log 2>&1; echo "bench rc=$?"
python scripts/summ.py gpurun_out/bench.json | head -12
if [ -n "$LAUNCHES" ]; then
  timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv --log-file gpurun_out/launches.csv \
     python bench.py $LAUNCHES > gpurun_out/launches_bench.log 2>&1; echo "launches rc=$?"
fi
for cp in $PROFILES; do
  c=${cp%%:*}; pol=${cp##*:}
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 1 -c 1 -f -o gpurun_out/prof_${c}_$pol \
     python scripts/profile_spmm.py --config $c --policy $pol --runs 2 > gpurun_out/prof_${c}_$pol.log 2>&1; echo "prof $c $pol rc=$?"
done
