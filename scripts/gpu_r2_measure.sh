#!/bin/bash
# Round-2 measurement session (one GPU box): bench lines (C5 default, C3, C2, shuffled C3/C5), one ncu --set full
# capture of every hot-path policy's k_spmm per config (roofline.traffic), the launch list of the default bench
# command, the reference arm, smoke.  Everything lands in gpurun_out/.
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
for c in ${CONFIGS:-c5 c3 c2 c3sh c5sh}; do
  extra=""
  case $c in c3sh|c5sh) extra="--no-cpu-baseline --no-cusparse";; esac
  timeout 1500 python bench.py --config $c $extra --out gpurun_out/bench_$c.json > gpurun_out/bench_$c.log 2>&1
  echo "bench $c rc=$?"
done
for c in ${PCONFIGS:-c5 c3 c2}; do
  timeout 1800 ncu --set full --clock-control none --import-source on -k regex:k_spmm -c 9 -f -o /tmp/prof_multi_$c \
     python scripts/profile_policies.py --config $c > gpurun_out/prof_multi_$c.log 2>&1
  echo "ncu multi $c rc=$?"
  ncu -i /tmp/prof_multi_$c.ncu-rep --page raw --csv > gpurun_out/prof_multi_$c.raw.csv 2>/dev/null
done
if [ -z "$NO_LAUNCHES" ]; then
  timeout 1800 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
     python bench.py --steps 3 --warmup 3 --policy-steps 3 --e2e-steps 3 --e2e-pipe-steps 3 --no-cpu-baseline \
     > gpurun_out/launches_bench.log 2>&1
  echo "launch list rc=$?"
fi
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/ref.log 2>&1; echo "reference rc=$?"
tail -2 gpurun_out/ref.log
