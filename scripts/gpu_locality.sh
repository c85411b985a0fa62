#!/bin/bash
# Locality recovery (§III.B, Fig. 7): on inputs whose original order has no row locality
# (c3sh: C3 with its rows shuffled; c3rl / c5rl: random-label R-MAT), every hot-path policy is built and timed by
# bench.py (with the LRU-model L2 ceiling per order), then one k_spmm launch per policy is captured by ncu with the
# L2 / DRAM counters.  Outputs: gpurun_out/loc_<config>.json (bench line), gpurun_out/loc_ncu_<config>_<policy>.csv.
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
POLS=${POLS:-identity,nnz_sort,plain_sort,cta_aware,hybrid_1,hybrid_2_1,cta_aware+mh,cta_aware+md,hybrid_2_1+md}
NCU_POLS=${NCU_POLS:-identity nnz_sort cta_aware hybrid_2_1 cta_aware+mh cta_aware+md hybrid_2_1+md}
METRICS=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,\
lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,\
l1tex__t_sector_hit_rate.pct,lts__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__m_xbar2l1tex_read_bytes.sum
for c in ${LOC_CONFIGS:-c3sh c3rl}; do
  timeout 1500 python bench.py --config $c --policies $POLS --steps 5 --warmup 3 --no-cpu-baseline \
     ${BENCH_EXTRA:---no-cusparse} --out gpurun_out/loc_$c.json > gpurun_out/loc_$c.log 2>&1
  echo "bench $c rc=$?"
  for pol in $NCU_POLS; do
    timeout 900 ncu --metrics $METRICS --clock-control none -k regex:k_spmm -s 1 -c 1 --csv \
       --log-file gpurun_out/loc_ncu_${c}_${pol}.csv python scripts/profile_spmm.py --config $c --policy $pol --runs 2 \
       > gpurun_out/loc_ncu_${c}_${pol}.log 2>&1
    echo "ncu $c $pol rc=$?"
  done
done
