#!/bin/bash
# ncu --set full of one k_spmm launch per env setting, exported on the box (raw + SASS source pages as CSV):
#   PROF_ENVS="SPMM_FUSE_PIPE=0 SPMM_FUSE_PIPE=2" PCONFIG=c2 PPOL=identity bash scripts/prof_env.sh
mkdir -p gpurun_out
for e in $PROF_ENVS; do
  tag=${PCONFIG:-c2}_${PPOL:-identity}_$(echo $e | tr '=' '_')
  env $e timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 1 -c 1 -f -o /tmp/prof_$tag \
     python scripts/profile_spmm.py --config ${PCONFIG:-c2} --policy ${PPOL:-identity} --runs 2 > gpurun_out/prof_$tag.log 2>&1; echo "prof $e rc=$?"
  ncu -i /tmp/prof_$tag.ncu-rep --page raw --csv > gpurun_out/raw_$tag.csv 2>/dev/null
  ncu -i /tmp/prof_$tag.ncu-rep --page source --csv --print-source sass > gpurun_out/sass_$tag.csv 2>/dev/null
  ncu -i /tmp/prof_$tag.ncu-rep --page details --csv > gpurun_out/details_$tag.csv 2>/dev/null
  [ -n "$KEEP_REP" ] && cp /tmp/prof_$tag.ncu-rep gpurun_out/
done
ls -la gpurun_out
