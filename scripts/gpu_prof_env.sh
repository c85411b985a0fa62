#!/bin/bash
# ncu --set full of the SpMM kernel under several env settings: PENVS="tag:K=V,K=V|tag2:..." CONFIG=c3 POLICY=cta_aware
# Only the raw-page CSV comes back (the .ncu-rep files are too large for gpurun_out) unless KEEP_REP=1.
mkdir -p gpurun_out
IFS='|' read -ra LIST <<< "$PENVS"
for e in "${LIST[@]}"; do
  tag=${e%%:*}; kv=${e#*:}
  out=gpurun_out/prof_${CONFIG:-c3}_${POLICY:-cta_aware}_$tag
  env $(echo $kv | tr ',' ' ') timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-k_spmm} -s ${SKIP:-1} -c 1 -f \
     -o /tmp/prof_$tag python scripts/profile_spmm.py --config ${CONFIG:-c3} --policy ${POLICY:-cta_aware} --runs 2 \
     > $out.log 2>&1; echo "prof $tag rc=$?"
  ncu -i /tmp/prof_$tag.ncu-rep --page raw --csv > $out.raw.csv 2>/dev/null
  ncu -i /tmp/prof_$tag.ncu-rep --page details --csv > $out.details.csv 2>/dev/null
  if [ -n "$KEEP_REP" ]; then cp /tmp/prof_$tag.ncu-rep $out.ncu-rep; fi
done
