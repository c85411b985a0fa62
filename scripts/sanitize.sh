#!/bin/bash
# compute-sanitizer over the whole hot path on a C1-sized matrix (every kernel: builders, chains, SpMM,
# features). Logs in gpurun_out/sanitize_*.log
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  timeout ${SAN_TIMEOUT:-1500} /usr/local/cuda/bin/compute-sanitizer --tool $tool --error-exitcode 9 --target-processes all \
     python scripts/sanitize_driver.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$? $(grep -c 'ERROR SUMMARY: 0 errors' gpurun_out/sanitize_$tool.log) clean-summaries"
  grep "ERROR SUMMARY" gpurun_out/sanitize_$tool.log | tail -1
done
