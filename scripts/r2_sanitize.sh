#!/bin/bash
# compute-sanitizer over scripts/sanitize_cases.py (every kernel family, small sizes)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/san
for tool in memcheck racecheck synccheck initcheck; do
  extra=""
  [ "$tool" = "memcheck" ] && extra="--leak-check no"
  [ "$tool" = "racecheck" ] && extra="--racecheck-report hazard"
  timeout 1500 /usr/local/cuda/bin/compute-sanitizer --tool $tool $extra --print-limit 40 \
    python scripts/sanitize_cases.py > gpurun_out/san/$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/san/summary.txt
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|ALL OK|FAILED|MISMATCH" gpurun_out/san/$tool.log >> gpurun_out/san/summary.txt
done
cat gpurun_out/san/summary.txt
