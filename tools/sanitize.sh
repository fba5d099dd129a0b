#!/bin/bash
# compute-sanitizer over tools/sanitize_cases.py: memcheck, racecheck (shared-memory hazards),
# synccheck (barrier misuse), initcheck.  Summaries go to $OUT (default gpurun_out/sanitize).
OUT=${OUT:-gpurun_out/sanitize}
mkdir -p "$OUT"
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 /usr/local/cuda/bin/compute-sanitizer --tool $tool --launch-timeout 120 --print-limit 2000 \
    --error-exitcode 9 python tools/sanitize_cases.py > "$OUT/$tool.log" 2>&1
  echo "$tool rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' "$OUT/$tool.log" | tail -1)"
done
