#!/bin/bash
# compute-sanitizer over the small cases of tests/tools/sanitize_cases.py (run on the GPU box):
#   bash scripts/sanitize.sh [outdir]
# One log per tool and case; the summary line of each log ("ERROR SUMMARY: n errors") is what
# profiles/sanitizer_r02.md records.
out=${1:-gpurun_out/sanitizer}
mkdir -p "$out"
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in ${VB_SAN_TOOLS:-memcheck synccheck racecheck}; do
  for c in ${VB_SAN_CASES:-c1 ragged_bf16 ragged_f32 pair w2 conv graph}; do
    timeout ${VB_SAN_TIMEOUT:-300} $CS --tool $tool --print-limit 20 --error-exitcode 9 --target-processes all \
      python tests/tools/sanitize_cases.py $c > "$out/${tool}_${c}.log" 2>&1
    echo "$tool $c rc=$? $(grep -h 'ERROR SUMMARY' "$out/${tool}_${c}.log" | tail -1) $(grep -h 'parity ok' "$out/${tool}_${c}.log")"
  done
done | tee "$out/summary.txt"
