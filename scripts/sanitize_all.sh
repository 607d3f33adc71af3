#!/bin/bash
# compute-sanitizer over every kernel of the path (scripts/sanitize_path.py, C1-sized), both select
# variants; summaries under gpurun_out/sanitize_<tool>_<variant>.log (GPU box)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  for fast in 1 0; do
    extra=""
    [ $tool = memcheck ] && extra="--leak-check no"
    LOWDIFF_FAST_SELECT=$fast timeout 1200 /usr/local/cuda/bin/compute-sanitizer --tool $tool $extra \
      --print-limit 200 python scripts/sanitize_path.py \
      > gpurun_out/sanitize_${tool}_fast${fast}.log 2>&1
    echo "$tool fast=$fast rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/sanitize_${tool}_fast${fast}.log | tail -1)"
  done
done
