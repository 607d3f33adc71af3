#!/bin/bash
# compute-sanitizer over every kernel of the path (scripts/sanitize_path.py, C1-sized): the fast and
# general grid selects and the opt-in one-CTA select; summaries under
# gpurun_out/sanitize_<tool>_<variant>.log (GPU box)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck initcheck; do
  for v in fast1 fast0 small; do
    extra=""
    [ $tool = memcheck ] && extra="--leak-check no"
    fast=1; small=0
    [ $v = fast0 ] && fast=0
    [ $v = small ] && small=1
    LOWDIFF_FAST_SELECT=$fast LOWDIFF_SELECT_SMALL=$small timeout 1200 /usr/local/cuda/bin/compute-sanitizer \
      --tool $tool $extra --print-limit 200 python scripts/sanitize_path.py \
      > gpurun_out/sanitize_${tool}_${v}.log 2>&1
    echo "$tool $v rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/sanitize_${tool}_${v}.log | tail -1)"
  done
done
