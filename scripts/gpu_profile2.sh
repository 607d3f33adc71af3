#!/bin/bash
# tests + bench + launch list + full ncu captures of a kernel list. Usage: gpu_profile2.sh <tag> <regex>...
set -u
TAG=$1; shift
OUT=gpurun_out
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > $OUT/gpu_tests_$TAG.log 2>&1
echo "tests rc=$?"; tail -3 $OUT/gpu_tests_$TAG.log
timeout 600 python bench.py --steps 10 --warmup 3 > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err
echo "bench rc=$?"; tail -5 $OUT/bench_$TAG.err
CMD="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$TAG.csv $CMD > $OUT/ncu_launches_$TAG.out 2>&1
echo "ncu launches rc=$?"
for K in "$@"; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$K -s 2 -c 1 -f -o $OUT/prof_${K}_$TAG $CMD > $OUT/ncu_${K}_$TAG.out 2>&1
  echo "ncu $K rc=$?"
done
