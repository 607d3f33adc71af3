#!/bin/bash
# Everything profiles/ holds for one round tag, in one GPU call:
#   full GPU tests, the default bench line (C3 + e2e + cpu_baseline), every config (C1..C5),
#   the ncu launch list, ncu --set full captures of the hot kernels, in-loop and recovery benches.
# Usage: gpu_round_profile.sh <tag>
set -u
TAG=$1; OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider > $OUT/gpu_tests_$TAG.log 2>&1
echo "tests rc=$?"; tail -1 $OUT/gpu_tests_$TAG.log
timeout 900 python bench.py > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err
echo "bench rc=$?"; tail -2 $OUT/bench_$TAG.err
bash scripts/bench_all.sh $TAG
CMD="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$TAG.csv $CMD > /dev/null 2>&1
echo "ncu launches rc=$?"
for K in stream_kernel select_kernel merge_kernel dense_kernel starts4_kernel; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$K -s 3 -c 1 -f -o /tmp/prof_${K}_$TAG $CMD > /dev/null 2>&1
  echo "ncu $K rc=$?"
  cp /tmp/prof_${K}_$TAG.ncu-rep $OUT/ 2>/dev/null
done
for C in 2 3 4; do
  timeout 600 python scripts/bench_inloop.py --config $C --iters 128 > $OUT/inloop_C${C}_$TAG.json 2> $OUT/inloop_C${C}_$TAG.err
  echo "inloop C$C rc=$?"
done
timeout 600 python scripts/bench_recovery.py > $OUT/recovery_$TAG.json 2> $OUT/recovery_$TAG.err
echo "recovery rc=$?"
python scripts/ncu_summarize.py $OUT/ncu_summary_$TAG.json /tmp/prof_*_$TAG.ncu-rep > /dev/null 2>&1
echo "summary rc=$?"
