#!/bin/bash
# Round-1 GPU evidence: tests, bench, ncu launch list, ncu full captures of the top kernels.
# Usage (on the GPU box via gpurun): bash scripts/gpu_profile.sh <tag>
set -u
TAG=${1:-r01}
OUT=gpurun_out
mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > $OUT/gpu_tests_$TAG.log 2>&1
echo "tests rc=$?"; tail -3 $OUT/gpu_tests_$TAG.log
timeout 600 python bench.py --steps 10 --warmup 3 > $OUT/bench_$TAG.json 2> $OUT/bench_$TAG.err
echo "bench rc=$?"; cat $OUT/bench_$TAG.json; tail -5 $OUT/bench_$TAG.err
CMD="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_$TAG.csv $CMD > $OUT/ncu_launches_$TAG.out 2>&1
echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:stream_kernel -s 16 -c 1 -f -o $OUT/prof_stream_$TAG $CMD > $OUT/ncu_stream_$TAG.out 2>&1
echo "ncu stream rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dense_kernel -c 1 -f -o $OUT/prof_dense_$TAG $CMD > $OUT/ncu_dense_$TAG.out 2>&1
echo "ncu dense rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:merge_kernel -c 1 -f -o $OUT/prof_window_$TAG $CMD > $OUT/ncu_window_$TAG.out 2>&1
echo "ncu window rc=$?"
ls -la $OUT
timeout 600 ncu --set full --clock-control none --import-source on -k regex:starts_kernel -c 2 -f -o $OUT/prof_starts_$TAG $CMD > $OUT/ncu_starts_$TAG.out 2>&1
echo "ncu starts rc=$?"
