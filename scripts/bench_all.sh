#!/bin/bash
# Bench every BASELINE config at N=1 (GPU box). Usage: bench_all.sh <tag>
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
for C in ${CONFIGS:-1 2 3 4 5}; do
  EXTRA=""
  [ $C = 5 ] && EXTRA="--grad-pool 4"
  [ $C = 4 ] && EXTRA="--grad-pool 8"
  timeout 900 python bench.py --config $C --steps 20 --warmup 5 --no-e2e --no-cpu-baseline $EXTRA > $OUT/bench_C${C}_$TAG.json 2> $OUT/bench_C${C}_$TAG.err
  echo "C$C rc=$?"; tail -2 $OUT/bench_C${C}_$TAG.err
  python -c "
import json;d=json.load(open('$OUT/bench_C${C}_$TAG.json'))
print('C$C', d['config']['workload'], 'GB/s', round(d['value'],1), 'ms/step', round(d['ms_per_step'],3), 'stream frac', round(d['roofline']['frac'],3))
print('   ', {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items()})" 2>&1 | tail -3
done
