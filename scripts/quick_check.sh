#!/bin/bash
# Fast GPU iteration loop: replay/update parity tests + C3/C4 benches. Usage: quick_check.sh <tag> [pytest -k expr]
TAG=${1:-q}; K=${2:-"replay or update or in_loop or end_to_end"}
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x -k "$K" -p no:cacheprovider > $OUT/quick_tests_$TAG.log 2>&1
echo "tests rc=$?"; tail -2 $OUT/quick_tests_$TAG.log
for C in ${CONFIGS:-3 4}; do
  EXTRA=""; [ $C = 4 ] && EXTRA="--grad-pool 8"; [ $C = 5 ] && EXTRA="--grad-pool 4"
  timeout 600 python bench.py --config $C --steps 10 --warmup 3 --no-e2e --no-cpu-baseline $EXTRA > $OUT/quick_C${C}_$TAG.json 2> $OUT/quick_C${C}_$TAG.err
  python -c "
import json;d=json.load(open('$OUT/quick_C${C}_$TAG.json'))
print('C$C', 'GB/s', round(d['value'],1), 'ms/step', round(d['ms_per_step'],3), 'stream frac', round(d['roofline']['frac'],3))
print('   ', {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items()})" 2>&1 | tail -3
done
