#!/bin/bash
# Select grid sweep (GPU box). Usage: select_variants.sh "16 37 74 148 296" "1 2 3"
OUT=gpurun_out; mkdir -p $OUT
for GQ in $1; do
  for C in $2; do
    EXTRA=""; [ $C = 5 ] && EXTRA="--grad-pool 4"; [ $C = 4 ] && EXTRA="--grad-pool 8"
    LOWDIFF_SELECT_GRID=$GQ timeout 600 python bench.py --config $C --steps 5 --warmup 3 --no-e2e --no-cpu-baseline $EXTRA > $OUT/bench_selg_${GQ}_C$C.json 2>/dev/null
    python -c "import json;d=json.load(open('$OUT/bench_selg_${GQ}_C$C.json'));k=d['kernels'];s=k['compress_select'];print('grid=$GQ C$C', round(d['ms_per_step'],3), 'select us/call', round(1000*s['ms_per_step']/s['launches_per_step'],1))"
  done
done
