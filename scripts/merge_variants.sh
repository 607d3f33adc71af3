#!/bin/bash
# Merge sparse/dense item threshold sweep (GPU box). Usage: merge_variants.sh "2048 512 128" "4 5 3"
OUT=gpurun_out; mkdir -p $OUT
for SM in $1; do
  for C in $2; do
    EXTRA=""; [ $C = 5 ] && EXTRA="--grad-pool 4"; [ $C = 4 ] && EXTRA="--grad-pool 8"
    LOWDIFF_MERGE_SPARSE_MAX=$SM timeout 600 python bench.py --config $C --steps 5 --warmup 3 --no-e2e --no-cpu-baseline $EXTRA > $OUT/bench_merge_${SM}_C$C.json 2>/dev/null
    python -c "import json;d=json.load(open('$OUT/bench_merge_${SM}_C$C.json'));k=d['kernels'];print('sparse_max=$SM C$C', round(d['ms_per_step'],3), 'merge', round(k['merge']['ms_per_step'],3), 'coalesce', round(k.get('coalesce',{'ms_per_step':0})['ms_per_step'],3))"
  done
done
