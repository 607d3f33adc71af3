#!/bin/bash
# Build liblowdiff with each set of extra nvcc flags, run the replay/update parity tests and the
# C3/C4 benches for it (GPU box). Usage: VARIANTS="flags1;flags2" variant_sweep.sh <tag>
TAG=${1:-v}; OUT=gpurun_out; mkdir -p $OUT
IFS=';' read -ra VS <<< "${VARIANTS:-}"
i=0
for V in "${VS[@]}"; do
  LOWDIFF_NVCC_EXTRA="$V" python -m paper_conf_sc_yaolhlzz25_b200.build --force > /dev/null 2>&1
  echo "== variant $i: $V"
  timeout 600 python -m pytest tests -m gpu -q -x -k "${TESTS:-replay or update or in_loop}" -p no:cacheprovider 2>&1 | tail -1
  for C in ${CONFIGS:-3 4}; do
    EXTRA=""; [ $C = 4 ] && EXTRA="--grad-pool 8"; [ $C = 5 ] && EXTRA="--grad-pool 4"
    timeout 600 python bench.py --config $C --steps 10 --warmup 3 --no-e2e --no-cpu-baseline $EXTRA > $OUT/var_${TAG}_${i}_C$C.json 2>/dev/null
    python -c "
import json;d=json.load(open('$OUT/var_${TAG}_${i}_C$C.json'))
print('  C$C', round(d['value'],1), 'GB/s', round(d['ms_per_step'],3), 'ms', {k: round(v['ms_per_step'],3) for k,v in d['kernels'].items() if k in ('replay_dense','compress_select','merge','compress_stream')})"
  done
  i=$((i+1))
done
python -m paper_conf_sc_yaolhlzz25_b200.build --force > /dev/null 2>&1
