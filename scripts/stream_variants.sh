#!/bin/bash
# Stream kernel variants (GPU box): TMA stages. Usage: stream_variants.sh "2 3 4" "3 5"
OUT=gpurun_out; mkdir -p $OUT
for ST in $1; do
  LOWDIFF_NVCC_EXTRA="-DLOWDIFF_STREAM_STAGES=$ST" python -m paper_conf_sc_yaolhlzz25_b200.build --force > /dev/null 2>&1
  for C in $2; do
    EXTRA=""; [ $C = 5 ] && EXTRA="--grad-pool 4"; [ $C = 4 ] && EXTRA="--grad-pool 8"
    LOWDIFF_STREAM_TMA=1 timeout 600 python bench.py --config $C --steps 10 --warmup 3 --no-e2e --no-cpu-baseline $EXTRA > $OUT/bench_st${ST}_C$C.json 2>/dev/null
    python -c "import json;d=json.load(open('$OUT/bench_st${ST}_C$C.json'));k=d['kernels']['compress_stream'];print('stages=$ST C$C', round(d['value'],1), 'stream ms/launch', round(k['ms_per_step']/k['launches_per_step'],4), 'frac', round(d['roofline']['frac'],3))"
  done
done
python -m paper_conf_sc_yaolhlzz25_b200.build --force > /dev/null 2>&1
