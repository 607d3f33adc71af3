#!/bin/bash
# Bench the replay kernel compiled for different CTAs/SM (run on the GPU box).
OUT=gpurun_out; mkdir -p $OUT
for MB in ${MINBS:-3 4}; do
  LOWDIFF_NVCC_EXTRA="-DLOWDIFF_REPLAY_MINB=$MB" python -m paper_conf_sc_yaolhlzz25_b200.build --force > /dev/null 2>&1
  timeout 300 python bench.py ${BENCH_ARGS:-} --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_minb$MB.json 2>/dev/null
  python -c "import json;d=json.load(open('$OUT/bench_minb$MB.json'));print($MB, round(d['value'],1), round(d['ms_per_step'],3), round(d['kernels']['replay_dense']['ms_per_step'],3))"
done
python -m paper_conf_sc_yaolhlzz25_b200.build --force > /dev/null 2>&1
