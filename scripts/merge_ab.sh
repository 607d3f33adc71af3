#!/bin/bash
# A/B of merge variant builds (vso/<name>.so) on the GPU box: bench merge ms/step per config.
# Usage: merge_ab.sh "base v1" ["4 2 5"]
VARS=${1:-base}; CFGS=${2:-"4 2 5"}
python -c "import __graft_entry__ as g; g.build()" > /dev/null
for V in $VARS; do
  SO=""; [ $V != base ] && SO="LOWDIFF_SO=$PWD/vso/$V.so"
  for C in $CFGS; do
    EX=""; [ $C = 4 ] && EX="--grad-pool 8"; [ $C = 5 ] && EX="--grad-pool 4"
    env $SO timeout 600 python bench.py --config $C --steps 10 --warmup 3 --no-e2e --no-cpu-baseline $EX > /tmp/mab.json 2>/dev/null
    python -c "import json;d=json.load(open('/tmp/mab.json'));k=d['kernels'];print('$V C$C', round(d['value'],1), round(d['ms_per_step'],3), 'merge', round(k['merge']['ms_per_step'],3), 'pack', round(k['merge_pack']['ms_per_step'],3))"
  done
done
