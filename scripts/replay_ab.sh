#!/bin/bash
# A/B of replay variant builds (vso/<name>.so, built here with LOWDIFF_SO/LOWDIFF_NVCC_EXTRA) on the
# GPU box: median replay ms per config. Usage: replay_ab.sh "base v1 v2" ["3 4 5"] [approx]
VARS=${1:-base}; CFGS=${2:-"3 4 5"}; APX=${3:-1}
python -c "import __graft_entry__ as g; g.build()" > /dev/null
for V in $VARS; do
  SO=""; [ $V != base ] && SO="LOWDIFF_SO=$PWD/vso/$V.so"
  for C in $CFGS; do
    EX=""; [ $C = 3 ] && EX="--ef-warmup 400"; [ $C = 4 ] && EX="--ef-warmup 400 --grad-pool 8"; [ $C = 5 ] && EX="--grad-pool 4"
    echo -n "$V C$C "
    env $SO timeout 300 python scripts/time_replay.py --config $C --approx $APX --reps 10 $EX | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['replay_ms_median'],3), d['sm_mhz_median'])"
  done
done
