#!/bin/bash
# margin-controller band sweep: per-call compress time in the EF steady state (graph-timed)
cd "$(dirname "$0")/.."
for band in "1.2,3" "1.1,2" "1.05,1.5" "1.02,1.3"; do
  for c in 2 3 4; do
    cy=16; [ $c = 4 ] && cy=8
    echo "band $band $(LOWDIFF_CAND_BAND=$band python scripts/time_compress.py --config $c --cycle $cy --reps 30 | tail -1)"
  done
done
