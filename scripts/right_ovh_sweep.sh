#!/bin/bash
# Right-update row-split cost model sweep: FT_RIGHT_OVH = per-CTA fixed cost in quarter tiles.
OUT=${1:-gpurun_out}
mkdir -p $OUT
for n in 2048 8192 16384; do
  reps=6; [ $n = 16384 ] && reps=3
  for o in 0 2 4 8; do
    echo "n=$n ovh=$o" >> $OUT/right_ovh.txt
    FT_RIGHT_OVH=$o timeout 300 python scripts/prof1.py $n $reps --no-panel-timing 2>&1 | tail -2 >> $OUT/right_ovh.txt
  done
done
