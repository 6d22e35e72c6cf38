#!/bin/bash
# Quick live timing of one build (graphs on): n = 2048 / 8192, ABFT on and off.
OUT=${1:-gpurun_out}
mkdir -p $OUT
for n in 2048 8192; do
  for a in 1 0; do
    echo "n=$n abft=$a" >> $OUT/quick.txt
    timeout 300 python scripts/prof1.py $n 6 --abft $a --no-panel-timing 2>&1 | tail -2 >> $OUT/quick.txt
  done
done
