#!/bin/bash
# C2 ABFT-overhead anatomy (one GPU): on/off totals and phase split, the per-column probe of one
# panel each way, and ncu launch lists of one reduction each way summarised per kernel.
OUT=${1:-gpurun_out}
N=${N:-2048}
mkdir -p $OUT
timeout 300 python scripts/time_c3.py $N 32 20 > $OUT/time_n$N.json 2>&1
for a in 1 0; do
  timeout 300 python scripts/prof1.py $N 3 --abft $a --probe 10 > $OUT/probe_n${N}_abft$a.txt 2>&1
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $OUT/launch_n${N}_abft$a.csv python scripts/prof1.py $N 2 --abft $a --no-panel-timing > /dev/null 2>&1
  python scripts/launch_summary.py $OUT/launch_n${N}_abft$a.csv --last-fraction 0.5 > $OUT/launch_n${N}_abft${a}_summary.txt 2>&1
done
