#!/bin/bash
# ABFT overhead anatomy (one GPU): live per-call and panel times with ABFT off / on, then ncu
# launch lists of one reduction each way, summarised per kernel.
OUT=${1:-gpurun_out}
mkdir -p $OUT
for n in 2048 8192; do
  for a in 0 1; do
    timeout 300 python scripts/prof1.py $n 6 --abft $a > $OUT/ovh_live_n${n}_abft$a.txt 2>&1
    timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
      --log-file $OUT/ovh_launch_n${n}_abft$a.csv python scripts/prof1.py $n 2 --abft $a > /dev/null 2>&1
    python scripts/launch_summary.py $OUT/ovh_launch_n${n}_abft$a.csv --last-fraction 0.5 \
      > $OUT/ovh_launch_n${n}_abft${a}_summary.txt 2>&1
  done
done
