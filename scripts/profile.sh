#!/bin/bash
# Profiling recipe (run under gpurun on ONE GPU): launch list of a short bench run and a
# full ncu capture of the dominant kernel (the DLAHR2 panel) and of the update GEMMs.
set -x
OUT=${1:-gpurun_out}
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $OUT/gpu.txt
python bench.py --steps 5 --warmup 3 > $OUT/bench.json 2> $OUT/bench.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python scripts/prof1.py 2048 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_panel -s 10 -c 1 -o $OUT/prof_panel \
    python scripts/prof1.py 2048 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_gemm_right -s 41 -c 1 -o $OUT/prof_right \
    python scripts/prof1.py 2048 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_gemm_left -s 20 -c 1 -o $OUT/prof_left \
    python scripts/prof1.py 2048 1 > /dev/null 2>&1
ls -la $OUT
