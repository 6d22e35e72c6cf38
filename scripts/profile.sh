#!/bin/bash
# Profiling recipe (run under gpurun on ONE GPU; B200_PROFILING.md):
#   1. the bench line (n = 2048) and bench lines at n = 8192 / 16384;
#   2. the ncu launch list of a short run of the SAME bench command;
#   3. per-launch DRAM traffic of every panel launch (n = 2048) -> panel_traffic.csv;
#   4. full ncu captures: the one-reduction panel (n = 2048, narrow), the two-reduction wide
#      panel and the update GEMMs (n = 8192).
set -x
OUT=${1:-gpurun_out}
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $OUT/gpu.txt
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err
timeout 900 python bench.py --n 8192 --nb 64 --steps 3 --warmup 3 --no-cpu-baseline > $OUT/bench_n8192.json 2> $OUT/bench_n8192.err
timeout 900 python bench.py --n 16384 --nb 64 --steps 2 --warmup 3 --no-cpu-baseline > $OUT/bench_n16384.json 2> $OUT/bench_n16384.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_bench.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $OUT/bench_under_ncu.json 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    -k regex:k_panel --csv --log-file $OUT/panel_traffic.csv python scripts/prof1.py 2048 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_panel -s 32 -c 1 -o $OUT/prof_panel \
    python scripts/prof1.py 2048 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_panel_wide -s 10 -c 1 -o $OUT/prof_panel_wide \
    python scripts/prof1.py 8192 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gemm_right -s 40 -c 1 -o $OUT/prof_right \
    python scripts/prof1.py 8192 1 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gemm_left -s 40 -c 1 -o $OUT/prof_left \
    python scripts/prof1.py 8192 1 > /dev/null 2>&1
ls -la $OUT
