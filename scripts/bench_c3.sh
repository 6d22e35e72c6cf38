#!/bin/bash
# Round-2 measurement recipe (one GPU, under gpurun): the FP64 peak, the bench line at C3 (+ C2
# keys), the reference arm, the ncu launch list of the same bench command (first reduction) and
# the per-launch DRAM traffic of every panel launch of one C3 reduction.
OUT=${1:-gpurun_out}
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem --format=csv > $OUT/gpu.txt
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o scripts/mb_dmma scripts/mb_dmma.cu && \
  timeout 120 ./scripts/mb_dmma $OUT/fp64_peak.json > $OUT/mb_dmma.txt 2>&1
cp $OUT/fp64_peak.json profiles/fp64_peak.json 2>/dev/null
timeout 1200 python bench.py ${BENCH_ARGS:---steps 5 --warmup 3} > $OUT/bench_c3.json 2> $OUT/bench_c3.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > $OUT/bench_ref.json 2> $OUT/bench_ref.err
if [ -z "$NO_NCU" ]; then
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 1500 --csv --log-file $OUT/launches_c3.csv \
    python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-c2 > $OUT/bench_under_ncu.json 2>&1
timeout 1200 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    -k regex:k_panel --csv --log-file $OUT/panel_traffic_c3.csv python scripts/prof1.py 16384 1 > /dev/null 2>&1
fi
ls -la $OUT
