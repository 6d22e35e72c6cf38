#!/bin/bash
# ncu --set full captures of the update GEMMs (and the wide panel) at C3 (one GPU, gpurun), plus the
# names of the FP64 / DMMA pipe metrics this ncu exposes.
OUT=${1:-gpurun_out/ncu_gemm}
mkdir -p $OUT
ncu --query-metrics 2>/dev/null | grep -i -E "dmma|fp64|tensor_op|pipe_tensor" > $OUT/metric_names.txt
for k in k_gemm_right k_gemm_left k_ytop_partial; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$k -s 100 -c 1 -o $OUT/prof_$k \
      python scripts/prof1.py 16384 1 --nb 64 --no-panel-timing > /dev/null 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_panel_wide -s 20 -c 1 -o $OUT/prof_panel_wide \
    python scripts/prof1.py 16384 1 --nb 64 --no-panel-timing > /dev/null 2>&1
ls -la $OUT
