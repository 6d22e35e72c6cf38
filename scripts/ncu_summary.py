#!/usr/bin/env python3
"""Key metrics of an ncu report (raw page) + top stall lines (source page).

  python scripts/ncu_summary.py report.ncu-rep [--lines N]
"""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_op_dmma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_tensor_subpipe_dmma.avg.pct_of_peak_sustained_active",
        "sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "launch__occupancy_limit_shared_mem",
        "smsp__average_warp_latency_per_inst_issued.ratio", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"]


def main():
    rep = sys.argv[1]
    nl = int(sys.argv[sys.argv.index("--lines") + 1]) if "--lines" in sys.argv else 15
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, u = rows[0], rows[1]
    for v in rows[2:]:
        print("kernel:", v[h.index("Kernel Name")][:80])
        for i, name in enumerate(h):
            if name in KEYS or ("warps_issue_stalled" in name and name.endswith("per_issue_active.ratio")
                                and float(v[i] or 0) > 0.3):
                print(f"  {name:75s} {v[i]:>14s} {u[i]}")
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    agg, tot, cur = {}, 0, None
    for r in csv.reader(io.StringIO(src)):
        if len(r) >= 2 and r[0] == "File Path":
            cur = r[1].split("/")[-1]
            continue
        if len(r) < 6 or r[0] in ("Line No", ""):
            continue
        try:
            s = int(r[4])
        except ValueError:
            continue
        agg[(cur, int(r[0]))] = (s, r[1][:90])
        tot += s
    print(f"top stall-sample lines (of {tot}):")
    for (f, l), (s, t) in sorted(agg.items(), key=lambda x: -x[1][0])[:nl]:
        print(f"  {s:7d} {100 * s / max(tot, 1):5.1f}% {f}:{l} {t}")


if __name__ == "__main__":
    main()
