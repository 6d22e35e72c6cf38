#!/usr/bin/env python3
"""Profiling driver: run `reps` ABFT reductions of the synthetic n x n matrix (one GPU).

  python scripts/prof1.py N [reps] [--nb NB] [--abft 0|1] [--probe PANEL] [--ablate MODE]

Prints per-call milliseconds (CUDA events), the panel kernel's share (live events) and,
with --probe, the per-column phase timestamps (clock64 cycles, CTA 0) of one panel.
Used under ncu (scripts/profile.sh) and for quick timing; never a bench value.
"""
import argparse
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("n", type=int)
    ap.add_argument("reps", type=int, nargs="?", default=1)
    ap.add_argument("--nb", type=int, default=0)
    ap.add_argument("--abft", type=int, default=1)
    ap.add_argument("--probe", type=int, default=-1)
    ap.add_argument("--ablate", type=int, default=0)
    ap.add_argument("--no-panel-timing", action="store_true", help="leave panel events off (CUDA graphs enabled)")
    a = ap.parse_args()
    import numpy as np
    import torch

    import paper_conf_ipps_jiald16_b200 as ft
    import synth

    n = a.n
    A = synth.matrix(n)
    dA0 = ft.fortran(torch.from_numpy(A).cuda())
    dA = ft.fortran(torch.empty((n, n), dtype=torch.float64, device="cuda"))
    tau = torch.zeros(n, dtype=torch.float64, device="cuda")
    L = ft.lib()
    L.ft_debug_time_panels.argtypes = [ctypes.c_int]
    L.ft_debug_panel_ms.restype = ctypes.c_double
    L.ft_debug_panel_launches.restype = ctypes.c_int
    dbg = None
    if a.probe >= 0:
        dbg = torch.zeros(2048 + 4 * 256 + 16, dtype=torch.int64, device="cuda")
        L.ft_debug_probe_panel.argtypes = [ctypes.c_int, ctypes.c_void_p]
        L.ft_debug_probe_panel(a.probe, ctypes.c_void_p(dbg.data_ptr()))
        L.ft_debug_ablate.argtypes = [ctypes.c_int]
        L.ft_debug_ablate(a.ablate)
    s = torch.cuda.current_stream()
    for it in range(a.reps):
        dA.copy_(dA0)
        L.ft_debug_time_panels(0 if a.no_panel_timing else 1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        _, res = ft.dgehrd(dA, tau=tau, nb=a.nb, abft=bool(a.abft), stream=s)
        e1.record(s)
        torch.cuda.synchronize()
        L.ft_debug_time_panels(0)
        ms = e0.elapsed_time(e1)
        pms = L.ft_debug_panel_ms()
        print(f"rep {it}: n={n} info={res.info} {ms:.3f} ms  panel {pms:.3f} ms "
              f"({L.ft_debug_panel_launches()} launches, {100 * pms / ms:.1f}%)  "
              f"{10 / 3 * n ** 3 / ms / 1e6:.1f} Gflop/s", flush=True)
    if dbg is not None:
        d = dbg.cpu().numpy()
        names = {0: "start", 1: "coldot", 2: "sync", 10: "c_loads", 4: "c_bar4a", 5: "c_part", 6: "c_bar4b",
                 11: "c_w", 12: "c_Gw_shfl", 9: "c_dlarfg",
                 3: "gemv_join", 7: "explicit/xchg", 14: "cmb_dots", 15: "cmb_gsum", 13: "cmb_leader", 8: "T_G_bar"}
        order = [0, 1, 2, 10, 4, 5, 6, 11, 12, 9, 3, 7, 14, 15, 13, 8]
        tot = {}
        ncol = 0
        for j in range(64):
            row = d[j * 16: j * 16 + 16]
            if row[0] == 0:
                continue
            ncol += 1
            prev = row[0]
            for sl in order[1:]:
                if row[sl] == 0:
                    continue
                tot[names[sl]] = tot.get(names[sl], 0) + (row[sl] - prev)
                prev = row[sl]
        mx = {}
        for j in range(64):
            row = d[1024 + j * 16: 1024 + j * 16 + 16]
            for sl in order[1:]:
                if row[sl] > 0:
                    mx[names[sl]] = mx.get(names[sl], 0) + row[sl]
        cta = d[2048:].reshape(-1, 4)
        cta = cta[cta[:, 2] > 0]
        if len(cta):  # per-CTA GEMV spans of column 8 (wide kernel): globaltimer ns
            t0 = cta[:, 1].min()
            dur = cta[:, 2] - cta[:, 1]
            print(f"per-CTA GEMV span, column 8: {len(cta)} CTAs, rows {cta[:, 3].min()}..{cta[:, 3].max()}, "
                  f"duration ns min {dur.min()} median {int(np.median(dur))} max {dur.max()}; "
                  f"start spread {cta[:, 1].max() - t0} ns, end spread {cta[:, 2].max() - cta[:, 2].min()} ns")
            order = np.argsort(cta[:, 0])
            print("  smid:dur_ns " + " ".join(f"{int(cta[q, 0])}:{int(dur[q])}" for q in order))
            print("  by CTA (bid:smid:dur_us) " + " ".join(f"{q}:{int(cta[q, 0])}:{dur[q] / 1e3:.0f}" for q in range(len(cta))))
        last_end = max(d[j * 16 + 8] for j in range(64))
        if d[3072] and d[3073]:
            print(f"CTA 0: prologue {d[0] - d[3072]} cycles, epilogue {d[3073] - last_end} cycles, "
                  f"kernel {d[3073] - d[3072]} cycles")
        print(f"probe panel {a.probe}: {ncol} columns, mean cycles per column by phase "
              f"(CTA 0 | max over CTAs of the phase):")
        for k2, v in tot.items():
            print(f"  {k2:12s} {v / max(ncol, 1):10.0f} {mx.get(k2, 0) / max(ncol, 1):10.0f}")


if __name__ == "__main__":
    main()
