#!/usr/bin/env python3
"""A/B of a debug toggle (ft_debug_<name>(0|1)): per-kernel-class live times (ft_debug_time_kernels)
of ABFT-on reductions, alternating the toggle; min over reps.  Never a bench value.

  python scripts/ab_toggle.py right_fold N NB [reps]
"""
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch

    import paper_conf_ipps_jiald16_b200 as ft
    import synth
    name, n, nb = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
    reps = int(sys.argv[4]) if len(sys.argv) > 4 else 5
    L = ft.lib()
    tog = getattr(L, "ft_debug_" + name)
    tog.argtypes = [ctypes.c_int]
    L.ft_debug_time_kernels.argtypes = [ctypes.c_int]
    L.ft_debug_kernel_ms.restype = ctypes.c_double
    L.ft_debug_kernel_ms.argtypes = [ctypes.c_int]
    A = synth.matrix(n)
    dA0 = ft.fortran(torch.from_numpy(A).cuda())
    dA = ft.fortran(torch.empty_like(dA0))
    tau = torch.zeros(n, dtype=torch.float64, device="cuda")
    best = {}
    for it in range(reps):
        for v in (1, 0):
            tog(v)
            dA.copy_(dA0)
            torch.cuda.synchronize()
            L.ft_debug_time_kernels(1)
            _, r = ft.dgehrd(dA, tau=tau, nb=nb, timing=True)
            torch.cuda.synchronize()
            L.ft_debug_time_kernels(0)
            assert r.info == 0 and r.report.detected == 0
            cur = [r.report.ms[0]] + [L.ft_debug_kernel_ms(i) for i in range(3)]
            b = best.setdefault(v, cur)
            best[v] = [min(x, y) for x, y in zip(b, cur)]
    tog(1)
    out = {"toggle": name, "n": n, "nb": nb}
    for v in (1, 0):
        out[f"on{v}"] = dict(zip(["total", "panel", "right", "left"], [round(x, 3) for x in best[v]]))
    print(json.dumps(out))


if __name__ == "__main__":
    main()
