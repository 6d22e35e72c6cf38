#!/usr/bin/env python3
"""Panel-kernel path A/B at one size (one GPU; never a bench value): one reduction per path setting
(ft_debug_panel_path bits: 0 default, 64 narrow kernel with the two-buffer cache, 128 narrow kernel,
no cache), live kernel-class times.

  python scripts/time_path.py [n] [nb] [bits ...]
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
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
    nb = int(sys.argv[2]) if len(sys.argv) > 2 else 64
    bits = [int(b) for b in sys.argv[3:]] or [0, 64, 128]
    A = synth.matrix(n)
    dA0 = ft.fortran(torch.from_numpy(A).cuda())
    dA = ft.fortran(torch.empty_like(dA0))
    tau = torch.zeros(n, dtype=torch.float64, device="cuda")
    L = ft.lib()
    L.ft_debug_panel_path.argtypes = [ctypes.c_int]
    L.ft_debug_time_kernels.argtypes = [ctypes.c_int]
    L.ft_debug_kernel_ms.restype = ctypes.c_double
    st = torch.cuda.current_stream()
    for b in bits:
        L.ft_debug_panel_path(b)
        for rep in range(2):
            dA.copy_(dA0)
            torch.cuda.synchronize()
            L.ft_debug_time_kernels(1)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            _, r = ft.dgehrd(dA, tau=tau, nb=nb)
            e1.record(st)
            torch.cuda.synchronize()
            ks = {c: round(L.ft_debug_kernel_ms(c), 2) for c in range(3)}
            L.ft_debug_time_kernels(0)
            if rep == 1:
                print(json.dumps({"bits": b, "info": r.info, "ms": round(e0.elapsed_time(e1), 2),
                                  "panel_ms": ks[0], "right_ms": ks[1], "left_ms": ks[2]}))
    L.ft_debug_panel_path(0)


if __name__ == "__main__":
    main()
