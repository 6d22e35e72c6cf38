#!/usr/bin/env python3
"""Quick C3 timing (one GPU, never a bench value): reps reductions of n x n (default 16384, nb 64),
ABFT on / off, CUDA events, and one timed call's phase split (report.ms) and kernel classes."""
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
    reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
    A = synth.matrix(n)
    dA0 = ft.fortran(torch.from_numpy(A).cuda())
    dA = ft.fortran(torch.empty_like(dA0))
    tau = torch.zeros(n, dtype=torch.float64, device="cuda")
    st = torch.cuda.current_stream()
    out = {"n": n, "nb": nb}
    for abft in (True, False, True, False):
        ts = []
        for _ in range(reps):
            dA.copy_(dA0)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            _, r = ft.dgehrd(dA, tau=tau, nb=nb, abft=abft)
            e1.record(st)
            torch.cuda.synchronize()
            assert r.info == 0
            ts.append(e0.elapsed_time(e1))
        out["ms_on" if abft else "ms_off"] = min(ts)
    L = ft.lib()
    L.ft_debug_time_kernels.argtypes = [ctypes.c_int]
    L.ft_debug_kernel_ms.restype = ctypes.c_double
    L.ft_debug_kernel_ms.argtypes = [ctypes.c_int]
    for abft in (True, False):
        dA.copy_(dA0)
        L.ft_debug_time_kernels(1)
        _, r = ft.dgehrd(dA, tau=tau, nb=nb, timing=True, abft=abft)
        torch.cuda.synchronize()
        L.ft_debug_time_kernels(0)
        sfx = "" if abft else "_off"
        out["phases" + sfx] = {k: round(r.report.ms[i], 2) for i, k in enumerate(
            ["total", "panel+ytop", "right", "left", "verify", "recovery", "copy", "encode"])}
        out["kernels" + sfx] = {k: round(L.ft_debug_kernel_ms(i), 2) for i, k in enumerate(["panel", "right", "left"])}
    out["gflops_on"] = 10.0 / 3.0 * n ** 3 / out["ms_on"] / 1e6
    out["overhead_pct"] = 100.0 * (out["ms_on"] - out["ms_off"]) / out["ms_off"]
    print(json.dumps(out))


if __name__ == "__main__":
    main()
