#!/usr/bin/env python3
"""Q formation timing (NEXT-3): ft_dorghr at n (default 16384, nb 64), protected (abft=1) and plain,
CUDA events on the stream; Gflop/s on 4/3 n^3 (DORGHR's flops for ilo = 1, ihi = n) and the fraction of
the measured FP64 DMMA peak (profiles/fp64_peak.json).  Prints one JSON line."""
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
    dA = ft.fortran(torch.from_numpy(A).cuda())
    tau, res = ft.dgehrd(dA, nb=nb)
    torch.cuda.synchronize()
    assert res.info == 0
    Q = ft.fortran(torch.empty((n, n), dtype=torch.float64, device="cuda"))
    out = {"n": n, "nb": nb}
    st = torch.cuda.current_stream()
    for abft in (True, False, True, False):
        ts = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            _, r = ft.dorghr(dA, tau, Q=Q, nb=nb, abft=abft, full=True)
            e1.record(st)
            torch.cuda.synchronize()
            assert r.info == 0
            ts.append(e0.elapsed_time(e1))
        out["ms_abft" if abft else "ms_plain"] = min(ts)
    _, r = ft.dorghr(dA, tau, Q=Q, nb=nb, abft=True, full=True, timing=True)
    torch.cuda.synchronize()
    out["phases_ms"] = {k: r.report.ms[i] for i, k in enumerate(["total", "-", "W (right kernel)", "left", "verify",
                                                                  "recovery", "copy", "-"])}
    fl = 4.0 / 3.0 * n ** 3
    peak = json.load(open(os.path.join(ROOT, "profiles", "fp64_peak.json")))["dmma_tflops_sustained"]
    out["gflops_abft"] = fl / out["ms_abft"] / 1e6
    out["gflops_plain"] = fl / out["ms_plain"] / 1e6
    out["frac_of_dmma_abft"] = out["gflops_abft"] / 1e3 / peak
    out["abft_overhead_pct"] = 100.0 * (out["ms_abft"] - out["ms_plain"]) / out["ms_plain"]
    print(json.dumps(out))


if __name__ == "__main__":
    main()
