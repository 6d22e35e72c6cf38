#!/usr/bin/env python3
"""Cost of the deterministic mode (opts.deterministic): reduction time with FP64-atomic column dots
(default) and with fixed-order sums, interleaved, CUDA events (one GPU; never a bench value).

  python scripts/time_det.py [n] [nb] [reps]
"""
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
    ts = {False: [], True: []}
    outs = {}
    for it in range(reps + 1):
        for det in (False, True):
            dA.copy_(dA0)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(st)
            _, r = ft.dgehrd(dA, tau=tau, nb=nb, deterministic=det)
            e1.record(st)
            torch.cuda.synchronize()
            assert r.info == 0
            if it > 0:
                ts[det].append(e0.elapsed_time(e1))
            if det:
                h = dA.clone()
                if "det" in outs:
                    outs["bitwise_equal_repeat"] = bool(torch.equal(outs["det"], h))
                outs["det"] = h
    out = {"n": n, "nb": nb, "ms_default": min(ts[False]), "ms_deterministic": min(ts[True]),
           "overhead_pct": 100.0 * (min(ts[True]) / min(ts[False]) - 1.0),
           "bitwise_equal_repeat": outs.get("bitwise_equal_repeat")}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
