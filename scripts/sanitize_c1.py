#!/usr/bin/env python3
"""compute-sanitizer driver (memcheck / racecheck / synccheck on C1): config C1 (n = 64,
nb = 16) fault-free and with a corrected soft error (recovery path), n = 300 (several CTAs of row
groups, ragged tiles), the T-checksum rollback, Q formation, n = 700 at nb = 64 (the TMA GEMM
pipelines), the deterministic mode and two virtual ranks.

  compute-sanitizer --tool memcheck python scripts/sanitize_c1.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import numpy as np
    import torch

    import paper_conf_ipps_jiald16_b200 as ft
    import synth

    runs = [(64, 16, []), (64, 16, [(1, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 40, 50, 51)]),
            (300, 32, [(2, ft.PHASE_AFTER_RIGHT, ft.SITE_A, 150, 200, 55)]),
            (300, 32, [(1, ft.PHASE_AFTER_PANEL, ft.SITE_T, 3, 10, 55)]),
            # nb = 64 (KT = 64 TMA GEMM pipelines, several row splits, right-only tiles above the
            # W rows, the M-part strip) fault-free and with a mid-update flip
            (700, 64, []), (700, 64, [(3, ft.PHASE_AFTER_RIGHT, ft.SITE_A, 400, 500, 54)])]
    for n, nb, faults in runs:
        A = synth.matrix(n)
        dA = ft.fortran(torch.from_numpy(A).cuda())
        tau, res = ft.dgehrd(dA, nb=nb, faults=faults)
        torch.cuda.synchronize()
        Q, info = ft.dorghr(dA, tau, nb=nb)
        torch.cuda.synchronize()
        print(f"n={n} nb={nb} faults={len(faults)} info={res.info} dorghr={info} events={res.events}", flush=True)
        assert res.info == 0 and info == 0
    A = synth.matrix(130)
    slabs = ft.shard(torch.from_numpy(A).cuda(), 16, 2)
    taus, res = ft.dgehrd_vranks(slabs, nb=16)
    torch.cuda.synchronize()
    print(f"vranks G=2 n=130 info={res.info}", flush=True)
    assert res.info == 0
    # deterministic mode (fixed-order column dots)
    A = synth.matrix(300)
    dA = ft.fortran(torch.from_numpy(A).cuda())
    tau, res = ft.dgehrd(dA, nb=32, deterministic=True)
    torch.cuda.synchronize()
    print(f"deterministic n=300 info={res.info}", flush=True)
    assert res.info == 0
    print("SANITIZE_DRIVER_OK")


if __name__ == "__main__":
    main()
