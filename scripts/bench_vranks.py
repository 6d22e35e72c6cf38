#!/usr/bin/env python3
"""Time the sharded (multi-GPU) path with G virtual ranks on ONE GPU against the single-GPU
path: the ranks share the SMs, so this measures the cost of the exchange protocol and the
per-rank launches, not a multi-GPU speedup.  Never a bench value.

  python scripts/bench_vranks.py N [reps] [--nb NB] [--G 1,2,4,8]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("n", type=int)
    ap.add_argument("reps", type=int, nargs="?", default=3)
    ap.add_argument("--nb", type=int, default=0)
    ap.add_argument("--G", default="1,2,4,8")
    a = ap.parse_args()
    import torch

    import paper_conf_ipps_jiald16_b200 as ft
    import synth
    n = a.n
    nb = a.nb or ft.default_nb(n)
    A = torch.from_numpy(synth.matrix(n)).cuda()
    gf = 10 / 3 * n ** 3 / 1e9
    for G in [int(x) for x in a.G.split(",")]:
        for abft in (True, False):
            ms = []
            for _ in range(a.reps + 1):
                if G == 1:
                    dA = ft.fortran(A.clone())
                    torch.cuda.synchronize()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    _, res = ft.dgehrd(dA, nb=nb, abft=abft)
                else:
                    slabs = ft.shard(A, nb, G)
                    torch.cuda.synchronize()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    _, res = ft.dgehrd_vranks(slabs, nb=nb, abft=abft)
                e1.record()
                torch.cuda.synchronize()
                assert res.info == 0, res.info
                ms.append(e0.elapsed_time(e1))
            best = min(ms[1:])
            print(f"n={n} nb={nb} G={G} abft={int(abft)}: {best:9.3f} ms  {gf / best * 1e3:8.1f} Gflop/s"
                  + ("" if G == 1 else f"  (virtual ranks on one GPU; detected={res.report.detected})"), flush=True)


if __name__ == "__main__":
    main()
