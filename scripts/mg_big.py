"""Sharded path at the bench size on one GPU: G virtual ranks (ft_dgehrd_vranks) against the
single-GPU reduction of the same matrix, fault-free and with one data fault.  Prints one JSON line
per case (n, G, time, max |H_vr - H_1| / max |H_1|, info, events).

usage: python scripts/mg_big.py [n] [G] [nb]
"""
import json
import sys
import time

import numpy as np
import torch

sys.path.insert(0, ".")
sys.path.insert(0, "tests")
import paper_conf_ipps_jiald16_b200 as ft  # noqa: E402
import synth  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
G = int(sys.argv[2]) if len(sys.argv) > 2 else 2
nb = int(sys.argv[3]) if len(sys.argv) > 3 else 64

A = torch.from_numpy(synth.matrix(n)).cuda()
dA = ft.fortran(A.clone())
t0 = time.time()
tau1, r1 = ft.dgehrd(dA, nb=nb)
torch.cuda.synchronize()
t1 = time.time() - t0
H1 = torch.triu(dA, -1)
s = H1.abs().max().item()
print(json.dumps({"case": "single", "n": n, "info": r1.info, "s": round(t1, 3)}), flush=True)
for faults in ((), ((3, ft.PHASE_BEFORE_PANEL, ft.SITE_A, n // 2 + 7, n // 2 + 100, 55),)):
    slabs = ft.shard(A, nb, G)
    torch.cuda.synchronize()
    t0 = time.time()
    taus, res = ft.dgehrd_vranks(slabs, nb=nb, faults=faults)
    torch.cuda.synchronize()
    tv = time.time() - t0
    Hv = torch.triu(ft.unshard(slabs, n, nb), -1)
    d = ((Hv - H1).abs().max() / s).item()
    dt = (taus[0][: n - 1] - tau1[: n - 1]).abs().max().item()
    ev = [e[0] for e in res.events][:8]
    print(json.dumps({"case": "vranks", "n": n, "G": G, "faults": len(faults), "info": res.info,
                      "s": round(tv, 3), "rel_H": d, "tau": dt, "detected": res.report.detected,
                      "events": ev}), flush=True)
    del slabs
