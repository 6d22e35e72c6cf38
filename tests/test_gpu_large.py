"""GPU parity on the large-n code path (BASELINE config C3's path), through the C ABI.

For n > 2560 the library runs a different set of kernels than the small configs: Y_top by its own
split GEMM (k_ytop_partial / k_ytop_finalize, with the area-1 verify-before-consume fused in), and,
for panel launches with >= 32 rows per CTA, the two-reduction wide panel kernel (ft_panel_wide.cu,
with its own fused verify).  These tests hold that path to the same bar as the small ones:

  * full oracle parity at n = 5000, nb = 64 (wide launches for the early panels, ragged tail);
  * faults in every phase and site on that path, each run compared with the oracle's fault-free
    reduction at the parity bar; fix lists equal the oracle's (prefix run with the same fault);
  * prefix parity at n = 16384 (C3) -- the working matrix (H and V so far, trailing block updated)
    and the maintained checksums after m = 2 nb columns, both sides stopped by the verify hook
    (SURVEY 8(c) "Large-n parity");
  * the C3 fault pattern (two trailing flips, a Y flip after the panel, a checksum
    flip) at panel 1 with prefix parity, and at panel 64 over the full n = 16384 reduction with the
    residual / orthogonality bounds and prefix parity of the final output.

Bar (R17/R18): norm-wise max-entry <= 1e-9 for H, V, tau (and the working matrix);
checksums <= 1e-10 ||A||_F; residual and orthogonality ratios <= 30.
"""
import ctypes

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
EPS = 2.0 ** -52
TOL = 1e-9

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_ipps_jiald16_b200 as ft  # noqa: E402

N5, NB = 5000, 64
N16 = 16384
ORA_SITE = {ft.SITE_A: oracle.SITE_A, ft.SITE_R: oracle.SITE_R, ft.SITE_C: oracle.SITE_C}


def rel(a, b):
    d = np.abs(a - b).max() if a.size else 0.0
    s = np.abs(b).max() if b.size else 1.0
    return d / (s if s > 0 else 1.0)


def wide_count(reset=False):
    L = ft.lib()
    L.ft_debug_wide_launches.argtypes = [ctypes.c_int]
    L.ft_debug_wide_launches.restype = ctypes.c_int64
    return int(L.ft_debug_wide_launches(1 if reset else 0))


def gpu_run(A, nb=NB, faults=(), stop_after_panel=-1, keep_device=False):
    n = A.shape[0]
    dA = ft.fortran(torch.from_numpy(A).cuda())
    chk = torch.zeros(2 * n + 1, dtype=torch.float64, device="cuda") if stop_after_panel >= 0 else None
    tau, res = ft.dgehrd(dA, nb=nb, faults=faults, stop_after_panel=stop_after_panel, dchk_out=chk)
    torch.cuda.synchronize()
    out = dA if keep_device else dA.cpu().numpy()
    return out, tau.cpu().numpy()[: max(n - 1, 0)], res, (chk.cpu().numpy() if chk is not None else None), tau


def check_hvt(Ag, tg, Ao, to, cols=None, tol=TOL):
    """H, V, tau against the oracle (columns [0, cols) only when given: prefix parity)."""
    n = Ao.shape[0]
    c = n if cols is None else cols
    H, Ho = np.triu(Ag, -1)[:, :c], np.triu(Ao, -1)[:, :c]
    V, Vo = np.tril(Ag, -2)[:, :c], np.tril(Ao, -2)[:, :c]
    t, t0 = tg[:c], to[:c]
    assert rel(H, Ho) <= tol, ("H", rel(H, Ho))
    assert np.abs(V - Vo).max() <= tol * max(1.0, np.abs(Vo).max()), ("V", np.abs(V - Vo).max())
    assert np.abs(t - t0).max() <= tol * max(1.0, np.abs(t0).max()), ("tau", np.abs(t - t0).max())


def resid_orth_gpu(A, dH_full, tau_d, nb=NB):
    """Residual / orthogonality ratios (R17) through the library's own Q formation, on the GPU."""
    n = A.shape[0]
    Q, info = ft.dorghr(dH_full, tau_d, nb=nb)
    assert info == 0
    H = torch.triu(dH_full, -1)
    Ad = torch.from_numpy(A).cuda()
    n1 = lambda M: float(M.abs().sum(0).max())  # 1-norm
    resid = n1(Ad - Q @ H @ Q.T) / (n * n1(Ad) * EPS)
    orth = n1(torch.eye(n, dtype=torch.float64, device="cuda") - Q.T @ Q) / (n * EPS)
    return resid, orth


def fixes(events, kinds=("FIX_DATA", "FIX_R", "FIX_C", "FIX_K", "FIX_Q", "FIX_QR", "FIX_QC", "FIX_QK")):
    return sorted((e[0], e[2], e[3]) for e in events if e[0] in kinds)


@pytest.fixture(scope="module")
def a5():
    A = synth.matrix(N5)
    Ao, to = oracle.dgehd2(A)
    return A, Ao, to


@pytest.fixture(scope="module")
def a16():
    return synth.matrix(N16)


# ------------------------------------------------------------------ n = 5000, full oracle parity
def test_parity_large_path_full_oracle(a5):
    A, Ao, to = a5
    wide_count(reset=True)
    dA, tg, res, _, tau_d = gpu_run(A, keep_device=True)
    assert res.info == 0 and res.report.detected == 0, res.events
    assert wide_count() >= 10  # the early panels ran the wide (two-reduction) kernel
    check_hvt(dA.cpu().numpy(), tg, Ao, to)
    resid, orth = resid_orth_gpu(A, dA, tau_d)
    assert resid <= 30 and orth <= 30, (resid, orth)
    assert res.report.max_drift_rel < 0.5


# faults on the large-n path: panel 2 (k = 128) runs the wide kernel with the split Y_top; panel 60
# (k = 3840) is a narrow launch of the same large-n configuration
LARGE_FAULTS = [
    (2, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 3000, 4000, 55),   # area 2 (wide panel's fused verify)
    (2, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 60, 3000, 52),     # area 1 (k_ytop_partial's fused verify)
    (2, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 1000, 130, 62),    # the panel column, catastrophic exponent bit
    (2, ft.PHASE_BEFORE_PANEL, ft.SITE_R, 2222, -1, 50),
    (2, ft.PHASE_BEFORE_PANEL, ft.SITE_C, -1, 2500, 55),
    (2, ft.PHASE_AFTER_PANEL, ft.SITE_Y, 2000, 5, 45),       # pre-update check (unfused e^T Y)
    (2, ft.PHASE_AFTER_PANEL, ft.SITE_Y, 50, 7, 50),         # a Y_top row (formed by the split GEMM)
    (2, ft.PHASE_AFTER_PANEL, ft.SITE_V, 2500, 7, 62),
    (2, ft.PHASE_AFTER_PANEL, ft.SITE_T, 3, 9, 55),          # T checksum -> roll back the right update
    (2, ft.PHASE_AFTER_RIGHT, ft.SITE_A, 3000, 4000, 51),    # mid-update: rollback (reverse computation)
    (2, ft.PHASE_AFTER_UPDATE, ft.SITE_A, 3500, 4500, 58),
    (60, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 4500, 4900, 55),  # narrow launch, large n
    (0, ft.PHASE_AT_END, ft.SITE_A, 4000, 100, 50),          # area 3 (Householder vector) at the end
    (0, ft.PHASE_AT_END, ft.SITE_A, 90, 3000, 47),           # finished H at the end
]


@pytest.mark.parametrize("fault", LARGE_FAULTS, ids=lambda f: f"p{f[0]}-ph{f[1]}-s{f[2]}-{f[3]}-{f[4]}-b{f[5]}")
def test_large_path_faults(a5, fault):
    A, Ao, to = a5
    panel, phase, site, i, j, bit = fault
    Ag, tg, res, _, _ = gpu_run(A, faults=[fault])
    assert res.info == 0, res.events
    assert res.report.detected >= 1 or res.report.rollbacks >= 1 or res.report.panel_redos >= 1, res.events
    check_hvt(Ag, tg, Ao, to)
    got = fixes(res.events)
    if phase == ft.PHASE_BEFORE_PANEL and site in ORA_SITE and panel <= 2:
        # the oracle's prefix run with the same flip at the same boundary locates the same words
        info, _, _, rep, _ = oracle.ft_dgehd2(A, NB, faults=[(panel, ORA_SITE[site], i, j, bit)],
                                              stop_after_panel=panel)
        assert info == 0
        assert got == fixes(rep.events()), (got, rep.events())
    elif site == ft.SITE_A and phase != ft.PHASE_AT_END:
        assert ("FIX_DATA", i, j) in got, res.events
    elif phase == ft.PHASE_AT_END:
        assert any(e[0] in ("FIX_Q", "FIX_DATA") and e[1] == -1 and (e[2], e[3]) == (i, j) for e in res.events)


# ------------------------------------------------------------------ n = 16384 (C3): prefix parity
def test_prefix_parity_c3(a16):
    """Working matrix and checksums after panel 1 (m = 128 columns), both sides stopped there."""
    A = a16
    wide_count(reset=True)
    Ag, tg, res, chk, _ = gpu_run(A, stop_after_panel=1)
    assert res.info == 0 and res.report.detected == 0, res.events
    assert wide_count() == 2
    info, Aw, tw, rep, chko = oracle.ft_dgehd2(A, NB, stop_after_panel=1)
    assert info == 0 and rep.detected == 0
    assert rel(Ag, Aw) <= TOL, rel(Ag, Aw)
    assert np.abs(tg[:128] - tw[:128]).max() <= TOL
    normF = np.linalg.norm(A)
    assert np.abs(chk - chko).max() <= 1e-10 * normF, np.abs(chk - chko).max() / normF


C3_PATTERN = [(ft.PHASE_BEFORE_PANEL, ft.SITE_A, 9000, 12000, 55), (ft.PHASE_BEFORE_PANEL, ft.SITE_A, 10001, 15001, 47),
              (ft.PHASE_AFTER_PANEL, ft.SITE_Y, 11000, 3, 60), (ft.PHASE_BEFORE_PANEL, ft.SITE_C, -1, 13000, 52)]


def test_c3_fault_pattern_prefix(a16):
    """The C3 simultaneous-fault pattern injected at panel 1: corrected, and the state after panel 2
    equals the oracle's (which injects the same A / c flips at boundary 1) at the parity bar."""
    A = a16
    faults = [(1,) + f for f in C3_PATTERN]
    Ag, tg, res, chk, _ = gpu_run(A, faults=faults, stop_after_panel=2)
    assert res.info == 0, res.events
    assert res.report.panel_redos >= 1, res.events
    ofaults = [(1, ORA_SITE[s], i, j, b) for (ph, s, i, j, b) in C3_PATTERN if s in ORA_SITE]
    info, Aw, tw, rep, chko = oracle.ft_dgehd2(A, NB, faults=ofaults, stop_after_panel=2)
    assert info == 0
    assert fixes(res.events) == fixes(rep.events()), (res.events, rep.events())
    assert fixes(res.events) == [("FIX_C", -1, 13000), ("FIX_DATA", 9000, 12000), ("FIX_DATA", 10001, 15001)]
    assert rel(Ag, Aw) <= TOL, rel(Ag, Aw)
    normF = np.linalg.norm(A)
    assert np.abs(chk - chko).max() <= 1e-10 * normF


def test_c3_fault_pattern_full(a16):
    """SURVEY 8(d) C3 row verbatim: the pattern at panel 64 (k = 4096) of the full n = 16384, nb = 64
    reduction.  Every flip is corrected; the result meets the residual / orthogonality bounds, its
    first 128 columns equal the oracle's prefix, and it agrees with the fault-free run."""
    A = a16
    faults = [(64,) + f for f in C3_PATTERN]
    dA, tg, res, _, tau_d = gpu_run(A, faults=faults, keep_device=True)
    assert res.info == 0, res.events
    assert fixes(res.events) == [("FIX_C", -1, 13000), ("FIX_DATA", 9000, 12000), ("FIX_DATA", 10001, 15001)]
    assert res.report.panel_redos >= 1
    resid, orth = resid_orth_gpu(A, dA, tau_d)
    assert resid <= 30 and orth <= 30, (resid, orth)
    info, Aw, tw, rep, _ = oracle.ft_dgehd2(A, NB, stop_after_panel=1)
    assert info == 0
    Ag = dA.cpu().numpy()
    check_hvt(Ag, tg, Aw, tw, cols=128)
    dB, tB, resB, _, _ = gpu_run(A, keep_device=True)
    assert resB.info == 0 and resB.report.detected == 0
    assert float((torch.triu(dA, -1) - torch.triu(dB, -1)).abs().max()) <= TOL * float(torch.triu(dB, -1).abs().max())


# ------------------------------------------------------------------ sharded path at the C3 size
def test_sharded_path_c3_size(a16):
    """The 1-D block-column cyclic path (what bench.py --gpus N runs) at n = 16384: two virtual ranks
    on this GPU (74 CTAs each, ~221 rows per CTA) give the single-GPU H to the parity bar, fault-free
    and with a data flip at panel 3 that the sharded verification corrects."""
    A = a16
    n = A.shape[0]
    dA = ft.fortran(torch.from_numpy(A).cuda())
    tau1, r1 = ft.dgehrd(dA, nb=NB)
    assert r1.info == 0
    H1 = torch.triu(dA, -1)
    s = float(H1.abs().max())
    for faults in ((), ((3, ft.PHASE_BEFORE_PANEL, ft.SITE_A, n // 2 + 7, n // 2 + 100, 55),)):
        slabs = ft.shard(torch.from_numpy(A).cuda(), NB, 2)
        taus, res = ft.dgehrd_vranks(slabs, nb=NB, faults=faults)
        torch.cuda.synchronize()
        assert res.info == 0, res.events
        assert res.report.detected == len(faults), res.events
        Hv = torch.triu(ft.unshard(slabs, n, NB), -1)
        assert float((Hv - H1).abs().max()) <= TOL * s
        assert float((taus[0][: n - 1] - tau1[: n - 1]).abs().max()) <= TOL
        del slabs, Hv
