"""GPU parity tests: the CUDA path (through the C ABI) against the CPU oracle.

Tolerances (readings R17/R18):
  * H, V, tau, Q: max|x_gpu - x_ora| / max|x_ora| <= 1e-9 (norm-wise max-entry)
  * ||A - Q H Q^T||_1 / (n ||A||_1 eps) <= 30 and ||I - Q^T Q||_1 / (n eps) <= 30
  * checksums at an iteration boundary: |chk_gpu - chk_ora| <= 1e-10 ||A||_F
  * fault runs: same tolerances as a fault-free run; located (i, j) equal the oracle's
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


def rel(a, b):
    d = np.abs(a - b).max() if a.size else 0.0
    s = np.abs(b).max() if b.size else 1.0
    return d / (s if s > 0 else 1.0)


def gpu_reduce(A, ilo=1, ihi=None, lda=None, **kw):
    n = A.shape[0]
    if lda is None or lda == n:
        dA = ft.fortran(torch.from_numpy(A).cuda())
    else:  # a padded leading dimension
        buf = torch.zeros(lda * n, dtype=torch.float64, device="cuda")
        dA = torch.as_strided(buf, (n, n), (1, lda))
        dA.copy_(torch.from_numpy(A).cuda())
    tau, res = ft.dgehrd(dA, ilo=ilo, ihi=ihi, **kw)
    torch.cuda.synchronize()
    return dA, tau, res


def check_against_oracle(A, dA, tau, ilo=1, ihi=None, nb=0, tol=TOL):
    n = A.shape[0]
    ihi = n if ihi is None else ihi
    Ao, to = oracle.dgehd2(A, ilo, ihi)
    Ag = dA.cpu().numpy()
    tg = tau.cpu().numpy()[: max(n - 1, 0)]
    H, Ho = np.triu(Ag, -1), np.triu(Ao, -1)
    assert rel(H, Ho) <= tol, ("H", rel(H, Ho))
    assert np.abs(tg - to).max(initial=0.0) <= tol * max(1.0, np.abs(to).max(initial=0.0)), "tau"
    if n > 2:
        V, Vo = np.tril(Ag, -2), np.tril(Ao, -2)
        assert np.abs(V - Vo).max() <= tol * max(1.0, np.abs(Vo).max()), ("V", np.abs(V - Vo).max())
    Q, info = ft.dorghr(dA, tau, ilo=ilo, ihi=ihi, nb=nb)
    assert info == 0
    Qg = Q.cpu().numpy()
    Qo = oracle.dorghr(Ao, to, ilo, ihi)
    assert np.abs(Qg - Qo).max(initial=0.0) <= tol, ("Q", np.abs(Qg - Qo).max())
    if n:
        an = np.linalg.norm(A, 1)
        res = np.linalg.norm(A - Qg @ H @ Qg.T, 1) / (n * max(an, 1e-300) * EPS)
        orth = np.linalg.norm(np.eye(n) - Qg.T @ Qg, 1) / (n * EPS)
        assert res <= 30 and orth <= 30, (res, orth)
    return H, Ho


# ------------------------------------------------------------------ fault-free parity
@pytest.mark.parametrize("n,nb", [(1, 16), (2, 16), (3, 16), (4, 16), (5, 16), (17, 16), (18, 16), (64, 16),
                                  (100, 32), (257, 32), (300, 64), (513, 64)])
@pytest.mark.parametrize("abft", [False, True])
def test_parity_small(n, nb, abft):
    A = synth.matrix(n, dist="uniform")
    dA, tau, res = gpu_reduce(A, nb=nb, abft=abft)
    assert res.info == 0, res.events
    assert res.report.detected == 0 and res.report.nevents == 0, res.events
    check_against_oracle(A, dA, tau, nb=nb)


@pytest.mark.parametrize("n,nb,dist", [(700, 32, "normal"), (1000, 64, "uniform")])
def test_parity_medium(n, nb, dist):
    A = synth.matrix(n, dist=dist)
    dA, tau, res = gpu_reduce(A, nb=nb)
    assert res.info == 0 and res.report.detected == 0
    check_against_oracle(A, dA, tau, nb=nb)
    assert res.report.max_drift_rel < 0.5  # fault-free checksum drift, units of n eps ||A||_F


@pytest.mark.parametrize("n,nb,abft,bits", [(64, 16, True, 8), (300, 32, False, 8), (513, 64, True, 8),
                                            (700, 32, True, 8), (513, 64, True, 64), (700, 32, False, 128),
                                            (300, 64, True, 8 | 128)])
def test_parity_explicit_path(n, nb, abft, bits):
    """Every column on the explicit two-reduction path (bit 8: the one-reduction column's
    cancellation fallback, ft_panel.cu) and/or the panel's smaller shared-memory modes (64: Y rows
    global, 128: V/Y/Z rows global -- the large-n layouts): same parity bar, and agreement with the
    default path to rounding."""
    A = synth.matrix(n, dist="uniform")
    L = ft.lib()
    L.ft_debug_panel_path.argtypes = [ctypes.c_int]
    L.ft_debug_panel_path(bits)
    try:
        dA, tau, res = gpu_reduce(A, nb=nb, abft=abft)
    finally:
        L.ft_debug_panel_path(0)
    assert res.info == 0 and res.report.detected == 0, res.events
    check_against_oracle(A, dA, tau, nb=nb)
    dA1, tau1, res1 = gpu_reduce(A, nb=nb, abft=abft)
    assert res1.info == 0
    H0, H1 = np.triu(dA.cpu().numpy(), -1), np.triu(dA1.cpu().numpy(), -1)
    assert np.abs(H0 - H1).max() <= 1e-11 * np.abs(H1).max()


def test_parity_unfused_ytop():
    """n = 2600 (> 2560): Y_top by its own GEMM kernels, the M-part by the right update, every
    panel launch still narrow (the one-reduction kernel) -- the full oracle bar."""
    n = 2600
    A = synth.matrix(n)
    dA, tau, res = gpu_reduce(A, nb=32)
    assert res.info == 0 and res.report.detected == 0
    check_against_oracle(A, dA, tau, nb=32)


def test_parity_c2_full_size():
    """BASELINE config C2 (n = 2048, nb = 32), the bench workload, full element-wise parity."""
    n = 2048
    A = synth.matrix(n)
    dA, tau, res = gpu_reduce(A, nb=32)
    assert res.info == 0 and res.report.detected == 0
    check_against_oracle(A, dA, tau, nb=32)


@pytest.mark.parametrize("n,nb,abft", [(600, 32, True), (600, 32, False), (1100, 64, True)])
def test_graph_replay(n, nb, abft):
    """Repeated fault-free calls on the same buffers: the 2nd call captures a CUDA graph, later
    calls replay it; every result must match the oracle, and a fault run on the same buffers
    (direct launches) must still detect and correct."""
    A = synth.matrix(n)
    At = torch.from_numpy(A).cuda()
    dA = ft.fortran(torch.empty((n, n), dtype=torch.float64, device="cuda"))
    tau = torch.zeros(n, dtype=torch.float64, device="cuda")
    Ho = None
    for it in range(4):
        dA.copy_(At)
        _, res = ft.dgehrd(dA, tau=tau, nb=nb, abft=abft)
        torch.cuda.synchronize()
        assert res.info == 0 and res.report.detected == 0, (it, res.events)
        H = np.triu(dA.cpu().numpy(), -1)
        if Ho is None:
            Ao, _ = oracle.dgehd2(A)
            Ho = np.triu(Ao, -1)
        assert rel(H, Ho) <= TOL, (it, rel(H, Ho))
    if abft:
        dA.copy_(At)
        _, res = ft.dgehrd(dA, tau=tau, nb=nb, faults=[(1, ft.PHASE_BEFORE_PANEL, ft.SITE_A, n // 2, n // 2 + 9, 55)])
        torch.cuda.synchronize()
        assert res.info == 0 and any(e[0] == "FIX_DATA" for e in res.events), res.events
        assert rel(np.triu(dA.cpu().numpy(), -1), Ho) <= TOL


@pytest.mark.parametrize("policy", [ft.POLICY_EAGER, ft.POLICY_PAPER])
def test_policies_fault_free(policy):
    A = synth.matrix(200, dist="normal")
    dA, tau, res = gpu_reduce(A, nb=32, policy=policy)
    assert res.info == 0 and res.report.detected == 0
    check_against_oracle(A, dA, tau, nb=32)


@pytest.mark.parametrize("n,ilo,ihi,nb", [(150, 4, 131, 32), (90, 1, 70, 16), (90, 20, 90, 16), (64, 30, 33, 16),
                                         (64, 10, 10, 16)])
@pytest.mark.parametrize("abft", [False, True])
def test_ilo_ihi(n, ilo, ihi, nb, abft):
    A = synth.matrix(n, seed=n + ilo + ihi, ilo=ilo, ihi=ihi)
    dA, tau, res = gpu_reduce(A, ilo=ilo, ihi=ihi, nb=nb, abft=abft)
    assert res.info == 0 and res.report.detected == 0, res.events
    check_against_oracle(A, dA, tau, ilo=ilo, ihi=ihi, nb=nb)
    tg = tau.cpu().numpy()
    assert np.all(tg[: ilo - 1] == 0.0) and np.all(tg[max(ihi - 1, 0): n - 1] == 0.0)


def test_padded_lda():
    A = synth.matrix(77)
    dA, tau, res = gpu_reduce(A, lda=83, nb=16)
    assert res.info == 0
    check_against_oracle(A, dA, tau, nb=16)


def test_exact_cases():
    """Already-Hessenberg input: tau = 0 and H = A exactly; symmetric input: tridiagonal H."""
    A = synth.hessenberg_matrix(96)
    dA, tau, res = gpu_reduce(A, nb=32)
    assert np.all(tau.cpu().numpy()[:95] == 0.0)
    assert np.array_equal(dA.cpu().numpy(), A)
    S = synth.symmetric_matrix(96)
    dS, tau, res = gpu_reduce(S, nb=32)
    H = np.triu(dS.cpu().numpy(), -1)
    assert np.abs(np.triu(H, 2)).max() <= 1e-13 * np.linalg.norm(S)


def test_dorghr_in_place():
    A = synth.matrix(130)
    dA, tau, res = gpu_reduce(A, nb=32)
    Qo = oracle.dorghr(*oracle.dgehd2(A))
    Q, info = ft.dorghr(dA, tau, Q=dA, nb=32)  # dQ aliases dA (ldq == lda)
    assert info == 0 and np.abs(Q.cpu().numpy() - Qo).max() <= TOL


def test_host_entry_point():
    A = synth.matrix(300)
    Ah = np.asfortranarray(A.copy())
    tau, res = ft.dgehrd_host(Ah, nb=32)
    assert res.info == 0
    Ao, to = oracle.dgehd2(A)
    assert rel(np.triu(Ah, -1), np.triu(Ao, -1)) <= TOL
    assert np.abs(tau - to).max() <= TOL


@pytest.mark.parametrize("n,nb,ilo,ihi", [(517, 32, 1, None), (300, 64, 7, 280)])
def test_host_entry_overlapped_copies(n, nb, ilo, ihi):
    """ft_dgehrd_host copies each iteration's finished columns back while the next panels run
    (and the untouched / last columns at the end): repeated calls (first call, graph capture,
    graph replay) all match the oracle, from pinned host memory like the bench."""
    import torch
    A = synth.matrix(n, ilo=ilo, ihi=ihi if ihi else n)
    Ao, to = oracle.dgehd2(A, ilo, ihi)
    pinned = torch.empty((n, n), dtype=torch.float64).pin_memory()
    for _ in range(3):
        Ah = pinned.numpy().T  # Fortran-ordered view of the pinned buffer
        Ah[:] = A
        tau, res = ft.dgehrd_host(Ah, ilo=ilo, ihi=ihi, nb=nb)
        assert res.info == 0 and res.report.detected == 0
        assert rel(np.triu(Ah, -1), np.triu(Ao, -1)) <= TOL
        assert np.abs(tau - to).max() <= TOL


def test_host_entry_with_fault():
    """A corrected fault on the host path: the matrix was touched by the recovery, so every
    column is copied back again at the end."""
    n = 300
    A = synth.matrix(n)
    Ao, to = oracle.dgehd2(A)
    Ah = np.asfortranarray(A.copy())
    tau, res = ft.dgehrd_host(Ah, nb=32, faults=[(2, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 150, 200, 55)])
    assert res.info == 0 and res.report.corrected >= 1, res.events
    assert rel(np.triu(Ah, -1), np.triu(Ao, -1)) <= TOL


# ------------------------------------------------------------------ checksum parity (Theorem 1)
@pytest.mark.parametrize("n,nb", [(64, 16), (300, 32), (513, 64), (256, 64), (320, 32)])
def test_checksums_at_every_boundary(n, nb):
    A = synth.matrix(n, dist="normal")
    normF = np.linalg.norm(A)
    npanel = (n - 2 + nb - 1) // nb
    for t in range(npanel):
        chk = torch.zeros(2 * n + 1, dtype=torch.float64, device="cuda")
        dA, tau, res = gpu_reduce(A, nb=nb, stop_after_panel=t, dchk_out=chk)
        assert res.info == 0
        info, Aw, tw, rep, chko = oracle.ft_dgehd2(A, nb, stop_after_panel=t)
        g = chk.cpu().numpy()
        assert np.abs(g - chko).max() <= 1e-10 * normF, (t, np.abs(g - chko).max())
        assert rel(dA.cpu().numpy(), Aw) <= TOL, t


@pytest.mark.parametrize("n,nb", [(256, 64), (320, 32), (513, 64), (1024, 32), (2048, 32)])
def test_right_update_row_fold_matches_tiles(n, nb):
    """The ABFT right update's column-checksum row c as a GEMV of the last row split (default)
    against c as one more DMMA tile row (ft_debug_right_fold(0)): H, tau and the maintained
    checksums at a mid boundary agree to rounding and both meet the oracle; flips of c before
    the panel and after the right update are still handled (located, or rolled back to the
    checkpoint that predates them)."""
    A = synth.matrix(n, dist="normal")
    L = ft.lib()
    L.ft_debug_right_fold.argtypes = [ctypes.c_int]
    t = ((n - 2 + nb - 1) // nb) // 2
    out = []
    for fold in (1, 0):
        L.ft_debug_right_fold(fold)
        try:
            chk = torch.zeros(2 * n + 1, dtype=torch.float64, device="cuda")
            dAs, _, rs = gpu_reduce(A, nb=nb, stop_after_panel=t, dchk_out=chk)
            dA, tau, res = gpu_reduce(A, nb=nb)
        finally:
            L.ft_debug_right_fold(1)
        assert rs.info == 0 and res.info == 0 and res.report.detected == 0, res.events
        check_against_oracle(A, dA, tau, nb=nb)
        out.append((dA.cpu().numpy(), chk.cpu().numpy()))
    (H1, c1), (H0, c0) = out
    assert rel(np.triu(H1, -1), np.triu(H0, -1)) <= 1e-11
    assert np.abs(c1 - c0).max() <= 1e-11 * np.linalg.norm(A)
    for ph, site, i, j in ((ft.PHASE_BEFORE_PANEL, ft.SITE_C, -1, n - 3), (ft.PHASE_AFTER_RIGHT, ft.SITE_C, -1, n - 3),
                           (ft.PHASE_AFTER_RIGHT, ft.SITE_K, -1, -1)):
        dA, tau, res = gpu_reduce(A, nb=nb, faults=[(1, ph, site, i, j, 52)])
        assert res.info == 0 and res.report.detected + res.report.rollbacks >= 1, res.events
        check_against_oracle(A, dA, tau, nb=nb)


@pytest.mark.parametrize("n,nb", [(300, 32), (2048, 32), (3000, 64)])
@pytest.mark.parametrize("site", [ft.SITE_R, ft.SITE_C, ft.SITE_K])
def test_end_check_deferred_and_fused(n, nb, site):
    """The end-of-iteration check (Alg. 3 l.12-13) of every iteration but the last is evaluated at
    the entry of the next panel launch (deferred, no last-CTA chain on the left update's tail); the
    last iteration's in the left update itself (fused).  A checksum flip after the right update
    fails it either way: the iteration is rolled back (ROLLBACK at that panel, reason 8) before
    anything of the next panel is stored, and the result meets the oracle."""
    A = synth.matrix(n)
    npan = (n - 2 + nb - 1) // nb
    i, j = (n // 3, -1) if site == ft.SITE_R else ((-1, n - 5) if site == ft.SITE_C else (-1, -1))
    for t in (1, npan - 1):  # deferred, fused
        dA, tau, res = gpu_reduce(A, nb=nb, faults=[(t, ft.PHASE_AFTER_RIGHT, site, i, j, 53)])
        assert res.info == 0, res.events
        rb = [e for e in res.events if e[0] == "ROLLBACK"]
        assert rb and rb[0][1] == t and rb[0][2] == 8, res.events
        check_against_oracle(A, dA, tau, nb=nb)


@pytest.mark.parametrize("n,nb", [(256, 64), (320, 32), (513, 64), (1024, 32)])
def test_left_update_fold_matches_tiles(n, nb):
    """The ABFT left update's checksum row/column folded into the last tile row / strip
    (default) against the same row/column as extra DMMA tiles (ft_debug_left_fold(0)): H, tau
    and the maintained checksums at a mid boundary agree to rounding; both meet the oracle."""
    A = synth.matrix(n, dist="normal")
    L = ft.lib()
    L.ft_debug_left_fold.argtypes = [ctypes.c_int]
    t = ((n - 2 + nb - 1) // nb) // 2
    out = []
    for fold in (1, 0):
        L.ft_debug_left_fold(fold)
        try:
            chk = torch.zeros(2 * n + 1, dtype=torch.float64, device="cuda")
            dAs, _, rs = gpu_reduce(A, nb=nb, stop_after_panel=t, dchk_out=chk)
            dA, tau, res = gpu_reduce(A, nb=nb)
        finally:
            L.ft_debug_left_fold(1)
        assert rs.info == 0 and res.info == 0 and res.report.detected == 0, res.events
        check_against_oracle(A, dA, tau, nb=nb)
        out.append((dA.cpu().numpy(), chk.cpu().numpy()))
    (H1, c1), (H0, c0) = out
    assert rel(np.triu(H1, -1), np.triu(H0, -1)) <= 1e-11  # panel atomics: rounding-level run-to-run
    assert np.abs(c1 - c0).max() <= 1e-11 * np.linalg.norm(A)


# ------------------------------------------------------------------ fault injection
def faulty(A, nb, faults, **kw):
    return gpu_reduce(A, nb=nb, faults=faults, **kw)


def fixes(events, kinds=("FIX_DATA", "FIX_R", "FIX_C", "FIX_K", "FIX_Q", "FIX_QR", "FIX_QC", "FIX_QK")):
    return sorted((e[0], e[2], e[3]) for e in events if e[0] in kinds)


ORA_SITE = {ft.SITE_A: oracle.SITE_A, ft.SITE_R: oracle.SITE_R, ft.SITE_C: oracle.SITE_C, ft.SITE_K: oracle.SITE_K}


@pytest.mark.parametrize("site,i,j,bit", [
    (ft.SITE_A, 40, 50, 51),   # C1 default: area 2 at panel 1, bit 51
    (ft.SITE_A, 40, 50, 62),   # catastrophic exponent flip (R14)
    (ft.SITE_A, 40, 50, 63),   # sign
    (ft.SITE_A, 5, 50, 55),    # area 1 (rows above the panel)
    (ft.SITE_A, 20, 16, 45),   # the panel column about to be factorized
    (ft.SITE_A, 60, 63, 52),   # last row / column
    (ft.SITE_R, 33, -1, 55),
    (ft.SITE_R, 3, -1, 62),
    (ft.SITE_C, -1, 61, 52),
    (ft.SITE_C, -1, 7, 50),    # checksum of a finished column
    (ft.SITE_K, -1, -1, 48),
])
def test_c1_before_panel_fault_matches_oracle(site, i, j, bit):
    n, nb = 64, 16
    A = synth.matrix(n)
    dA, tau, res = faulty(A, nb, [(1, ft.PHASE_BEFORE_PANEL, site, i, j, bit)])
    assert res.info == 0, res.events
    check_against_oracle(A, dA, tau, nb=nb)
    info, Af, tf, rep, _ = oracle.ft_dgehd2(A, nb, faults=[(1, ORA_SITE[site], i, j, bit)])
    assert info == 0
    ora_fix = [(k, a, b) for (k, a, b) in fixes(rep.events())]
    assert fixes(res.events) == ora_fix, (res.events, rep.events())


@pytest.mark.parametrize("bit", list(range(0, 64, 3)) + [52, 62, 63])
@pytest.mark.parametrize("site,i,j", [(ft.SITE_A, 40, 50), (ft.SITE_A, 10, 40), (ft.SITE_R, 45, -1),
                                      (ft.SITE_C, -1, 45)])
def test_bit_sweep_detect_or_harmless(site, i, j, bit):
    """R16: a flip with |delta| > tau_abs is detected and corrected; a smaller one is harmless."""
    n, nb = 64, 16
    A = synth.matrix(n, dist="normal")
    dA, tau, res = faulty(A, nb, [(2, ft.PHASE_BEFORE_PANEL, site, i, j, bit)])
    assert res.info == 0, res.events
    check_against_oracle(A, dA, tau, nb=nb)
    delta = [e[4] for e in res.events if e[0] == "INJECT"][0]
    tau_abs = 2.0 * n * EPS * np.linalg.norm(A)
    if not (abs(delta) <= tau_abs):
        assert res.report.detected >= 1, (bit, delta, res.events)


@pytest.mark.parametrize("phase", [ft.PHASE_AFTER_PANEL, ft.PHASE_AFTER_RIGHT, ft.PHASE_AFTER_UPDATE])
@pytest.mark.parametrize("i,j,bit", [(40, 70, 51), (70, 90, 56), (10, 80, 63), (40, 70, 60)])
def test_mid_iteration_faults(phase, i, j, bit):
    n, nb = 128, 32
    A = synth.matrix(n)
    dA, tau, res = faulty(A, nb, [(1, phase, ft.SITE_A, i, j, bit)])
    assert res.info == 0, res.events
    assert res.report.detected >= 1
    check_against_oracle(A, dA, tau, nb=nb)


@pytest.mark.parametrize("site,i,j,bit", [(ft.SITE_Y, 50, 3, 45), (ft.SITE_Y, 100, 0, 62), (ft.SITE_Y, 10, 5, 51),
                                          (ft.SITE_V, 60, 2, 50), (ft.SITE_V, 80, 7, 62)])
def test_workspace_faults_redo_panel(site, i, j, bit):
    """R15: Y/V corrupted between the panel and the updates -> pre-update check -> redo."""
    n, nb = 128, 32
    A = synth.matrix(n)
    dA, tau, res = faulty(A, nb, [(1, ft.PHASE_AFTER_PANEL, site, i, j, bit)])
    assert res.info == 0, res.events
    assert res.report.panel_redos >= 1 or res.report.rollbacks >= 1, res.events
    check_against_oracle(A, dA, tau, nb=nb)


@pytest.mark.parametrize("i,j,bit", [(30, 3, 50), (100, 40, 62), (90, 70, 45)])
def test_area3_and_finished_h_corrected_at_end(i, j, bit):
    n, nb = 128, 32
    A = synth.matrix(n)
    # (i >= j+2 in a finished column: stored Householder vector; else finished H)
    dA, tau, res = faulty(A, nb, [(0, ft.PHASE_AT_END, ft.SITE_A, i, j, bit)])
    assert res.info == 0, res.events
    check_against_oracle(A, dA, tau, nb=nb)
    assert any(e[0] in ("FIX_Q", "FIX_DATA") and e[1] == -1 for e in res.events), res.events


def test_c3_style_simultaneous_faults():
    """C3 pattern at reduced size: two trailing flips (distinct rows/cols), a panel-workspace
    flip (AFTER_PANEL) and a checksum flip, all in one iteration."""
    n, nb = 512, 64
    A = synth.matrix(n)
    faults = [(3, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 300, 400, 55),
              (3, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 350, 450, 47),
              (3, ft.PHASE_AFTER_PANEL, ft.SITE_Y, 380, 3, 60),
              (3, ft.PHASE_BEFORE_PANEL, ft.SITE_C, -1, 420, 52)]
    dA, tau, res = faulty(A, nb, faults)
    assert res.info == 0, res.events
    check_against_oracle(A, dA, tau, nb=nb)
    got = fixes(res.events)
    assert ("FIX_DATA", 300, 400) in got and ("FIX_DATA", 350, 450) in got and ("FIX_C", -1, 420) in got


def test_uncorrectable_is_reported():
    """A rectangle of equal flips cannot be decoded: info = FT_E_UNCORRECTABLE, never a wrong answer."""
    n, nb = 64, 16
    A = np.ones((n, n)) + np.eye(n)  # entries 1.0: flipping mantissa bit 51 adds exactly +0.5 to each
    f = [(0, ft.PHASE_BEFORE_PANEL, ft.SITE_A, i, j, 51) for (i, j) in [(30, 40), (30, 50), (35, 40), (35, 50)]]
    dA, tau, res = faulty(A, nb, f)
    assert res.info == ft.FT_E_UNCORRECTABLE
    assert res.report.uncorrectable >= 1


@pytest.mark.parametrize("site,i,j", [("area3", 53, 16), ("area1", 31, 127), ("area2", 63, 127)])
def test_fig2_workload_matches_oracle(site, i, j):
    """NEXT-2, the paper's Fig. 2 workload: ABFT off, one soft error after iteration 1
    (N = 158, nb = 32, bit 52 of A(i, j)).  The GPU's polluted reduction equals the oracle's
    (unprotected reduction of the same corrupted matrix: ora_ft_dgehd2 with detection disabled) at the
    parity bar, and the propagation pattern -- which entries of the packed H / V differ from the
    fault-free result -- is the paper's: one entry (area 3), one row of H (area 1), almost all of H
    after column 32 and much of V (area 2); the polluted-entry counts agree within 1 %."""
    n, nb = 158, 32
    A = synth.matrix(n)
    Ao, to = oracle.dgehd2(A)
    dA, tau, res = faulty(A, nb, [(1, ft.PHASE_BEFORE_PANEL, ft.SITE_A, i, j, 52)], abft=False)
    assert res.info == 0 and res.report.detected == 0
    Ag, tg = dA.cpu().numpy(), tau.cpu().numpy()[: n - 1]
    info, Af, tf, rep, _ = oracle.ft_dgehd2(A, nb, c_thr=1e300, faults=[(1, oracle.SITE_A, i, j, 52)])
    assert info == 0 and rep.detected == 0
    assert rel(Ag, Af) <= TOL, rel(Ag, Af)
    assert np.abs(tg - tf).max() <= TOL * max(1.0, np.abs(tf).max())
    thr = 1e-12 * np.abs(Ao).max()
    dg, do = np.abs(Ag - Ao) > thr, np.abs(Af - Ao) > thr
    assert abs(int(dg.sum()) - int(do.sum())) <= max(1, do.sum() // 100), (dg.sum(), do.sum())
    Hm = np.triu(np.ones((n, n), bool), -1)
    if site == "area3":
        assert dg.sum() == 1 and dg[i, j]
    elif site == "area1":
        assert list(np.unique(np.nonzero(dg)[0])) == [i] and dg[i, 33:].mean() > 0.9
    else:
        assert dg[:, 33:][Hm[:, 33:]].mean() > 0.9 and dg[:, 33:][~Hm[:, 33:]].mean() > 0.3


def test_wide_panel_kernel_large():
    """n = 6144, nb = 64: the early panels have >= 32 rows per CTA and run the two-reduction
    wide kernel (ft_panel_wide.cu); the late ones the one-reduction kernel.  The oracle is too
    slow here, so: agreement with the all-one-reduction-kernel run (explicit path forced) to
    rounding, and the backward-error / orthogonality bounds of the north star, on the GPU."""
    n, nb = 6144, 64
    A = synth.matrix(n)
    dA, tau, res = gpu_reduce(A, nb=nb)
    assert res.info == 0 and res.report.detected == 0
    L = ft.lib()
    L.ft_debug_panel_path.argtypes = [ctypes.c_int]
    L.ft_debug_panel_path(8)
    try:
        dB, tauB, resB = gpu_reduce(A, nb=nb)
    finally:
        L.ft_debug_panel_path(0)
    assert resB.info == 0
    H, HB = torch.triu(dA, -1), torch.triu(dB, -1)
    assert float((H - HB).abs().max()) <= 1e-10 * float(HB.abs().max())
    # the last reflectors are ill-conditioned functions of the data (two correct implementations
    # differ by ~1e-12 at n = 1024 and ~5e-9 at n = 6144 there, R18); H above is norm-wise 1e-10
    assert float((tau - tauB).abs().max()) <= 1e-7
    Q, info = ft.dorghr(dA, tau, nb=nb)
    assert info == 0
    Ad = torch.from_numpy(A).cuda()
    eps = 2.0 ** -52
    n1 = lambda M: float(M.abs().sum(0).max())  # 1-norm
    resid = n1(Ad - Q @ H @ Q.T) / (n * n1(Ad) * eps)
    orth = n1(torch.eye(n, dtype=torch.float64, device="cuda") - Q.T @ Q) / (n * eps)
    assert resid <= 30 and orth <= 30, (resid, orth)


# ------------------------------------------------------------------ T (block-reflector factor)
@pytest.mark.parametrize("n,nb,i,j,bit", [(128, 32, 3, 10, 55), (128, 32, 0, 0, 52), (128, 32, 7, 31, 62),
                                          (600, 32, 5, 20, 45), (300, 64, 40, 60, 63)])
def test_t_fault_after_panel_rolled_back(n, nb, i, j, bit):
    """R15 extended to T: a flip in the upper triangle of T between the panel and the updates
    (the entries W' = T^T W reads) fails the T checksum where the right update forms W'; the
    right update is rolled back and the panel redone.  Result at the oracle bar."""
    A = synth.matrix(n)
    dA, tau, res = faulty(A, nb, [(1, ft.PHASE_AFTER_PANEL, ft.SITE_T, i, j, bit)])
    assert res.info == 0, res.events
    assert any(e[0] == "ROLLBACK" and e[1] == 1 and e[2] == 32 for e in res.events), res.events
    assert res.report.rollbacks >= 1
    check_against_oracle(A, dA, tau, nb=nb)


@pytest.mark.parametrize("phase,i,j", [(ft.PHASE_AFTER_PANEL, 10, 3),   # strict lower triangle: never read
                                       (ft.PHASE_AFTER_RIGHT, 3, 10),   # after W' = T^T W was formed
                                       (ft.PHASE_AFTER_UPDATE, 2, 2)])
def test_t_fault_harmless_positions(phase, i, j):
    """T words the remaining steps of the iteration never read: no detection, no effect."""
    n, nb = 128, 32
    A = synth.matrix(n)
    dA, tau, res = faulty(A, nb, [(1, phase, ft.SITE_T, i, j, 61)])
    assert res.info == 0, res.events
    assert res.report.detected == 0 and res.report.rollbacks == 0, res.events
    check_against_oracle(A, dA, tau, nb=nb)


def test_policy_paper_fault_detect_rollback_locate_redo():
    """POLICY_PAPER (R11, the paper's own detection): the scalar |sum r - sum c| test at the end of
    the iteration (Alg. 3 l.12-13) -> reverse computation (l.14) -> location by recomputation and
    correction -> redo.  A flip mid-update in area 2 and one before the panel."""
    n, nb = 256, 32
    A = synth.matrix(n)
    for f in [(2, ft.PHASE_AFTER_RIGHT, ft.SITE_A, 150, 200, 55), (3, ft.PHASE_AFTER_UPDATE, ft.SITE_A, 130, 220, 57),
              (2, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 120, 230, 54)]:
        dA, tau, res = faulty(A, nb, [f], policy=ft.POLICY_PAPER)
        assert res.info == 0, (f, res.events)
        assert res.report.rollbacks >= 1, (f, res.events)
        assert ("FIX_DATA", f[3], f[4]) in fixes(res.events), (f, res.events)
        check_against_oracle(A, dA, tau, nb=nb)


# ------------------------------------------------------------------ NEXT-4: symmetric tridiagonal reduction
@pytest.mark.parametrize("n,nb", [(64, 16), (300, 32), (1000, 64)])
def test_dsytrd_matches_oracle(n, nb):
    """ft_dsytrd (DSYTRD 'L' semantics on the protected path): d, e, tau and V equal the oracle's
    reduction of the symmetric matrix (pinned to LAPACK dsytrd in test_oracle.py) at the parity bar;
    the strict upper triangle of the caller's array is not touched; Q T Q^T reproduces A."""
    S = synth.symmetric_matrix(n)
    A = np.asfortranarray(np.tril(S) + 7.0 * np.triu(np.ones((n, n)), 1))  # garbage above: not referenced
    dA = ft.fortran(torch.from_numpy(A).cuda())
    d, e, tau, res = ft.dsytrd(dA, nb=nb)
    torch.cuda.synchronize()
    assert res.info == 0 and res.report.detected == 0, res.events
    Ao, to = oracle.dgehd2(S)
    sc = np.abs(Ao).max()
    assert np.abs(d.cpu().numpy() - np.diag(Ao)).max() <= TOL * sc
    assert np.abs(e.cpu().numpy() - np.diag(Ao, -1)).max() <= TOL * sc
    assert np.abs(tau.cpu().numpy() - to).max() <= TOL
    Ag = dA.cpu().numpy()
    assert np.abs(np.tril(Ag, -2) - np.tril(Ao, -2)).max() <= TOL
    assert np.array_equal(np.triu(Ag, 1), np.triu(A, 1))
    tpad = torch.cat([tau, torch.zeros(1, dtype=torch.float64, device="cuda")])
    Q, info = ft.dorghr(dA, tpad, nb=nb)
    Qg = Q.cpu().numpy()
    T = np.diag(d.cpu().numpy()) + np.diag(e.cpu().numpy(), -1) + np.diag(e.cpu().numpy(), 1)
    assert np.linalg.norm(S - Qg @ T @ Qg.T, 1) / (n * np.linalg.norm(S, 1) * EPS) <= 30


def test_dsytrd_fault_corrected():
    """The ABFT machinery on the symmetric path: a flip in the trailing block before a panel is located
    and corrected; the tridiagonal meets the oracle bar."""
    n, nb = 300, 32
    S = synth.symmetric_matrix(n)
    dA = ft.fortran(torch.from_numpy(S).cuda())
    d, e, tau, res = ft.dsytrd(dA, nb=nb, faults=[(2, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 150, 200, 55)])
    torch.cuda.synchronize()
    assert res.info == 0 and ("FIX_DATA", 150, 200) in fixes(res.events), res.events
    Ao, to = oracle.dgehd2(S)
    assert np.abs(e.cpu().numpy() - np.diag(Ao, -1)).max() <= TOL * np.abs(Ao).max()
