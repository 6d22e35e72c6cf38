"""Checksum-protected Q formation (NEXT-3; ft_dorghr with opts.abft = 1) against the
oracle's DORGHR (ora_dorghr, pinned to LAPACK dorghr in test_oracle.py).

Q = H(ilo) ... H(ihi-1) is accumulated backward with the DMMA update kernels while a row checksum
r = Q e, a column checksum c = e^T Q and kappa = e^T Q e ride through every left update (Theorem 1,
P:268-274).  Bar: Q within 1e-9 of the oracle (norm-wise max entry, R18) and orthogonality ratio
<= 30 (R17), with and without injected soft errors; errors are located at the positions the
propagation rules predict (a data error only travels along its own column: left multiplications
never mix columns), never corrected wrongly.
"""
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


def reduced(n, nb, seed=None, ilo=1, ihi=None):
    A = synth.matrix(n, seed=seed, ilo=ilo, ihi=ihi if ihi else n)
    dA = ft.fortran(torch.from_numpy(A).cuda())
    tau, res = ft.dgehrd(dA, nb=nb, ilo=ilo, ihi=ihi)
    torch.cuda.synchronize()
    assert res.info == 0
    Ao, to = oracle.dgehd2(A, ilo, ihi)
    Qo = oracle.dorghr(Ao, to, ilo, ihi)
    return A, dA, tau, Qo


def orth_ratio(Q):
    n = Q.shape[0]
    return np.linalg.norm(np.eye(n) - Q.T @ Q, 1) / (n * EPS)


@pytest.mark.parametrize("n,nb,ilo,ihi", [(64, 16, 1, None), (300, 32, 1, None), (517, 64, 1, None),
                                          (150, 32, 4, 131), (1000, 32, 1, None)])
def test_protected_q_matches_oracle(n, nb, ilo, ihi):
    A, dA, tau, Qo = reduced(n, nb, ilo=ilo, ihi=ihi)
    for abft in (True, False):
        Q, res = ft.dorghr(dA, tau, ilo=ilo, ihi=ihi, nb=nb, abft=abft, full=True)
        torch.cuda.synchronize()
        assert res.info == 0 and res.report.detected == 0, res.events
        Qg = Q.cpu().numpy()
        assert np.abs(Qg - Qo).max() <= TOL, (abft, np.abs(Qg - Qo).max())
        assert orth_ratio(Qg) <= 30


def fixes(events):
    return [(e[0], e[2], e[3]) for e in events if e[0].startswith("FIX")]


@pytest.mark.parametrize("phase,t,i,j,bit", [
    (ft.PHASE_BEFORE_PANEL, 4, 200, 250, 55),    # inside the block the iteration updates
    (ft.PHASE_BEFORE_PANEL, 4, 100, 100, 52),    # diagonal entry not yet reached (Q = I there)
    (ft.PHASE_AFTER_UPDATE, 6, 260, 270, 50),
    (ft.PHASE_BEFORE_PANEL, 8, 299, 299, 63),    # sign of the last diagonal entry
    (ft.PHASE_AT_END, 0, 123, 45, 47),
])
def test_q_data_fault_corrected(phase, t, i, j, bit):
    """A flipped word of Q mid-accumulation: the left updates carry the error down its column only,
    the final verification finds one flagged column and the flagged rows, and every polluted entry is
    repaired with the row formula; Q meets the oracle bar."""
    n, nb = 300, 32
    A, dA, tau, Qo = reduced(n, nb)
    Q, res = ft.dorghr(dA, tau, nb=nb, faults=[(t, phase, ft.SITE_A, i, j, bit)], full=True)
    torch.cuda.synchronize()
    assert res.info == 0, res.events
    assert res.report.detected >= 1
    fx = fixes(res.events)
    assert ("FIX_DATA", i, j) in fx, fx
    assert all(k == "FIX_DATA" and jj == j for (k, ii, jj) in fx), fx  # one column only
    Qg = Q.cpu().numpy()
    assert np.abs(Qg - Qo).max() <= TOL, np.abs(Qg - Qo).max()
    assert orth_ratio(Qg) <= 30


@pytest.mark.parametrize("phase,site,i,j,bit,fix", [
    (ft.PHASE_BEFORE_PANEL, ft.SITE_R, 150, -1, 55, "FIX_R"),
    (ft.PHASE_AFTER_UPDATE, ft.SITE_R, 280, -1, 50, "FIX_R"),
    (ft.PHASE_BEFORE_PANEL, ft.SITE_C, -1, 220, 53, "FIX_C"),
    (ft.PHASE_AFTER_UPDATE, ft.SITE_C, -1, 40, 51, "FIX_C"),
    (ft.PHASE_BEFORE_PANEL, ft.SITE_K, -1, -1, 49, "FIX_K"),
])
def test_q_checksum_fault_rolled_back_and_refreshed(phase, site, i, j, bit, fix):
    """A flipped checksum word: the iteration's sum check (sum r = sum c = kappa) fails, the left
    update is added back with the retained W' (reverse computation), the full verification
    locates the word and refreshes it from the data, and the accumulation is redone."""
    n, nb = 300, 32
    A, dA, tau, Qo = reduced(n, nb)
    Q, res = ft.dorghr(dA, tau, nb=nb, faults=[(5, phase, site, i, j, bit)], full=True)
    torch.cuda.synchronize()
    assert res.info == 0, res.events
    assert res.report.rollbacks >= 1, res.events
    fx = fixes(res.events)
    assert fx and all(k == fix for (k, _, _) in fx), fx
    Qg = Q.cpu().numpy()
    assert np.abs(Qg - Qo).max() <= TOL
    assert orth_ratio(Qg) <= 30


def test_q_catastrophic_flip_is_refused_not_wrong():
    """Exponent bit 62 of a Q entry inside the updated block becomes ~1e308 / inf and is consumed by
    the update before any check (no verify-before-consume in Q formation): the add-back cannot undo it
    (R14), so the call reports FT_E_UNCORRECTABLE -- or corrects it -- but never returns a wrong Q."""
    n, nb = 300, 32
    A, dA, tau, Qo = reduced(n, nb)
    Q, res = ft.dorghr(dA, tau, nb=nb, faults=[(4, ft.PHASE_BEFORE_PANEL, ft.SITE_A, 200, 250, 62)], full=True)
    torch.cuda.synchronize()
    if res.info == 0:
        assert np.abs(Q.cpu().numpy() - Qo).max() <= TOL
    else:
        assert res.info == ft.FT_E_UNCORRECTABLE and res.report.uncorrectable >= 1
