"""NEXT-1 on the GPU: the weighted checksum pair (opts.weighted = 1, w_i = i + 1) against the oracle's
weighted bookkeeping and decoder v3 (oracle.ft_dgehd2(..., weighted=True), pinned in test_oracle.py).

r_w = L w and c_w = w^T L ride as column / row n+1 of the augmented array through the same DMMA
update tiles (Theorem 1 holds for any weight vector); the decoder locates each error of a
tied or L-shaped pattern by D_w / D = w, which the single pair cannot.
Bar: the parity bar of test_gpu.py; weighted checksums at every boundary <= 1e-10 n ||A||_F.
"""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
TOL = 1e-9

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_ipps_jiald16_b200 as ft  # noqa: E402


def rel(a, b):
    return np.abs(a - b).max() / max(np.abs(b).max(), 1e-300)


def run(A, nb, faults=(), stop=-1, weighted=True, **kw):
    n = A.shape[0]
    dA = ft.fortran(torch.from_numpy(A).cuda())
    chk = torch.zeros(4 * n + 3, dtype=torch.float64, device="cuda") if stop >= 0 else None
    tau, res = ft.dgehrd(dA, nb=nb, faults=faults, stop_after_panel=stop, dchk_out=chk, weighted=weighted, **kw)
    torch.cuda.synchronize()
    return dA.cpu().numpy(), tau.cpu().numpy()[: n - 1], res, (chk.cpu().numpy() if chk is not None else None)


def fixes(events):
    return sorted((e[0], e[2], e[3]) for e in events if e[0].startswith("FIX"))


@pytest.mark.parametrize("n,nb", [(64, 16), (300, 32), (517, 64), (2700, 64)])
def test_weighted_fault_free_parity(n, nb):
    A = synth.matrix(n)
    Ag, tg, res, _ = run(A, nb)
    assert res.info == 0 and res.report.detected == 0, res.events
    Ao, to = oracle.dgehd2(A)
    assert rel(np.triu(Ag, -1), np.triu(Ao, -1)) <= TOL
    assert np.abs(tg - to).max() <= TOL * max(1.0, np.abs(to).max())


@pytest.mark.parametrize("n,nb", [(64, 16), (300, 32), (256, 64)])
def test_weighted_checksums_at_every_boundary(n, nb):
    A = synth.matrix(n, dist="normal")
    normF = np.linalg.norm(A)
    for t in range((n - 2 + nb - 1) // nb):
        Ag, _, res, chk = run(A, nb, stop=t)
        assert res.info == 0
        info, Aw, tw, rep, chko = oracle.ft_dgehd2(A, nb, stop_after_panel=t, weighted=True)
        assert rel(Ag, Aw) <= TOL, t
        assert np.abs(chk[: 2 * n + 1] - chko[: 2 * n + 1]).max() <= 1e-10 * normF, t
        assert np.abs(chk[2 * n + 1:] - chko[2 * n + 1:]).max() <= 1e-10 * n * normF, t


def tied_positions(W, lo, count, rng):
    ok = (W >= 0.5) & (W < 1.0) & ((W.view(np.uint64) >> np.uint64(51)) & np.uint64(1) == 0)
    rows, cols, out = set(), set(), []
    for i, j in zip(*np.nonzero(ok)):
        if i >= lo and j >= lo and i not in rows and j not in cols and rng.random() < 0.3:
            out.append((int(i), int(j)))
            rows.add(i)
            cols.add(j)
        if len(out) == count:
            break
    return out


@pytest.mark.parametrize("n,nb,seed", [(128, 32, 1), (300, 32, 2), (600, 64, 3)])
def test_ten_tied_flips_located_by_the_weighted_pair(n, nb, seed):
    """Ten flips at one boundary whose discrepancies tie (+0.25 each, mantissa bit 51 of values in
    [0.5, 1)): the single pair refuses (uncorrectable), the weighted pair corrects all ten; the GPU's
    fix list equals the oracle's and the result meets the parity bar."""
    A = synth.matrix(n)
    _, W, _, _, _ = oracle.ft_dgehd2(A, nb, stop_after_panel=0)  # the working matrix at boundary 1
    pos = tied_positions(np.asfortranarray(W), nb + 8, 10, np.random.default_rng(seed))
    assert len(pos) == 10
    faults = [(1, ft.PHASE_BEFORE_PANEL, ft.SITE_A, i, j, 51) for (i, j) in pos]
    Ag, tg, res, _ = run(A, nb, faults=faults)
    assert res.info == 0, res.events
    got = fixes(res.events)
    assert sorted((i, j) for (k, i, j) in got if k == "FIX_DATA") == sorted(pos), got
    info, Af, tf, rep, _ = oracle.ft_dgehd2(A, nb, faults=[(1, oracle.SITE_A, i, j, 51) for (i, j) in pos],
                                            weighted=True)
    assert info == 0
    assert got == fixes(rep.events()), (got, rep.events())
    Ao, to = oracle.dgehd2(A)
    assert rel(np.triu(Ag, -1), np.triu(Ao, -1)) <= TOL
    # the paper's single pair: the same run stops uncorrectable
    _, _, res1, _ = run(A, nb, faults=faults, weighted=False)
    assert res1.info == ft.FT_E_UNCORRECTABLE


def test_l_shape_corrected_rectangle_refused():
    """errors not forming a rectangle are correctable -- with the weighted pair an L-shape is
    (two in a row, two in a column); a rectangle of equal flips is still refused, never wrong."""
    n, nb = 128, 32
    A = np.asfortranarray(synth.matrix(n) * 0.5 + 0.5)  # values in [0.5, 1)
    Ao, to = oracle.dgehd2(A)
    L = [(1, ft.PHASE_BEFORE_PANEL, ft.SITE_A, i, j, 50) for (i, j) in [(60, 70), (60, 90), (100, 70)]]
    Ag, tg, res, _ = run(A, nb, faults=L)
    assert res.info == 0, res.events
    assert {(i, j) for (k, i, j) in fixes(res.events) if k == "FIX_DATA"} == {(60, 70), (60, 90), (100, 70)}
    assert rel(np.triu(Ag, -1), np.triu(Ao, -1)) <= TOL
    R = [(0, ft.PHASE_BEFORE_PANEL, ft.SITE_A, i, j, 51) for (i, j) in [(60, 70), (60, 90), (100, 70), (100, 90)]]
    _, _, res, _ = run(np.ones((n, n)) + np.eye(n), nb, faults=R)
    assert res.info == ft.FT_E_UNCORRECTABLE


@pytest.mark.parametrize("site,i,j,bit,kind", [(ft.SITE_RW, 77, -1, 55, "FIX_RW"), (ft.SITE_CW, -1, 150, 52, "FIX_CW"),
                                               (ft.SITE_RW, 5, -1, 62, "FIX_RW")])
def test_weighted_words_refreshed(site, i, j, bit, kind):
    n, nb = 300, 32
    A = synth.matrix(n)
    Ag, tg, res, _ = run(A, nb, faults=[(2, ft.PHASE_BEFORE_PANEL, site, i, j, bit)])
    assert res.info == 0, res.events
    assert (kind, i, j) in fixes(res.events), res.events
    Ao, to = oracle.dgehd2(A)
    assert rel(np.triu(Ag, -1), np.triu(Ao, -1)) <= TOL


@pytest.mark.parametrize("phase,i,j,bit", [(ft.PHASE_AFTER_RIGHT, 150, 200, 55), (ft.PHASE_AFTER_UPDATE, 170, 220, 57),
                                           (ft.PHASE_AT_END, 120, 30, 50)])
def test_weighted_mid_iteration_and_end_faults(phase, i, j, bit):
    n, nb = 300, 32
    A = synth.matrix(n)
    Ag, tg, res, _ = run(A, nb, faults=[(2, phase, ft.SITE_A, i, j, bit)])
    assert res.info == 0, res.events
    assert res.report.detected >= 1
    Ao, to = oracle.dgehd2(A)
    assert rel(np.triu(Ag, -1), np.triu(Ao, -1)) <= TOL
