"""Pins of the CPU oracle against things other than itself (-m "not gpu").

Each test states what fixes the expected value:
  * a library routine (LAPACK dgehrd/dorghr via scipy) for the whole reduction,
  * the n = 3 worked example (tests/golden/n3_closed_form.json),
  * exact special cases (already-Hessenberg, symmetric -> tridiagonal,
    integer-valued encoding),
  * invariants of a similarity (trace, Frobenius norm, eigenvalues, Q e1 = e1,
    Q^T Q = I, residual),
  * Theorem 1: maintained checksums equal recomputed ones,
  * brute force over every <= 2-fault placement of the decoder (R12),
  * the paper's Fig. 2 propagation pattern.
"""
import itertools
import json
import os

import numpy as np
import pytest
from scipy.linalg import lapack

import synth

EPS = 2.0 ** -52
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def resid_ratio(A, H, Q):
    n = A.shape[0]
    return np.linalg.norm(A - Q @ H @ Q.T, 1) / (n * np.linalg.norm(A, 1) * EPS)


def orth_ratio(Q):
    n = Q.shape[0]
    return np.linalg.norm(np.eye(n) - Q.T @ Q, 1) / (n * EPS)


# ---------------------------------------------------------------- LAPACK pin
@pytest.mark.parametrize("n,dist", [(5, "uniform"), (64, "uniform"), (64, "normal"),
                                    (129, "normal"), (300, "uniform")])
def test_matches_lapack_dgehrd(ora, n, dist):
    A = synth.matrix(n, dist=dist)
    Ao, tau = ora.dgehd2(A)
    hq, tq, info = lapack.dgehrd(A)
    assert info == 0
    H, Hl = np.triu(Ao, -1), np.triu(hq, -1)
    assert np.abs(H - Hl).max() / np.abs(Hl).max() <= 1e-12
    assert np.abs(tau - tq[: n - 1]).max() <= 1e-12 * max(1.0, np.abs(tq).max())
    V, Vl = np.tril(Ao, -2), np.tril(hq, -2)
    assert np.abs(V - Vl).max() <= 1e-10
    Q = ora.dorghr(Ao, tau)
    Ql, info = lapack.dorghr(hq, tq)
    assert info == 0
    assert np.abs(Q - Ql).max() <= 1e-12


@pytest.mark.parametrize("n,ilo,ihi", [(40, 1, 40), (40, 5, 40), (40, 1, 31), (40, 7, 29), (40, 20, 21), (40, 40, 40)])
def test_ilo_ihi_matches_lapack(ora, n, ilo, ihi):
    A = synth.matrix(n, seed=7 + ilo + 3 * ihi, ilo=ilo, ihi=ihi)
    Ao, tau = ora.dgehd2(A, ilo, ihi)
    hq, tq, info = lapack.dgehrd(A, lo=ilo - 1, hi=ihi - 1)
    assert info == 0
    assert np.abs(np.triu(Ao, -1) - np.triu(hq, -1)).max() <= 1e-12 * np.abs(hq).max()
    assert np.abs(tau - tq[: n - 1]).max() <= 1e-12
    # tau is zero outside the active block (LAPACK contract)
    assert np.all(tau[: ilo - 1] == 0.0) and np.all(tau[max(ihi - 1, 0):] == 0.0)
    Q = ora.dorghr(Ao, tau, ilo, ihi)
    Ql, _ = lapack.dorghr(hq, tq, lo=ilo - 1, hi=ihi - 1)
    assert np.abs(Q - Ql).max() <= 1e-12
    H = np.triu(Ao, -1)
    assert resid_ratio(A, H, Q) <= 30 and orth_ratio(Q) <= 30


# ---------------------------------------------------------------- tiny cases
@pytest.mark.parametrize("n", [0, 1, 2])
def test_no_reflectors(ora, n):
    A = synth.matrix(n) if n else np.zeros((0, 0))
    Ao, tau = ora.dgehd2(A)
    assert np.array_equal(Ao, A)
    assert np.all(tau == 0.0)
    if n:
        assert np.array_equal(ora.dorghr(Ao, tau), np.eye(n))


def test_n3_closed_form(ora):
    g = json.load(open(os.path.join(GOLDEN, "n3_closed_form.json")))
    A = np.array(g["A"], dtype=np.float64)
    Ao, tau = ora.dgehd2(A)
    np.testing.assert_allclose(tau, g["tau"], rtol=0, atol=1e-15)
    assert Ao[1, 0] == g["beta"]
    np.testing.assert_allclose(Ao[2, 0], g["v"][2], rtol=0, atol=1e-16)
    np.testing.assert_allclose(np.triu(Ao, -1), g["H"], rtol=0, atol=4e-15)


# ---------------------------------------------------------------- exact cases
def test_already_hessenberg_is_identity_bitwise(ora):
    A = synth.hessenberg_matrix(50)
    Ao, tau = ora.dgehd2(A)
    assert np.all(tau == 0.0)
    assert np.array_equal(Ao, A)
    assert np.array_equal(ora.dorghr(Ao, tau), np.eye(50))


def test_symmetric_gives_tridiagonal(ora):
    S = synth.symmetric_matrix(80)
    Ao, tau = ora.dgehd2(S)
    H = np.triu(Ao, -1)
    assert np.abs(np.triu(H, 2)).max() <= 1e-14 * np.linalg.norm(S)
    # and H is symmetric up to rounding
    assert np.abs(H - H.T).max() <= 1e-13 * np.linalg.norm(S)


def test_encoding_exact_on_integers(ora):
    rng = np.random.default_rng(3)
    A = rng.integers(-1000, 1000, size=(37, 37)).astype(np.float64)
    r, c, k = ora.encode(A)
    Ai = A.astype(np.int64)
    assert np.array_equal(r, Ai.sum(axis=1).astype(np.float64))
    assert np.array_equal(c, Ai.sum(axis=0).astype(np.float64))
    assert k == float(Ai.sum())


# ---------------------------------------------------------------- invariants
@pytest.mark.parametrize("dist", ["uniform", "normal"])
def test_similarity_invariants(ora, dist):
    n = 16
    A = synth.matrix(n, seed=99, dist=dist)
    Ao, tau = ora.dgehd2(A)
    H = np.triu(Ao, -1)
    Q = ora.dorghr(Ao, tau)
    assert abs(np.trace(H) - np.trace(A)) <= 10 * n * EPS * np.linalg.norm(A)
    assert abs(np.linalg.norm(H) - np.linalg.norm(A)) <= 10 * n * EPS * np.linalg.norm(A)
    ea = np.sort_complex(np.linalg.eigvals(A))
    eh = np.sort_complex(np.linalg.eigvals(H))
    assert np.abs(ea - eh).max() <= 1e-10 * np.linalg.norm(A)
    e1 = np.zeros(n); e1[0] = 1.0
    assert np.array_equal(Q @ e1, e1) and np.array_equal(Q[0], e1)
    assert resid_ratio(A, H, Q) <= 30
    assert orth_ratio(Q) <= 30


@pytest.mark.parametrize("n", [256, 400])
def test_residual_and_orthogonality_paper_magnitudes(ora, n):
    """Table II / III: MAGMA-level residuals ~1e-18..1e-17, orthogonality ~4e-17."""
    A = synth.matrix(n)
    Ao, tau = ora.dgehd2(A)
    H = np.triu(Ao, -1)
    Q = ora.dorghr(Ao, tau)
    paper_res = np.linalg.norm(A - Q @ H @ Q.T, 1) / (n * np.linalg.norm(A, 1))
    paper_orth = np.linalg.norm(Q @ Q.T - np.eye(n), 1) / n
    assert paper_res < 1e-16 and paper_orth < 1e-15
    assert resid_ratio(A, H, Q) <= 30 and orth_ratio(Q) <= 30


# ---------------------------------------------------------------- ABFT bookkeeping
def _logical(Ao, ilo, ihi, cdone):
    n = Ao.shape[0]
    L = Ao.copy()
    for j in range(max(ilo - 1, 0), min(cdone, ihi - 1)):
        L[j + 2: ihi, j] = 0.0
    return L


@pytest.mark.parametrize("n,nb,dist,ilo,ihi", [(64, 16, "uniform", 1, 64), (200, 32, "normal", 1, 200),
                                               (150, 32, "uniform", 4, 131)])
def test_theorem1_checksums_at_every_boundary(ora, n, nb, dist, ilo, ihi):
    """Theorem 1: r = L e and c = e^T L stay valid; kappa = e^T L e (R22)."""
    A = synth.matrix(n, dist=dist, ilo=ilo, ihi=ihi)
    normF = np.linalg.norm(A)
    npanel = (ihi - 2 - (ilo - 1) + nb) // nb
    for t in range(npanel):
        info, Aw, tau, rep, chk = ora.ft_dgehd2(A, nb, ilo, ihi, stop_after_panel=t)
        assert info == 0
        cdone = min(ilo - 1 + (t + 1) * nb, ihi - 1)
        L = _logical(Aw, ilo, ihi, cdone)
        r, c, k = chk[:n], chk[n:2 * n], chk[2 * n]
        unit = n * EPS * normF
        assert np.abs(r - L.sum(axis=1)).max() <= 0.5 * unit
        assert np.abs(c - L.sum(axis=0)).max() <= 0.5 * unit
        assert abs(k - L.sum()) <= 0.5 * unit * np.sqrt(n)
    # the fault-free run leaves A identical to the plain reduction and reports nothing
    info, Af, tauf, rep, _ = ora.ft_dgehd2(A, nb, ilo, ihi)
    Ao, tau = ora.dgehd2(A, ilo, ihi)
    assert info == 0 and rep.detected == 0 and rep.nevents == 0
    assert np.array_equal(Af, Ao) and np.array_equal(tauf, tau)
    assert rep.max_drift < 0.5


# ---------------------------------------------------------------- injector
@pytest.mark.parametrize("bit", [0, 30, 51, 52, 62, 63])
def test_flip_is_one_bit(ora, bit):
    x = 0.7312
    y = ora.flip(x, bit)
    a = np.array([x]).view(np.uint64)[0]
    b = np.array([y]).view(np.uint64)[0]
    assert bin(int(a ^ b)).count("1") == 1 and int(a ^ b) == 1 << bit


# ---------------------------------------------------------------- decoder truth tables
def _decoder_case(ora, n=8, seed=0):
    A = synth.matrix(n, seed=seed, dist="normal")
    r, c, k = ora.encode(A)
    tau = 2.0 * n * EPS * np.linalg.norm(A)
    return A, r, c, k, tau


def _apply(A, r, c, k, site, bit, ora):
    A, r, c = A.copy(order="F"), r.copy(), c.copy()
    kind, i, j = site
    if kind == "A":
        A[i, j] = ora.flip(A[i, j], bit)
    elif kind == "r":
        r[i] = ora.flip(r[i], bit)
    elif kind == "c":
        c[j] = ora.flip(c[j], bit)
    else:
        k = ora.flip(k, bit)
    return A, r, c, k


def _sites(n):
    s = [("A", i, j) for i in range(n) for j in range(n)]
    s += [("r", i, -1) for i in range(n)] + [("c", -1, j) for j in range(n)] + [("k", -1, -1)]
    return s


def _exact(A0, r0, c0, k0, L, r, c, k, n):
    scale = n * EPS * max(1.0, np.abs(A0).max()) * 8
    return (np.abs(L - A0).max() <= scale and np.abs(r - r0).max() <= scale * n
            and np.abs(c - c0).max() <= scale * n and abs(k - k0) <= scale * n * n)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_decoder_every_single_fault_corrected(ora, seed):
    n = 8
    A, r, c, k, tau = _decoder_case(ora, n, seed)
    for site in _sites(n):
        for bit in (45, 51, 62, 63):
            Af, rf, cf, kf = _apply(A, r, c, k, site, bit, ora)
            res, L, r2, c2, k2, rep = ora.decode(Af, rf, cf, kf, tau)
            assert res == 1, (site, bit, rep.events())
            assert _exact(A, r, c, k, L, r2, c2, k2, n), (site, bit)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_decoder_never_miscorrects_two_faults(ora, seed):
    """Brute force over every pair of fault sites x bit pairs (R12): exact or refused."""
    n = 8
    A, r, c, k, tau = _decoder_case(ora, n, seed)
    sites = _sites(n)
    bitpairs = [(45, 51), (51, 51), (62, 45), (63, 51), (52, 60), (62, 63)]
    corrected = refused = 0
    for s1, s2 in itertools.combinations(sites, 2):
        for b1, b2 in bitpairs:
            Af, rf, cf, kf = _apply(A, r, c, k, s1, b1, ora)
            Af, rf, cf, kf = _apply(Af, rf, cf, kf, s2, b2, ora)
            res, L, r2, c2, k2, rep = ora.decode(Af, rf, cf, kf, tau)
            if res == 1:
                assert _exact(A, r, c, k, L, r2, c2, k2, n), (s1, s2, b1, b2, rep.events())
                corrected += 1
            else:
                assert res == 2, (s1, s2, b1, b2)
                refused += 1
    assert corrected > 0.8 * (corrected + refused)


def test_decoder_refuses_rectangle_and_l_shape(ora):
    """errors forming a rectangle are not correctable.  A tied rectangle and an
    L-shape whose syndromes pair with nothing must be refused.  (With one checksum
    pair some 3-error patterns have exactly the syndrome of a 2-error pattern; no
    decoder can tell them apart -- DESIGN.md, decoder limits.)"""
    n = 8
    A, r, c, k, tau = _decoder_case(ora, n, 5)
    for pattern in ([(1, 2, 0.25), (1, 5, 0.25), (4, 2, 0.25), (4, 5, 0.25)],
                    [(1, 2, 0.25), (1, 5, 0.5), (4, 2, 1.0)]):
        Af = A.copy(order="F")
        for (i, j, d) in pattern:
            Af[i, j] += d
        res, *_ = ora.decode(Af, r, c, k, tau)
        assert res == 2


# ---------------------------------------------------------------- end-to-end fault runs
def _fault_free(ora, A, nb, ilo=1, ihi=None):
    Ao, tau = ora.dgehd2(A, ilo, ihi if ihi else A.shape[0])
    return Ao, tau


@pytest.mark.parametrize("site,i,j,bit", [
    (0, 40, 50, 51),    # C1 default: area 2 at panel 1, bit 51
    (0, 5, 50, 62),     # area 1 (rows above the panel), catastrophic exponent flip
    (0, 40, 50, 63),    # sign
    (0, 20, 16, 45),    # panel column being factorised next
    (1, 33, -1, 55),    # r
    (2, -1, 61, 52),    # c
    (3, -1, -1, 48),    # kappa
])
def test_c1_single_fault_corrected(ora, site, i, j, bit):
    n, nb = 64, 16
    A = synth.matrix(n)
    Ao, tau = _fault_free(ora, A, nb)
    info, Af, tauf, rep, _ = ora.ft_dgehd2(A, nb, faults=[(1, site, i, j, bit)])
    assert info == 0, rep.events()
    ev = rep.events()
    assert any(e[0] == "DETECT" and e[1] == 1 for e in ev)
    if site == 0:
        assert any(e[0] == "FIX_DATA" and e[2] == i and e[3] == j for e in ev)
    H, Hf = np.triu(Ao, -1), np.triu(Af, -1)
    assert np.abs(H - Hf).max() / np.abs(H).max() <= 1e-12
    assert np.abs(tau - tauf).max() <= 1e-12


def test_area3_fault_corrected_at_end(ora):
    n, nb = 64, 16
    A = synth.matrix(n)
    Ao, tau = _fault_free(ora, A, nb)
    # stored Householder vector (finished column 3) hit at boundary 2 (area 3)
    info, Af, tauf, rep, _ = ora.ft_dgehd2(A, nb, faults=[(2, 0, 30, 3, 50)])
    assert info == 0
    assert any(e[0] == "FIX_Q" and e[2] == 30 and e[3] == 3 for e in rep.events())
    assert np.abs(Af - Ao).max() <= 1e-14


def test_finished_h_fault_corrected_at_end(ora):
    n, nb = 64, 16
    A = synth.matrix(n)
    Ao, tau = _fault_free(ora, A, nb)
    info, Af, tauf, rep, _ = ora.ft_dgehd2(A, nb, faults=[(-1, 0, 3, 10, 50)])
    assert info == 0
    assert any(e[0] == "FIX_DATA" and e[1] == -1 for e in rep.events())
    assert np.abs(np.triu(Af, -1) - np.triu(Ao, -1)).max() <= 1e-13


def test_simultaneous_faults(ora):
    n, nb = 128, 32
    A = synth.matrix(n, dist="normal")
    Ao, tau = _fault_free(ora, A, nb)
    faults = [(2, 0, 80, 100, 55), (2, 0, 90, 110, 47), (2, 2, -1, 120, 52)]
    info, Af, tauf, rep, _ = ora.ft_dgehd2(A, nb, faults=faults)
    assert info == 0, rep.events()
    assert np.abs(np.triu(Af, -1) - np.triu(Ao, -1)).max() <= 1e-12 * np.abs(Ao).max()


# ---------------------------------------------------------------- Fig. 2
def test_fig2_propagation_patterns(ora):
    """ABFT off (threshold disabled), one error after iteration 1, N=158, nb=32."""
    n, nb = 158, 32
    A = synth.matrix(n)
    Ao, tau = ora.dgehd2(A)
    off = 1e300  # no detection: the error propagates as in the paper's heat maps

    def diff(i, j):
        info, Af, tf, rep, _ = ora.ft_dgehd2(A, nb, c_thr=off, faults=[(1, 0, i, j, 52)])
        return np.abs(Af - Ao) > 1e-12 * np.abs(Ao).max()

    d = diff(53, 16)           # area 3: finished Householder vector, does not propagate
    assert d.sum() == 1 and d[53, 16]
    d = diff(31, 127)          # area 1: pollutes one row of H (row 31, columns after the panel)
    rows = np.unique(np.nonzero(d)[0])
    assert list(rows) == [31] and d[31, 33:].mean() > 0.9
    d = diff(63, 127)          # area 2: pollutes almost all of H after column 32, and much of Q
    H = np.triu(np.ones((n, n), bool), -1)
    assert d[:, 33:][H[:, 33:]].mean() > 0.9
    assert d[:, 33:][~H[:, 33:]].mean() > 0.3


@pytest.mark.parametrize("seed", [0, 1])
def test_decoder_borderline_flips_never_refused_or_wrong(ora, seed):
    """Flips whose syndrome sits between tau_abs and tau_abs*sqrt(n) (the sum tolerance):
    every single checksum-word flip is corrected, every data flip is corrected or left
    below the detection threshold (R16), none is refused or miscorrected."""
    n = 16
    A = synth.matrix(n, seed=seed, dist="normal")
    r, c, k = ora.encode(A)
    tau = 2.0 * n * EPS * np.linalg.norm(A)
    for bit in range(0, 20):
        for site in [("r", 3, -1), ("c", -1, 5), ("A", 7, 9), ("A", 0, 15)]:
            Af, rf, cf, kf = _apply(A, r, c, k, site, bit, ora)
            res, L, r2, c2, k2, rep = ora.decode(Af, rf, cf, kf, tau)
            assert res in (0, 1), (site, bit, rep.events())
            assert np.abs(L - A).max() <= 2 * tau, (site, bit)


# ---------------------------------------------------------------- NEXT-1: weighted checksum pair
def _wsums(L):
    n = L.shape[0]
    w = np.arange(1, n + 1, dtype=float)
    rw, cw = L @ w, w @ L
    return rw, cw, float(rw.sum()), float(cw.sum())


@pytest.mark.parametrize("n,nb,dist", [(64, 16, "normal"), (200, 32, "uniform"), (150, 64, "normal")])
def test_weighted_theorem1_at_every_boundary(ora, n, nb, dist):
    """Theorem 1 holds for any weight vector: r_w = L w, c_w = w^T L and the corners
    e^T L w, w^T L e maintained per reflector equal their recomputation at every boundary, and the
    plain pair is unchanged by carrying the weighted one."""
    A = synth.matrix(n, dist=dist)
    normF = np.linalg.norm(A)
    npanel = (n - 2 + nb - 1) // nb
    for t in range(npanel):
        info, Aw, tw, rep, chk = ora.ft_dgehd2(A, nb, stop_after_panel=t, weighted=True)
        assert info == 0 and rep.detected == 0
        info0, Aw0, _, _, chk0 = ora.ft_dgehd2(A, nb, stop_after_panel=t)
        assert np.array_equal(Aw, Aw0) and np.array_equal(chk[: 2 * n + 1], chk0)
        L = _logical(Aw, 1, n, min((t + 1) * nb, n - 1))
        rw, cw, krw, kcw = _wsums(L)
        unit = n * EPS * normF * n  # weighted sums carry weights up to n
        assert np.abs(chk[2 * n + 1: 3 * n + 1] - rw).max() <= 0.5 * unit, t
        assert np.abs(chk[3 * n + 1: 4 * n + 1] - cw).max() <= 0.5 * unit, t
        assert abs(chk[4 * n + 1] - krw) <= 0.5 * unit * n and abs(chk[4 * n + 2] - kcw) <= 0.5 * unit * n


def _wcase(ora, n=8, seed=0):
    A = synth.matrix(n, seed=seed, dist="normal")
    r, c, k = ora.encode(A)
    rw, cw, krw, kcw = _wsums(A)
    tau = 2.0 * n * EPS * np.linalg.norm(A)
    return A, r, c, k, rw, cw, krw, kcw, tau


def _wapply(st, site, bit, ora):
    A, r, c, k, rw, cw = st[0].copy(order="F"), st[1].copy(), st[2].copy(), st[3], st[4].copy(), st[5].copy()
    kind, i, j = site
    if kind == "A":
        A[i, j] = ora.flip(A[i, j], bit)
    elif kind == "r":
        r[i] = ora.flip(r[i], bit)
    elif kind == "c":
        c[j] = ora.flip(c[j], bit)
    elif kind == "rw":
        rw[i] = ora.flip(rw[i], bit)
    elif kind == "cw":
        cw[j] = ora.flip(cw[j], bit)
    else:
        k = ora.flip(k, bit)
    return A, r, c, k, rw, cw


def _wsites(n):
    return _sites(n) + [("rw", i, -1) for i in range(n)] + [("cw", -1, j) for j in range(n)]


def _wexact(A0, L, r0, r, c0, c, rw0, rw, cw0, cw, n):
    scale = n * EPS * max(1.0, np.abs(A0).max()) * 8
    return (np.abs(L - A0).max() <= scale and np.abs(r - r0).max() <= scale * n and np.abs(c - c0).max() <= scale * n
            and np.abs(rw - rw0).max() <= scale * n * n and np.abs(cw - cw0).max() <= scale * n * n)


@pytest.mark.parametrize("seed", [0, 1])
def test_weighted_decoder_singles_and_never_miscorrects_pairs(ora, seed):
    """Decoder v3 brute force (n = 8): every single fault at every site -- data, r, c, kappa, r_w,
    c_w -- is corrected; every pair of sites x bit pairs is corrected exactly or refused, never
    wrong; and it corrects at least as many pairs as the single pair's decoder (v2)."""
    n = 8
    A, r, c, k, rw, cw, krw, kcw, tau = _wcase(ora, n, seed)
    st = (A, r, c, k, rw, cw)
    for site in _wsites(n):
        for bit in (45, 51, 62, 63):
            Af, rf, cf, kf, rwf, cwf = _wapply(st, site, bit, ora)
            res, L, r2, c2, k2, rw2, cw2, krw2, kcw2, rep = ora.decode_w(Af, rf, cf, kf, rwf, cwf, krw, kcw, tau)
            assert res == 1, (site, bit, rep.events())
            assert _wexact(A, L, r, r2, c, c2, rw, rw2, cw, cw2, n), (site, bit)
    sites = _wsites(n)
    bitpairs = [(45, 51), (51, 51), (62, 45), (52, 60)]
    ok_w = ok_v2 = refused = 0
    for s1, s2 in itertools.combinations(sites, 2):
        for b1, b2 in bitpairs:
            f = _wapply(st, s1, b1, ora)
            f = _wapply(f, s2, b2, ora)
            res, L, r2, c2, k2, rw2, cw2, krw2, kcw2, rep = ora.decode_w(*f, krw, kcw, tau)
            if res == 1:
                assert _wexact(A, L, r, r2, c, c2, rw, rw2, cw, cw2, n), (s1, s2, b1, b2, rep.events())
                ok_w += 1
            else:
                assert res == 2
                refused += 1
            if s1[0] in "Ark" and s2[0] in "Ark":
                res2, *_ = ora.decode(*f[:4], tau)
                ok_v2 += res2 == 1
    assert ok_w > 0.9 * (ok_w + refused) and ok_w >= ok_v2, (ok_w, refused, ok_v2)


@pytest.mark.parametrize("seed", range(6))
def test_weighted_decoder_fixes_ten_tied_flips(ora, seed):
    """ten flips in one iteration with tied discrepancies (entries 1.0, mantissa bit
    51: every delta is exactly +0.5) defeat the single pair (v2 refuses: pairing by value is
    ambiguous); the weighted pair locates each by D_w / D = w and corrects all ten.  Rectangles
     are still refused."""
    n = 64
    rng = np.random.default_rng(seed)
    A = np.ones((n, n)) + np.eye(n)
    r, c, k = ora.encode(A)
    rw, cw, krw, kcw = _wsums(A)
    tau = 2.0 * n * EPS * np.linalg.norm(A)
    rows = rng.choice(n, 10, replace=False)
    cols = rng.choice(n, 10, replace=False)
    Af = A.copy(order="F")
    for i, j in zip(rows, cols):
        Af[i, j] = ora.flip(Af[i, j], 51)
    assert ora.decode(Af, r, c, k, tau)[0] == 2
    res, L, *_ , rep = ora.decode_w(Af, r, c, k, rw, cw, krw, kcw, tau)
    assert res == 1, rep.events()
    assert np.abs(L - A).max() <= 1e-14
    Ar = A.copy(order="F")
    for (i, j) in [(3, 7), (3, 20), (40, 7), (40, 20)]:
        Ar[i, j] = ora.flip(Ar[i, j], 51)
    assert ora.decode_w(Ar, r, c, k, rw, cw, krw, kcw, tau)[0] == 2


def _tied_positions(W, lo, count, rng):
    """count positions (distinct rows and columns, both >= lo) of values in [0.5, 1) whose mantissa
    bit 51 is clear: flipping it adds exactly +0.25 to each (a tie pattern)."""
    n = W.shape[0]
    bits = W.view(np.uint64)
    ok = (np.abs(W) >= 0.5) & (np.abs(W) < 1.0) & ((bits >> np.uint64(51)) & np.uint64(1) == 0) & (W > 0)
    rows, cols, out = set(), set(), []
    for i, j in zip(*np.nonzero(ok)):
        if i >= lo and j >= lo and i not in rows and j not in cols and rng.random() < 0.3:
            out.append((int(i), int(j)))
            rows.add(i)
            cols.add(j)
        if len(out) == count:
            break
    return out


def test_weighted_end_to_end_tied_flips(ora):
    """The unblocked ABFT reduction with the weighted pair on (weighted=1): ten flips with tied
    discrepancies (+0.25 each) in the trailing matrix at boundary 1 are all located and corrected,
    and the reduction equals the fault-free one; with the single pair the same run stops
    uncorrectable (R12 refuses the ambiguous pairing)."""
    n, nb = 128, 32
    A = synth.matrix(n)
    Ao, tau = _fault_free(ora, A, nb)
    _, W, _, _, _ = ora.ft_dgehd2(A, nb, stop_after_panel=0)  # the working matrix at boundary 1
    pos = _tied_positions(np.asfortranarray(W), 40, 10, np.random.default_rng(1))
    assert len(pos) == 10
    faults = [(1, 0, i, j, 51) for (i, j) in pos]
    info, Af, tf, rep, _ = ora.ft_dgehd2(A, nb, faults=faults, weighted=True)
    assert info == 0, rep.events()
    assert sorted((e[2], e[3]) for e in rep.events() if e[0] == "FIX_DATA") == sorted(pos)
    assert np.abs(np.triu(Af, -1) - np.triu(Ao, -1)).max() <= 1e-12 * np.abs(Ao).max()
    info1, *_ = ora.ft_dgehd2(A, nb, faults=faults)
    assert info1 == 1


def test_symmetric_hessenberg_is_lapack_dsytrd(ora):
    """NEXT-4 pin: for symmetric A the unblocked Householder Hessenberg reduction (DGEHD2 conventions,
    R1) is LAPACK's DSYTRD (uplo 'L'): the same diagonal d, subdiagonal e, tau and reflectors V."""
    from scipy.linalg import lapack
    for n in (17, 120, 333):
        S = synth.symmetric_matrix(n)
        c, d, e, tau, info = lapack.dsytrd(S, lower=1)
        assert info == 0
        Ao, to = ora.dgehd2(S)
        sc = max(np.abs(d).max(), np.abs(e).max())  # norm-wise (R18)
        assert np.abs(np.diag(Ao) - d).max() <= 1e-12 * sc
        assert np.abs(np.diag(Ao, -1) - e).max() <= 1e-12 * sc
        # the last reflectors are ill-conditioned functions of the data (R18): two correct codes differ
        # by ~1e-12 there; a convention error (sign, scaling, index) would be O(1)
        assert np.abs(to - tau).max() <= 1e-10
        assert np.abs(np.tril(Ao, -2) - np.tril(c, -2)).max() <= 1e-10
