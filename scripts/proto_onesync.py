#!/usr/bin/env python3
"""Prototype (numpy) of the one-reduction-per-column DLAHR2 column loop used by k_panel.

Plain DLAHR2 (LAPACK reading R2) needs two grid-wide reductions per column: s1 = V^T b0
(for b = b0 - V T^T s1) and then ||x||^2 of the new b.  The one-sync form reduces, from
b0 alone, s1 = V^T b0, sx = V_x^T b0_x, bb = b0_x.b0_x, b0(c+1) (x = rows >= c+2), and
gets everything else from quantities every CTA holds:
    w      = T^T s1
    ||x||^2 = bb - 2 w.sx + w^T G w        G = V_x^T V_x (Gram over rows >= c+2, downdated)
    alpha  = b0(c+1) - V(c+1,:) w
    t      = V^T v = V(c+1,:)^T + scale (sx - G w)
    y      = A0(:, c+1) + scale (A0(:, c+2:) b0_x - Z w)   Z = A0(:, c+2:) V_x (downdated)
A guard falls back to the explicit two-reduction column when ||x||^2 < gamma * bb
(cancellation).  This script checks the algebra against the plain loop and counts guard
trips on the bench's input distributions.
"""
import sys

import numpy as np

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))


def dlarfg(alpha, xx):
    if xx == 0.0:
        return 0.0, alpha, 1.0
    beta = -np.copysign(np.sqrt(alpha * alpha + xx), alpha)
    return (beta - alpha) / beta, beta, 1.0 / (alpha - beta)


def panel(A, k, ib, onesync, gamma, stats, carry_k=False):
    n = A.shape[0]
    A0 = A.copy()
    rows = np.arange(n)
    V = np.zeros((n, ib))
    Y = np.zeros((n, ib))
    T = np.zeros((ib, ib))
    Z = np.zeros((n, ib))
    G = np.zeros((ib, ib))
    Km = np.zeros((ib, ib))  # K = Gp T^T (carry_k): G w = K s1 - V(c+1,:)^T q
    tprev = None
    for j in range(ib):
        c = k + j
        act = rows >= k + 1
        b0 = np.where(act, A0[:, c] - Y[:, :j] @ V[c, :j], 0.0)
        xm = rows >= c + 2
        s1 = V[:, :j].T @ b0
        sx = V[xm, :j].T @ b0[xm]
        bb = b0[xm] @ b0[xm]
        b0c1 = b0[c + 1]
        vr1 = V[c + 1, :j].copy()
        if onesync and j > 0:
            # Gram over rows >= c+2: previous Gram (rows >= c+1) minus row c+1, new column from t
            vr0 = V[c, :j - 1]
            G[:j - 1, :j - 1] -= np.outer(vr1[:j - 1], vr1[:j - 1])
            gcol = tprev[:j - 1] - vr0 * 1.0 - vr1[:j - 1] * V[c + 1, j - 1]
            G[:j - 1, j - 1] = gcol
            G[j - 1, :j - 1] = gcol
            G[j - 1, j - 1] = xxprev * scaleprev ** 2 - V[c + 1, j - 1] ** 2
            # Z over columns >= c+2
            Z[:, :j] -= np.outer(A0[:, c + 1], vr1)
        w = T[:j, :j].T @ s1
        fast = onesync
        if onesync and carry_k:
            Gw = Km[:j, :j] @ s1 - vr1 * (vr1 @ w)
            xx = bb - 2.0 * (w @ sx) + w @ Gw
            alpha = b0c1 - vr1 @ w
            if not (xx >= gamma * (bb + w @ Gw)):
                fast = False
                stats["trip"] += 1
        elif onesync:
            Gw = G[:j, :j] @ w
            xx = bb - 2.0 * (w @ sx) + w @ Gw
            alpha = b0c1 - vr1 @ w
            if not (xx >= gamma * bb):
                fast = False
                stats["trip"] += 1
        b = b0 - V[:, :j] @ w
        if not fast:
            alpha = b[c + 1]
            xx = b[xm] @ b[xm]
        tau, beta, scale = dlarfg(alpha, xx) if c + 2 < n else (0.0, alpha, 1.0)
        if c + 2 >= n:
            xx = 0.0
        v = np.zeros(n)
        v[c + 1] = 1.0
        v[xm] = scale * b[xm]
        V[:, j] = v
        A[act & (rows <= c), c] = b[act & (rows <= c)]
        A[c + 1, c] = beta
        A[xm, c] = v[xm]
        if fast:
            g = A0[:, c + 2:] @ b0[c + 2:]
            u = scale * (g - Z[:, :j] @ w)
            t = vr1 + scale * (sx - Gw)
        else:
            u = scale * (A0[:, c + 2:] @ b[c + 2:])
            t = V[:, :j].T @ v
        Z[:, j] = u
        y = np.where(act, A0[:, c + 1] + u, 0.0)
        Y[:, j] = np.where(act, tau * (y - Y[:, :j] @ t), 0.0)
        if carry_k:  # K_new = Gp_new T_new^T by the rank-2 update of ft_panel.cu (tcol_gram)
            st = T[:j, :j] @ t
            su = T[:j, :j] @ vr1
            g_ = t - vr1
            sigma = scale * scale * xx
            tc = -tau * st
            Kn = np.zeros((ib, ib))
            Kn[:j, :j] = Km[:j, :j] - np.outer(vr1, su) + np.outer(g_, tc)
            Kn[:j, j] = g_ * tau
            Kn[j, :j] = (st - su) + sigma * tc
            Kn[j, j] = sigma * tau
            Km = Kn
        T[:j, j] = -tau * (T[:j, :j] @ t)
        T[j, j] = tau
        tprev, xxprev, scaleprev = t, xx, scale
        stats["cols"] += 1
    return V, Y, T


def blocked(A, nb, onesync, gamma=1.0 / 64, stats=None, carry_k=False):
    A = A.copy()
    n = A.shape[0]
    tau = np.zeros(n - 1)
    k = 0
    while k < n - 2:
        ib = min(nb, n - 2 - k)
        e = k + ib
        A0 = A.copy()
        V, Y, T = panel(A, k, ib, onesync, gamma, stats, carry_k)
        tau[k:e] = np.diag(T)
        Ytop = A0[: k + 1, k + 1:] @ V[k + 1:, :] @ T
        Yf = Y.copy()
        Yf[: k + 1] = Ytop
        A[: k + 1, k + 1:e] -= Ytop @ V[k + 1:e].T
        A[:, e:] -= Yf @ V[e:].T
        W = V[k + 1:].T @ A[k + 1:, e:]
        A[k + 1:, e:] -= V[k + 1:] @ (T.T @ W)
        k = e
    return A, tau


def main():
    import oracle
    import synth

    for dist in ("uniform", "normal"):
        for n, nb in ((130, 16), (300, 32), (517, 32), (1024, 32)):
            A = synth.matrix(n, dist=dist) if "dist" in synth.matrix.__code__.co_varnames else synth.matrix(n)
            Ao, to = oracle.dgehd2(A)
            st = {"trip": 0, "cols": 0}
            H1, t1 = blocked(A, nb, True, stats=st)
            H0, t0 = blocked(A, nb, False, stats={"trip": 0, "cols": 0})
            Ho = np.triu(Ao, -1)
            d1 = np.abs(np.triu(H1, -1) - Ho).max() / np.abs(Ho).max()
            d0 = np.abs(np.triu(H0, -1) - Ho).max() / np.abs(Ho).max()
            dt = np.abs(t1 - to).max()
            print(f"{dist:8s} n={n:5d} nb={nb}: one-sync |dH|={d1:.2e} |dtau|={dt:.2e}  plain |dH|={d0:.2e}"
                  f"  guard trips {st['trip']}/{st['cols']}")


if __name__ == "__main__":
    main()
