"""CPU pins of the panel's one-reduction column algebra (ft_panel.cu).

scripts/proto_onesync.py is a numpy model of the blocked reduction whose DLAHR2 column loop
evaluates ||x||^2, alpha, e^T x, t and y from the reduction of b0 alone (the carried Gram
G = V_x^T V_x, or K = G T^T updated by the rank-2 recurrence of tcol_gram, and Z = A V_x),
with the explicit column as the cancellation fallback.  In exact arithmetic it is the plain
loop, so H and tau must match the oracle (the unblocked DGEHD2 definition, pinned in
test_oracle.py) to rounding; and the guard must trip rarely on the bench's inputs.
"""
import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "scripts"))

import oracle  # noqa: E402
import proto_onesync as P  # noqa: E402
import synth  # noqa: E402


@pytest.mark.parametrize("dist", ["uniform", "normal"])
@pytest.mark.parametrize("n,nb", [(70, 16), (161, 32)])
@pytest.mark.parametrize("carry_k", [False, True])
def test_onesync_model_matches_oracle(dist, n, nb, carry_k):
    A = synth.matrix(n, dist=dist)
    Ao, to = oracle.dgehd2(A)
    st = {"trip": 0, "cols": 0}
    H, tau = P.blocked(A, nb, True, stats=st, carry_k=carry_k)
    Ho = np.triu(Ao, -1)
    assert np.abs(np.triu(H, -1) - Ho).max() <= 1e-12 * np.abs(Ho).max()
    assert np.abs(tau - to).max() <= 1e-11
    assert st["trip"] <= 2, st  # the explicit fallback is the exception, not the rule


def test_onesync_guard_on_hessenberg_input():
    """Already-Hessenberg input: x = 0 in every column, so ||x||^2 must come out exactly 0
    (tau = 0, H = A) -- the expansion cannot leave rounding noise there."""
    n = 40
    A = np.triu(synth.matrix(n), -1)
    H, tau = P.blocked(A, 16, True, stats={"trip": 0, "cols": 0}, carry_k=True)
    assert np.all(tau == 0.0)
    assert np.array_equal(np.triu(H, -1), A)
