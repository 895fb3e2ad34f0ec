"""Pins for the oracle's Kuhn-Munkres solver (Sec. III): brute
force over all S! rearrangements (Eq. 3), the LP dual certificate,
scipy's independent solver, and the zero-optimum of a tile shuffle."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_yangin17_b200 import synth


def _check_certificate(E, r, c, p, q):
    E = E.astype(np.int64)
    S = E.shape[0]
    assert sorted(r.tolist()) == list(range(S))
    assert c == sum(int(E[r[v], v]) for v in range(S))
    assert (p[:, None] + q[None, :] <= E).all(), "dual feasibility"
    assert all(p[r[v]] + q[v] == E[r[v], v] for v in range(S)), "complementary slackness"
    assert int(p.sum() + q.sum()) == c, "strong duality => optimal"


@pytest.mark.parametrize("S", [1, 2, 3, 4, 5, 6, 7, 8])
def test_hungarian_vs_brute_force(S):
    rng = np.random.default_rng(100 + S)
    for hi in (3, 1000, 200000):
        E = rng.integers(0, hi, size=(S, S)).astype(np.int32)
        r, c, p, q = oracle.hungarian(E)
        assert c == oracle.brute_force(E)[0]
        _check_certificate(E, r, c, p, q)


def test_hungarian_dual_certificate_images():
    I, T = synth.make_pair("smooth", 128, 8, 3, seed=1)
    E = oracle.error_matrix(I, T, 8)
    _check_certificate(E, *oracle.hungarian(E))


def test_hungarian_vs_scipy():
    scipy_opt = pytest.importorskip("scipy.optimize")
    for fam in ("smooth", "noise"):
        I, T = synth.make_pair(fam, 128, 8, 3, seed=2)
        E = oracle.error_matrix(I, T, 8)
        rows, cols = scipy_opt.linear_sum_assignment(E)
        assert oracle.hungarian(E)[1] == int(E[rows, cols].astype(np.int64).sum())


def test_hungarian_shuffle_optimum_zero():
    I, T = synth.make_pair("shuffle", 128, 8, 3, seed=3)
    E = oracle.error_matrix(I, T, 8)
    r, c, p, q = oracle.hungarian(E)
    assert c == 0
