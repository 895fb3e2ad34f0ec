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


# --- pins for tests/_certificate.py (the check the GPU auction is held to) ---
from tests._certificate import eps_cs_violations, is_permutation  # noqa: E402


@pytest.mark.parametrize("S", [2, 3, 5, 8])
def test_certificate_accepts_lp_duals_and_rejects_suboptimal(S):
    """Hungarian column duals q give prices p = -(S+1) q that satisfy CS with
    eps = 0 on the optimum; an assignment strictly worse than the brute-force
    optimum admits no certificate, in particular not this one."""
    rng = np.random.default_rng(300 + S)
    for hi in (4, 1000):
        E = rng.integers(0, hi, size=(S, S)).astype(np.int32)
        r, c, p, q = oracle.hungarian(E)
        assert c == oracle.brute_force(E)[0]
        price = -(S + 1) * q
        assert eps_cs_violations(E, r, price, eps=0) == 0
        for _ in range(20):
            bad = rng.permutation(S).astype(np.int32)
            cb = sum(int(E[bad[v], v]) for v in range(S))
            assert is_permutation(bad)
            if cb > c:
                assert eps_cs_violations(E, bad, price, eps=1) > 0


def test_certificate_implies_optimality_exhaustive():
    """Brute force on tiny S: every (r, p) pair with p from a small grid that
    passes the eps = 1 check is optimal (the scaling argument in
    tests/_certificate.py)."""
    import itertools
    rng = np.random.default_rng(7)
    S = 3
    for _ in range(30):
        E = rng.integers(0, 3, size=(S, S)).astype(np.int32)
        opt = oracle.brute_force(E)[0]
        for perm in itertools.permutations(range(S)):
            r = np.array(perm)
            for p in itertools.product(range(-4 * (S + 1), 4 * (S + 1) + 1, 2), repeat=S - 1):
                price = np.array((0,) + p)
                if eps_cs_violations(E, r, price) == 0:
                    assert sum(int(E[r[v], v]) for v in range(S)) == opt
