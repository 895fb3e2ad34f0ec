"""GPU exact assignment: the paper's optimization
algorithm (Sec. III), min-weight perfect matching of input tiles to
target slots with w_{u,v} = E(I_u, T_v), solved by
pm_optimal_assignment (eps-scaling auction, reading R16).

Pins, each independent of the CUDA path: the optimum cost of the oracle's
Kuhn-Munkres solver (itself pinned to brute force, LP duality and scipy in
test_oracle_hungarian.py), brute force over all S! rearrangements for S <= 8,
closed forms (a tile shuffle has optimum 0; identical images too), and the
eps-CS certificate of tests/_certificate.py, which proves optimality on its
own and is checked at sizes the oracle cannot reach in seconds."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402
from tests._certificate import eps_cs_violations, is_permutation  # noqa: E402

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

DEV = torch.device("cuda:0")


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).to(DEV)


def _solve_and_certify(E_np):
    perm, c, rounds, price = pm.optimal_assignment(dev(E_np))
    r = perm.cpu().numpy()
    p = price.cpu().numpy()
    S = E_np.shape[0]
    assert is_permutation(r)
    assert c == int(E_np.astype(np.int64)[r, np.arange(S)].sum())
    assert eps_cs_violations(E_np, r, p) == 0
    return r, c, rounds


@pytest.mark.parametrize("S", [1, 2, 3, 4, 5, 6, 7, 8])
def test_assignment_vs_brute_force(S):
    rng = np.random.default_rng(500 + S)
    for hi in (1, 2, 4, 1000, 195841):
        E = rng.integers(0, hi, size=(S, S)).astype(np.int32)
        _, c, _ = _solve_and_certify(E)
        assert c == oracle.brute_force(E)[0]


@pytest.mark.parametrize("S", [9, 31, 64, 100, 257])
def test_assignment_random_matrices_vs_hungarian(S):
    rng = np.random.default_rng(900 + S)
    for hi in (3, 50, 195841):
        E = rng.integers(0, hi, size=(S, S)).astype(np.int32)
        _, c, _ = _solve_and_certify(E)
        assert c == oracle.hungarian(E)[1]


@pytest.mark.parametrize("fam", ["smooth", "noise", "ties", "transposition"])
@pytest.mark.parametrize("N,M,C", [(128, 8, 3), (90, 10, 3), (200, 5, 1)])
def test_assignment_images_vs_hungarian(fam, N, M, C):
    I, T = synth.make_pair(fam, N, M, C, seed=11)
    E = oracle.error_matrix(I, T, M)
    _, c, _ = _solve_and_certify(E)
    assert c == oracle.hungarian(E)[1]


@pytest.mark.parametrize("fam", ["smooth", "noise"])
def test_assignment_config2_vs_hungarian(fam):
    """BASELINE config 2 (S = 1024), the bench workload."""
    I, T = synth.config_pair(2, fam, seed=0)
    E = oracle.error_matrix(I, T, 16)
    r, c, _ = _solve_and_certify(E)
    assert c == oracle.hungarian(E)[1]
    # the optimum is never worse than Algorithm 2's local optimum
    perm, *_ = pm.local_search(dev(E))
    assert c <= oracle.cost(E, perm.cpu().numpy())


def test_assignment_shuffle_and_identical_are_zero():
    for fam in ("shuffle", "identical"):
        I, T = synth.make_pair(fam, 256, 16, 3, seed=4)
        E = oracle.error_matrix(I, T, 16)
        _, c, _ = _solve_and_certify(E)
        assert c == 0


def test_assignment_config3_certificate():
    """S = 4096 (BASELINE config 3 and the paper's Table III size): the
    certificate alone proves optimality; E comes from the GPU kernel that
    test_gpu_parity.py holds bit-exact to the oracle."""
    I, T = synth.config_pair(3, "smooth", seed=0)
    Ed = pm.error_matrix(dev(I), dev(T), 16)
    _solve_and_certify(Ed.cpu().numpy())


def test_assignment_padded_ld():
    rng = np.random.default_rng(3)
    S = 77
    big = rng.integers(0, 1000, size=(S, S + 13)).astype(np.int32)
    E = big[:, :S].copy()
    Ed = dev(big)[:, :S]
    perm, c, _, price = pm.optimal_assignment(Ed)
    assert c == oracle.hungarian(E)[1]
    assert eps_cs_violations(E, perm.cpu().numpy(), price.cpu().numpy()) == 0


def test_assignment_rejects_out_of_range_weights():
    E = np.zeros((16, 16), dtype=np.int32)
    E[3, 5] = -1
    with pytest.raises(pm.PMError) as ei:
        pm.optimal_assignment(dev(E))
    assert ei.value.status == pm.PM_ERR_INVALID
    E[3, 5] = 1 << 24
    with pytest.raises(pm.PMError):
        pm.optimal_assignment(dev(E))


@pytest.mark.parametrize("gs", ["0", "1", "256"])
@pytest.mark.parametrize("knobs", [("8", "3"), ("2", "0"), ("64", "20")])
@pytest.mark.parametrize("keep,smem", [("0", "1"), ("1", "0")])
def test_assignment_schedule_knobs_stay_exact(gs, knobs, keep, smem):
    """Exactness does not depend on the eps schedule, on where the
    Gauss-Seidel tail takes over, on keeping eps-CS pairs across phases or on
    where the tail keeps its prices (any eps0 >= 1, any divisor, final eps = 1)."""
    with pm.tuning(auction_gs=int(gs), auction_keep=int(keep), auction_smem_price=int(smem),
                   auction_theta=int(knobs[0]), auction_eps_shift=int(knobs[1])):
        _schedule_case()


def _schedule_case():
    rng = np.random.default_rng(77)
    for S in (5, 64, 130):
        E = rng.integers(0, 2000, size=(S, S)).astype(np.int32)
        _, c, _ = _solve_and_certify(E)
        assert c == oracle.hungarian(E)[1]
    I, T = synth.make_pair("smooth", 128, 8, 3, seed=5)
    E = oracle.error_matrix(I, T, 8)
    _, c, _ = _solve_and_certify(E)
    assert c == oracle.hungarian(E)[1]
