"""Pins for the oracle's Algorithm 2 replay, Algorithm 1
 and Eq. (2): hand-traced examples, the closed-form special
cases of DESIGN.md (identical / transposition), invariants (permutation,
strict decrease, 2-swap local optimality, >= optimum) and a second,
vectorised formulation."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_yangin17_b200 import synth


def test_cost_definition_hand():
    E = np.array([[3, 7, 2], [6, 1, 5], [2, 9, 6]], dtype=np.int32)
    # r = slot -> tile; Error = E[r0][0] + E[r1][1] + E[r2][2]
    assert oracle.cost(E, np.array([0, 1, 2])) == 3 + 1 + 6
    assert oracle.cost(E, np.array([2, 1, 0])) == 2 + 1 + 2
    assert oracle.cost(E, np.array([1, 2, 0])) == 6 + 9 + 2


def test_cost_int64_no_overflow():
    S = 8
    E = np.full((S, S), 2**31 - 1, dtype=np.int32)
    assert oracle.cost(E, np.arange(S)) == S * (2**31 - 1)


def test_alg2_hand_trace_n4():
    # S = 4: groups (0-indexed) P_1 = {(0,1),(2,3)}, P_2 = {(0,3),(1,2)}, P_3 = {(0,2),(1,3)}.
    # rows = input tiles, columns = target slots.
    E = np.array([[3, 7, 2, 8],
                  [6, 1, 5, 4],
                  [2, 9, 6, 3],
                  [7, 4, 1, 5]], dtype=np.int32)
    # Round 1, P_1: (0,1): 3+1=4 > 6+7=13? no.  (2,3): 6+5=11 > E[3][2]+E[2][3]=1+3=4: swap -> r=[0,1,3,2]
    #   P_2: (0,3): a=0,b=2: E[0][0]+E[2][3]=3+3=6 > E[2][0]+E[0][3]=2+8=10? no
    #        (1,2): a=1,b=3: E[1][1]+E[3][2]=1+1=2 > E[3][1]+E[1][2]=4+5=9? no
    #   P_3: (0,2): a=0,b=3: 3+1=4 > E[3][0]+E[0][2]=7+2=9? no
    #        (1,3): a=1,b=2: 1+3=4 > E[2][1]+E[1][3]=9+4=13? no
    # Round 2: same evaluations, no swap -> stop.  rounds = 2 (reading R10).
    assert oracle.edge_coloring(4).tolist() == [[[0, 1], [2, 3]], [[0, 3], [1, 2]], [[0, 2], [1, 3]]]
    r, rounds, swaps, per, st = oracle.local_search(E)
    assert r.tolist() == [0, 1, 3, 2]
    assert (rounds, swaps, per.tolist(), st) == (2, 1, [1, 0], 0)
    assert oracle.cost(E, r) == 3 + 1 + 1 + 3


def test_alg2_hand_trace_order_matters():
    # A swap in P_1 changes what P_2 sees (slot-indexed reading R5).
    # tiles 0..3; slot costs chosen so that after P_1 swaps (0,1), pair (0,3) in P_2 fires.
    E = np.array([[9, 0, 9, 9],
                  [5, 9, 9, 0],
                  [9, 9, 0, 9],
                  [0, 9, 9, 5]], dtype=np.int32)
    # r=[0,1,2,3], d=[9,9,0,5]
    # P_1 (0,1): 9+9=18 > E[1][0]+E[0][1]=5+0=5 -> swap, r=[1,0,2,3]
    #     (2,3): 0+5=5 > E[3][2]+E[2][3]=9+9=18? no
    # P_2 (0,3): a=1,b=3: E[1][0]+E[3][3]=5+5=10 > E[3][0]+E[1][3]=0+0=0 -> swap, r=[3,0,2,1]
    #     (1,2): a=0,b=2: E[0][1]+E[2][2]=0 > ... no
    # P_3 (0,2): a=3,b=2: 0+0 > ... no;  (1,3): a=0,b=1: 0+0 no.  Round 2: nothing.  cost 0.
    r, rounds, swaps, per, st = oracle.local_search(E)
    assert r.tolist() == [3, 0, 2, 1]
    assert (rounds, swaps, per.tolist()) == (2, 2, [2, 0])
    assert oracle.cost(E, r) == 0


def test_alg2_strict_gt_stops_on_ties_above_optimum():
    # Identity is 2-swap optimal only thanks to strict '>' ties (reading R6);
    # the optimum is a 3-cycle of cost 0, which no single swap reaches.
    E = np.full((4, 4), 10, dtype=np.int32)
    E[0, 0] = E[1, 1] = E[2, 2] = 5
    E[1, 0] = E[2, 1] = E[0, 2] = 0
    E[3, 3] = 0
    r, rounds, swaps, per, st = oracle.local_search(E)
    assert r.tolist() == [0, 1, 2, 3] and (rounds, swaps) == (1, 0)
    assert oracle.cost(E, r) == 15
    assert oracle.brute_force(E)[0] == 0
    assert oracle.hungarian(E)[1] == 0


def test_alg2_identical_images():
    I, T = synth.make_pair("identical", 64, 8, 3, seed=0)
    E = oracle.error_matrix(I, T, 8)
    r, rounds, swaps, per, st = oracle.local_search(E)
    assert (r == np.arange(64)).all() and (rounds, swaps) == (1, 0)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_alg2_transposition_closed_form(seed):
    # T = I with tiles p, q exchanged: by the L1 triangle inequality only the pair
    # (p, q) can fire, and after it every d = 0: exactly 1 swap, 2 rounds, cost 0.
    I, T = synth.make_pair("transposition", 128, 8, 3, seed=seed)
    E = oracle.error_matrix(I, T, 8)
    moved = np.nonzero(np.diag(E))[0]
    assert len(moved) == 2
    r, rounds, swaps, per, st = oracle.local_search(E)
    expect = np.arange(E.shape[0])
    expect[moved[0]], expect[moved[1]] = moved[1], moved[0]
    assert (r == expect).all() and (rounds, swaps, oracle.cost(E, r)) == (2, 1, 0)


def _two_opt_ok(E, r):
    F = E[r].astype(np.int64)          # F[u][v] = E[r[u]][v]: tile at slot u placed at v
    d = np.diag(F)
    return bool(((d[:, None] + d[None, :]) <= (F + F.T)).all())


@pytest.mark.parametrize("fam", ["smooth", "noise", "ties", "shuffle"])
def test_alg2_invariants(fam):
    I, T = synth.make_pair(fam, 128, 8, 3, seed=7)
    E = oracle.error_matrix(I, T, 8)
    r, rounds, swaps, per, st = oracle.local_search(E)
    assert st == 0
    assert sorted(r.tolist()) == list(range(E.shape[0])), "r stays a bijection (P:57)"
    assert _two_opt_ok(E, r), "no pair can improve on exit (Alg. 2 line 11)"
    assert per[-1] == 0 and (per[:-1] > 0).all() and per.sum() == swaps
    assert oracle.cost(E, r) <= oracle.cost(E, np.arange(E.shape[0]))
    assert oracle.cost(E, r) >= oracle.hungarian(E)[1]
    assert rounds <= 30


def test_alg2_each_round_strictly_decreases_cost():
    I, T = synth.make_pair("smooth", 128, 8, 3, seed=8)
    E = oracle.error_matrix(I, T, 8)
    r = np.arange(E.shape[0], dtype=np.int32)
    prev = oracle.cost(E, r)
    while True:
        r, rounds, swaps, per, st = oracle.local_search(E, r0=r, max_rounds=1)
        c = oracle.cost(E, r)
        if swaps == 0:
            assert c == prev
            break
        assert c < prev
        prev = c


def test_alg2_resume_is_exact():
    # a round depends only on (E, r): resuming from a round boundary is bit-identical
    I, T = synth.make_pair("noise", 128, 8, 3, seed=9)
    E = oracle.error_matrix(I, T, 8)
    full = oracle.local_search(E)
    part = oracle.local_search(E, max_rounds=2)
    assert part[4] == 3
    rest = oracle.local_search(E, r0=part[0])
    assert (rest[0] == full[0]).all()
    assert part[1] + rest[1] == full[1] and part[2] + rest[2] == full[2]


@pytest.mark.parametrize("fam,N,M", [("smooth", 128, 8), ("noise", 96, 8), ("ties", 64, 4), ("smooth", 90, 10)])
def test_alg2_two_formulations_agree(fam, N, M):
    I, T = synth.make_pair(fam, N, M, 3, seed=11)
    E = oracle.error_matrix(I, T, M)
    a = oracle.local_search(E)
    b = oracle.local_search_np(E)
    assert (a[0] == b[0]).all() and a[1:3] == b[1:3] and (a[3] == b[3]).all()


@pytest.mark.parametrize("S", [2, 3, 5, 6, 7, 8])
def test_alg2_vs_brute_force_small(S):
    rng = np.random.default_rng(S)
    for _ in range(40):
        E = rng.integers(0, 4, size=(S, S)).astype(np.int32)   # small range forces ties
        opt, _ = oracle.brute_force(E)
        r, rounds, swaps, per, st = oracle.local_search(E)
        assert st == 0 and sorted(r.tolist()) == list(range(S))
        assert oracle.cost(E, r) >= opt
        assert _two_opt_ok(E, r)
        assert oracle.hungarian(E)[1] == opt


def test_alg1_serial_invariants_and_difference():
    I, T = synth.make_pair("smooth", 128, 8, 3, seed=0)
    E = oracle.error_matrix(I, T, 8)
    r1, k1, s1, st1 = oracle.serial_local_search(E)
    r2 = oracle.local_search(E)[0]
    assert st1 == 0 and sorted(r1.tolist()) == list(range(256))
    assert _two_opt_ok(E, r1)
    # the serial and parallel orders differ, so do their results
    assert not (r1 == r2).all()


def test_alg1_hand_trace():
    # Algorithm 1 on the n=4 matrix of test_alg2_hand_trace_n4, lexicographic u<v:
    # (0,1) no; (0,2): a=0,b=2: 3+6=9 > E[2][0]+E[0][2]=2+2=4 -> swap r=[2,1,0,3]
    # (0,3): a=2,b=3: E[2][0]+E[3][3]=2+5=7 > E[3][0]+E[2][3]=7+3=10? no
    # (1,2): a=1,b=0: E[1][1]+E[0][2]=1+2=3 > E[0][1]+E[1][2]=7+5? no
    # (1,3): a=1,b=3: 1+5=6 > E[3][1]+E[1][3]=4+4=8? no
    # (2,3): a=0,b=3: E[0][2]+E[3][3]=2+5=7 > E[3][2]+E[0][3]=1+8=9? no.  Round 2: none.
    E = np.array([[3, 7, 2, 8], [6, 1, 5, 4], [2, 9, 6, 3], [7, 4, 1, 5]], dtype=np.int32)
    r, k, s, st = oracle.serial_local_search(E)
    assert r.tolist() == [2, 1, 0, 3] and (k, s) == (2, 1)


def test_render_identity_and_hand_example():
    # slot u of R shows input tile r[u]
    img = np.arange(16, dtype=np.uint8).reshape(4, 4)          # tiles [0,1,4,5] [2,3,6,7] [8,9,12,13] [10,11,14,15]
    assert (oracle.render(img, 2, np.arange(4)) == img).all()
    R = oracle.render(img, 2, np.array([3, 2, 1, 0]))
    assert R.tolist() == [[10, 11, 8, 9], [14, 15, 12, 13], [2, 3, 0, 1], [6, 7, 4, 5]]


def test_render_optimum_of_shuffle_reproduces_target():
    # T is a tile permutation of I, so the optimum (cost 0) renders T exactly
    I, T = synth.make_pair("shuffle", 96, 8, 3, seed=4)
    E = oracle.error_matrix(I, T, 8)
    r, c, p, q = oracle.hungarian(E)
    assert c == 0 and (oracle.render(I, 8, r) == T).all()


def test_render_cost_identity():
    # Eq. (2): the total error equals the pixelwise L1 distance of R and T
    I, T = synth.make_pair("smooth", 64, 8, 3, seed=5)
    E = oracle.error_matrix(I, T, 8)
    r = oracle.local_search(E)[0]
    R = oracle.render(I, 8, r)
    assert oracle.cost(E, r) == int(np.abs(R.astype(np.int64) - T.astype(np.int64)).sum())
