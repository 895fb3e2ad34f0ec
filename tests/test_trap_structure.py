"""Structure of the edge groups that PM_LS_TRAP (k_trap.cu) relies on, checked
on the oracle's colouring (itself pinned to the paper's printed K_16 groups,
P:154-203, and Theorem 1).  No GPU needed.

TRAP numbers the pairs of class c by k: pair 0 = (u0, S-1) with
u0 = (c + (m+1)/2) mod m, pair k >= 1 = (u0 + k, u0 - k) mod m ("first" and
"second" slot).  It relies on three facts, each tested here for many S:
  1. every group has exactly that form (offsets k and m - k from u0);
  2. the stencil: pair k of class c+1 holds the first slot of pair k+1 and
     the second slot of pair k-1 of class c, with the reflections pair K
     (first <- its own second), pair 1 (second <- first of pair 0) and pair 0
     (second = S-1) -- also across the round boundary (class m-1 -> 0);
  3. the partner of a slot y advances by 2 (mod m) from one class to the next
     while neither it nor y meets S-1, and a slot's pair index changes by at
     most one per class (the light cone of the overlapped tiling)."""
import numpy as np
import pytest

import oracle

EVEN_S = [4, 6, 16, 20, 64, 100, 256, 1024]


def _pairs_by_k(S, c, group):
    m = S - 1
    K = S // 2 - 1
    u0 = (c + (m + 1) // 2) % m
    first = np.full(K + 1, -1)
    second = np.full(K + 1, -1)
    for u, v in group:
        u, v = int(u), int(v)
        if S - 1 in (u, v):
            x = v if u == S - 1 else u
            assert x == u0, "S-1 is paired with the fixed point u0"
            first[0], second[0] = u0, S - 1
            continue
        ou, ov = (u - u0) % m, (v - u0) % m
        assert ou + ov == m, "a pair is mirror-symmetric about u0"
        k = min(ou, ov)
        assert 1 <= k <= K
        first[k] = u if ou == k else v
        second[k] = v if ou == k else u
    assert (first >= 0).all() and (second >= 0).all(), "every pair index occurs once"
    return first, second


@pytest.mark.parametrize("S", EVEN_S)
def test_groups_have_the_pair_index_form(S):
    groups = oracle.edge_coloring(S)
    for c in range(S - 1):
        _pairs_by_k(S, c, groups[c])


@pytest.mark.parametrize("S", EVEN_S)
def test_three_point_stencil_between_consecutive_classes(S):
    groups = oracle.edge_coloring(S)
    m, K = S - 1, S // 2 - 1
    fs = [_pairs_by_k(S, c, groups[c]) for c in range(m)]
    for c in range(m):
        f0, s0 = fs[c]
        f1, s1 = fs[(c + 1) % m]          # class m-1 -> class 0 of the next round
        for k in range(K + 1):
            want_first = s0[K] if k == K else f0[k + 1]
            if k == 0:
                want_second = S - 1
            elif k == 1:
                want_second = f0[0]
            else:
                want_second = s0[k - 1]
            assert f1[k] == want_first, (S, c, k)
            assert s1[k] == want_second, (S, c, k)


@pytest.mark.parametrize("S", EVEN_S)
def test_partner_advances_by_two_and_pair_index_moves_by_at_most_one(S):
    groups = oracle.edge_coloring(S)
    m, K = S - 1, S // 2 - 1
    partner = np.zeros((m, S), dtype=np.int64)
    index = np.zeros((m, S), dtype=np.int64)
    for c in range(m):
        f, s = _pairs_by_k(S, c, groups[c])
        for k in range(K + 1):
            partner[c, f[k]], partner[c, s[k]] = s[k], f[k]
            index[c, f[k]] = index[c, s[k]] = k
    for c in range(m):
        c1 = (c + 1) % m
        for y in range(m):
            p0, p1 = partner[c, y], partner[c1, y]
            if S - 1 not in (p0, p1):
                assert p1 == (p0 + 2) % m, (S, c, y)
            assert abs(index[c1, y] - index[c, y]) <= 1, (S, c, y)
        assert index[c1, S - 1] == 0
