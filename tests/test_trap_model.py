"""A plain-Python model of PM_LS_TRAP's decomposition (k_trap.cu), replayed on
the CPU and compared with the oracle's Alg. 2 replay (oracle.local_search).
No GPU needed: it checks the *design* -- chunks of W owned pairs, phases of
T classes replayed on the extended range [k0-T, k1+T) with the valid range
shrinking by one pair per side and class, publication of the owned pairs'
slots only, E read only through the staged per-tile runs (two stride-2 runs
p0 + 2j and s0 + 2j, j <= T, E[t][S-1], and E[t][u0 .. u0+2T+1] for the
pair-0 light cone) -- and counts any E read that would fall outside the
staged entries (there must be none: the coverage argument behind the
kernel's pointer scheme).

Independent of the CUDA code (written from the paper's groups and DESIGN.md
§6.3); slots of class c: pair 0 = (u0, S-1), pair k = (u0+k, u0-k) mod m."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_yangin17_b200 import synth


def _trap_model(E, W, T):
    S = E.shape[0]
    m, K, H = S - 1, S // 2 - 1, S // 2
    r = np.arange(S)
    d = E[r, np.arange(S)].astype(np.int64)
    nch = -(-(K + 1) // W)
    rounds, swaps, misses, per = 0, 0, 0, []
    while True:
        rsw = 0
        for c0 in range(0, m, T):
            Tp = min(T, m - c0)
            u0 = (c0 + H) % m
            r_new, d_new = r.copy(), d.copy()
            for ch in range(nch):
                k0, k1 = ch * W, min(ch * W + W, K + 1)
                a, b = max(k0 - Tp, 0), min(k1 + Tp, K + 1)
                low = a == 0
                # local copy of the extended range's slots (state + staged runs)
                slots = [(u0 + k) % m for k in range(a, b)] + [(u0 - k) % m for k in range(max(a, 1), b)]
                if low:
                    slots.append(S - 1)
                tile = {x: int(r[x]) for x in slots}
                dd = {x: int(d[x]) for x in slots}
                staged = {}
                cone = set()
                if low:
                    cone = {(u0 + k) % m for k in range(0, Tp + 1)} | {(u0 - k) % m for k in range(1, Tp + 1)} | {S - 1}
                for x in slots:
                    g = tile[x]
                    fx = x == S - 1
                    p0 = u0 if fx else (2 * c0 + 1 - x) % m
                    s0 = u0 if fx else x
                    cols = {(p0 + 2 * j) % m for j in range(T + 1)} | {(s0 + 2 * j) % m for j in range(T + 1)} | {S - 1}
                    if x in cone:
                        cols |= {(u0 + z) % m for z in range(2 * T + 2)}
                    staged[g] = cols

                def e(g, col):
                    nonlocal misses
                    if col not in staged[g]:
                        misses += 1
                    return int(E[g, col])

                for t in range(Tp):
                    lo = 0 if low else a + t
                    hi = K + 1 if b == K + 1 else b - t
                    u = (u0 + t) % m
                    for k in range(lo, hi):
                        x1 = (u + k) % m
                        x2 = S - 1 if k == 0 else (u - k) % m
                        ta, tb = tile[x1], tile[x2]
                        e_bu, e_av = e(tb, x1), e(ta, x2)
                        if dd[x1] + dd[x2] > e_bu + e_av:
                            tile[x1], tile[x2] = tb, ta
                            dd[x1], dd[x2] = e_bu, e_av
                            if k0 <= k < k1:
                                rsw += 1
                # publish the owned pairs' slots (class c0 + Tp - 1)
                u = (u0 + Tp - 1) % m
                for k in range(k0, k1):
                    for x in ((u + k) % m, S - 1 if k == 0 else (u - k) % m):
                        r_new[x], d_new[x] = tile[x], dd[x]
            r, d = r_new, d_new
        rounds += 1
        swaps += rsw
        per.append(rsw)
        if rsw == 0:
            return r, rounds, swaps, np.array(per), misses


@pytest.mark.parametrize("N,M,fam,W,T", [(64, 8, "smooth", 5, 4), (64, 8, "noise", 9, 8), (96, 8, "smooth", 6, 5),
                                         (128, 8, "ties", 17, 16), (128, 8, "transposition", 3, 2),
                                         (64, 8, "noise", 2, 6)])   # W < T: global buffers (grid mode) only
def test_trap_model_matches_alg2_replay(N, M, fam, W, T):
    I, Tg = synth.make_pair(fam, N, M, 3, seed=3)
    E = oracle.error_matrix(I, Tg, M)
    ref = oracle.local_search(E)
    r, rounds, swaps, per, misses = _trap_model(E, W, T)
    assert misses == 0, "an E read outside the staged runs"
    assert (r == ref[0]).all()
    assert (rounds, swaps) == (ref[1], ref[2])
    assert (per == ref[3][: len(per)]).all()
