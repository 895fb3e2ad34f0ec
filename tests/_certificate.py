"""Optimality certificate of an assignment (test infrastructure).

For integer weights E (S x S, rows = input tiles u, columns = target slots v)
and costs C = (S + 1) * E, an assignment r (r[v] = input tile at slot v) with
prices p satisfying eps-complementary slackness with eps = 1,

    C[r[v]][v] + p[v] <= min_w ( C[r[v]][w] + p[w] ) + 1     for every v,

has sum_v C[r[v]][v] <= OPT_C + S (sum the inequalities against an optimal
bijection; the prices cancel), and since every C-cost is a multiple of S + 1,
sum_v E[r[v]][v] = OPT: r solves Eq. (3) / the matching of P:94.
This check shares nothing with the CUDA path or the oracle."""
import numpy as np


def eps_cs_violations(E, r, price, eps: int = 1) -> int:
    E = np.asarray(E, dtype=np.int64)
    S = E.shape[0]
    r = np.asarray(r, dtype=np.int64)
    p = np.asarray(price, dtype=np.int64)
    C = E * (S + 1)
    reduced = C + p[None, :]                       # [u][w]
    best = reduced.min(axis=1)                     # per input tile u
    lhs = reduced[r, np.arange(S)]                 # slot v held by u = r[v]
    return int((lhs > best[r] + eps).sum())


def is_permutation(r) -> bool:
    r = np.asarray(r)
    return sorted(r.tolist()) == list(range(len(r)))
