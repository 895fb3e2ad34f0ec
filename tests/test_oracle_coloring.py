"""Pins for the oracle's edge colouring: Theorem 1 and the printed
edge groups P_1..P_16 of K_16 (tests/golden/k16_groups.txt)."""
import os

import numpy as np
import pytest

import oracle


def _read_golden(path):
    groups = {}
    for line in open(path):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        i, rest = line.split(":")
        groups[int(i)] = [tuple(int(x) - 1 for x in p.split(",")) for p in rest.split()]
    return groups


def test_k16_matches_printed_table(golden_dir):
    gold = _read_golden(os.path.join(golden_dir, "k16_groups.txt"))
    assert sorted(gold) == list(range(1, 17))
    assert gold[16] == []                      # P_16 = empty
    got = oracle.edge_coloring(16)
    assert got.shape == (15, 8, 2)
    for i in range(1, 16):
        assert [tuple(map(int, p)) for p in got[i - 1]] == gold[i], f"P_{i}"


@pytest.mark.parametrize("n", list(range(1, 65)))
def test_theorem1_counts_and_cover(n):
    m = oracle.num_colors(n)
    assert m == (0 if n < 2 else (n - 1 if n % 2 == 0 else n))
    g = oracle.edge_coloring(n)
    seen = set()
    for cls in g:
        verts = []
        for u, v in cls:
            if u < 0:
                continue
            assert 0 <= u < v < n
            seen.add((int(u), int(v)))
            verts += [int(u), int(v)]
        assert len(verts) == len(set(verts)), "a group is a matching (no shared tile, P:137)"
        if n % 2 == 0:
            assert len(verts) == n, "even n: every group is a perfect matching"
        else:
            assert len(verts) == n - 1
    if n >= 2:
        assert len(seen) == n * (n - 1) // 2, "every pair appears in exactly one group"
        assert sum(int((c[:, 0] >= 0).sum()) for c in g) == n * (n - 1) // 2


def test_groups_are_fixed_by_S_only():
    # groups depend only on S
    assert (oracle.edge_coloring(38) == oracle.edge_coloring(38)).all()
