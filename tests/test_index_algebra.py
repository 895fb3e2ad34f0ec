"""CPU pins of index algebra used by the CUDA path (no GPU): written from the
paper's groups (Theorem 1; class c pairs slots u0 + k and u0 - k
mod m, u0 = c + (m+1)/2, pair 0 = (u0, S-1)) and the definition of the
sigma-permuted copy Ep[t][q] = E[t][2q mod m], q < m + 48 -- not from the
kernels' code.

* The first sparse scan's pair-space tiles (k_sparse.cu scan_full_ep): for
  pairs k0 .. k0+255 over classes c0 .. c0+31, row t+kk of side A holds slot
  baseA + t + kk and row t+255-kk of side B slot baseB + t + 255 - kk, with
  baseA = u0(c0) + k0 and baseB = u0(c0) - k0 - 255 (mod m): these must be
  the two slots of pair k0+kk in class c0+t.  The partner's sigma-position
  c + (m+1)/2 - sigma(y) must index E[r[y]][partner] in Ep.
* The E kernel's fused copy (k_sad.cu epilogue): column v < m goes to
  q = v/2 (even v) or v/2 + S/2 (odd v), and also to q + m when q < 48; the
  two runs of a 64-column tile are contiguous.  (For m < 48 the extension
  wraps more than once: q + m, q + 2m, ...)
"""
import numpy as np
import pytest


def _classes(S):
    m = S - 1 if S % 2 == 0 else S
    return m, (m + 1) // 2


def _sigma(y, m):
    return (y * ((m + 1) // 2)) % m


@pytest.mark.parametrize("S", [8, 16, 256, 1024, 4096, 300])
def test_scan_tile_rows_are_the_pairs_slots(S):
    m, H = _classes(S)
    KR = (m - 1) // 2
    P, B = 256, 32
    rng = np.random.default_rng(S)
    for _ in range(20):
        k0 = 1 + int(rng.integers(0, max(KR, 1))) // P * P
        c0 = int(rng.integers(0, m)) // B * B
        baseA = (c0 + H + k0) % m
        baseB = (c0 + H - k0 - (P - 1)) % m
        for t in range(B):
            c = c0 + t
            if c >= m:
                continue
            u0 = (c + H) % m
            for kk in range(0, P, 7):
                k = k0 + kk
                if k > KR:
                    break
                first, second = (u0 + k) % m, (u0 - k) % m
                assert (baseA + t + kk) % m == first
                assert (baseB + t + (P - 1) - kk) % m == second
                # the pair is a pair of class c: sum == 2c+1 (mod m)
                assert (first + second) % m == (2 * c + 1) % m
                # the streamed sigma-position of each slot's partner in class c
                for y, p in ((first, second), (second, first)):
                    q = (c + H - _sigma(y, m)) % m
                    assert (2 * q) % m == p


@pytest.mark.parametrize("S", [16, 64, 256, 1024, 16384])
def test_sigma_copy_placement(S):
    m = S - 1
    rng = np.random.default_rng(1)
    row = rng.integers(0, 1 << 20, size=S)
    ref = row[(2 * np.arange(m + 48)) % m]             # the definition
    got = np.full(m + 48, -1, dtype=np.int64)
    for v in range(m):                                 # the epilogue's placement
        q = v // 2 if v % 2 == 0 else v // 2 + S // 2
        assert q == ((v + m) // 2 if v % 2 else v // 2)
        got[q] = row[v]
        qq = q + m                                     # the cyclic extension (wraps again when m < 48)
        while qq < m + 48:
            got[qq] = row[v]
            qq += m
    assert (got == ref).all()
    # a 64-column tile's even and odd columns land in two contiguous runs
    for col0 in range(0, m - 64, 64):
        ev = [(col0 + 2 * i) // 2 for i in range(32)]
        od = [(col0 + 2 * i + 1) // 2 + S // 2 for i in range(32)]
        assert ev == list(range(col0 // 2, col0 // 2 + 32))
        assert od == list(range(col0 // 2 + S // 2, col0 // 2 + S // 2 + 32))
