"""Pins for the oracle's Step 1 (tiling) and Eq. (1).

Each test ties the C loop nest to something other than itself: hand-computed
values, closed forms of the L1 sum, symmetry, and the tile-permutation
structure.  No expected value here comes from the CUDA path."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_yangin17_b200 import synth


def test_tiles_hand_example():
    # 4x4 grayscale image 0..15, M = 2: g = 2, raster tile order (reading R4).
    img = np.arange(16, dtype=np.uint8).reshape(4, 4)
    t = oracle.tiles(img, 2)
    assert t.tolist() == [[0, 1, 4, 5], [2, 3, 6, 7], [8, 9, 12, 13], [10, 11, 14, 15]]


def test_tiles_rgb_order():
    # (y, x, c) byte order inside a tile; 2x2 RGB image, M = 1 -> 4 tiles of 3 bytes
    img = np.arange(12, dtype=np.uint8).reshape(2, 2, 3)
    assert oracle.tiles(img, 1).tolist() == [[0, 1, 2], [3, 4, 5], [6, 7, 8], [9, 10, 11]]


def test_error_hand_example():
    # N = 2, M = 1, grayscale: tiles are single pixels, E[u][v] = |I_u - T_v|.
    I = np.array([[1, 5], [9, 0]], dtype=np.uint8)
    T = np.array([[4, 4], [0, 200]], dtype=np.uint8)
    E = oracle.error_matrix(I, T, 1)
    assert E.tolist() == [[3, 3, 1, 199],
                          [1, 1, 5, 195],
                          [5, 5, 9, 191],
                          [4, 4, 0, 200]]


def test_error_hand_rgb_tile():
    # one 2x2 RGB tile each (N = M = 2): sum over 12 channel values, by hand
    I = np.zeros((2, 2, 3), dtype=np.uint8)
    T = np.zeros((2, 2, 3), dtype=np.uint8)
    I[0, 0] = (10, 20, 30)   # |10-0|+|20-0|+|30-0| = 60
    T[1, 1] = (0, 255, 7)    # 0 + 255 + 7 = 262
    I[1, 1] = (1, 255, 9)    # |1-0|+|255-255|+|9-7| = 3 (overrides the T term)
    assert oracle.error_matrix(I, T, 2).tolist() == [[60 + 3]]


@pytest.mark.parametrize("a,b", [(0, 0), (7, 200), (255, 0), (0, 255), (128, 127)])
def test_error_constant_images(a, b):
    # closed form: constant images give E == P * |a - b|, P = M*M*C
    N, M, C = 16, 4, 3
    I = np.full((N, N, C), a, dtype=np.uint8)
    T = np.full((N, N, C), b, dtype=np.uint8)
    E = oracle.error_matrix(I, T, M)
    assert E.shape == (16, 16)
    assert (E == M * M * C * abs(a - b)).all()


def test_error_black_white_is_max():
    N, M, C = 32, 16, 3
    I = np.zeros((N, N, C), dtype=np.uint8)
    T = np.full((N, N, C), 255, dtype=np.uint8)
    assert (oracle.error_matrix(I, T, M) == 255 * M * M * C).all()   # 195840, reading R11


def test_error_identical_images_symmetric_zero_diag():
    I, _ = synth.make_pair("noise", 32, 4, 3, seed=1)
    E = oracle.error_matrix(I, I, 4)
    assert (np.diag(E) == 0).all()
    assert (E == E.T).all()
    assert (E[~np.eye(E.shape[0], dtype=bool)] > 0).all()


def test_error_single_pixel_change():
    # changing one target pixel by delta changes exactly column v0, each entry by <= |delta|
    N, M, C = 24, 4, 3
    I, T = synth.make_pair("noise", N, M, C, seed=2)
    E0 = oracle.error_matrix(I, T, M)
    T2 = T.copy()
    y, x, c = 9, 13, 1
    T2[y, x, c] = 255 - T2[y, x, c]
    delta = abs(int(T2[y, x, c]) - int(T[y, x, c]))
    E1 = oracle.error_matrix(I, T2, M)
    v0 = (y // M) * (N // M) + (x // M)
    diff = E1 - E0
    assert (np.delete(diff, v0, axis=1) == 0).all()
    assert (np.abs(diff[:, v0]) <= delta).all()
    assert np.abs(diff[:, v0]).max() > 0


def test_error_tile_permutation_structure():
    # T = seeded tile shuffle of I: for each slot v there is an input tile with zero error
    I, T = synth.make_pair("shuffle", 32, 8, 3, seed=3)
    E = oracle.error_matrix(I, T, 8)
    assert ((E == 0).sum(axis=0) >= 1).all()


def test_error_matches_numpy_broadcast():
    # second, independently written formulation (reshape + broadcast)
    for fam, N, M, C in [("smooth", 48, 8, 3), ("noise", 30, 5, 1), ("ties", 24, 6, 3)]:
        I, T = synth.make_pair(fam, N, M, C, seed=4)
        assert (oracle.error_matrix(I, T, M) == oracle.error_matrix_np(I, T, M)).all()


def test_error_rows_and_entry_consistent():
    I, T = synth.make_pair("smooth", 64, 8, 3, seed=5)
    E = oracle.error_matrix(I, T, 8)
    part = oracle.error_matrix(I, T, 8, rows=(13, 40))
    assert (part == E[13:40]).all()
    for u, v in [(0, 0), (63, 0), (5, 62), (63, 63)]:
        assert oracle.error_entry(I, T, 8, u, v) == E[u, v]


def test_error_triangle_inequality():
    # L1 is a metric (reading R1): E(I_a, T_b) <= E(I_a, I_c) + E(I_c, T_b)
    I, T = synth.make_pair("smooth", 32, 8, 3, seed=6)
    EIT = oracle.error_matrix(I, T, 8).astype(np.int64)
    EII = oracle.error_matrix(I, I, 8).astype(np.int64)
    lhs = EIT[:, None, :]
    rhs = EII[:, :, None] + EIT[None, :, :]
    assert (lhs <= rhs).all()
