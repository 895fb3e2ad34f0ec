"""Pins of oracle.histogram_match (Sec. II: the input image's intensity
distribution is adjusted to the target's before Step 1; reading R12 in
DESIGN.md: histogram specification on cumulative pixel counts, per channel,
level k -> min{z : C_T(z) >= C_I(k)}).  Each pin is fixed by the definition
or by an independent formulation, not by re-typing the oracle's loops."""
import numpy as np
import pytest

import oracle
from paper_conf_ipps_yangin17_b200 import synth


def _sorted_rank_formulation(I, T):
    # independent formulation: the level of the C_I(k)-th smallest target
    # pixel (1-based) is min{z : C_T(z) >= C_I(k)}, for every input level k
    I3 = I if I.ndim == 3 else I[:, :, None]
    T3 = T if T.ndim == 3 else T[:, :, None]
    out = np.empty_like(I3)
    for c in range(I3.shape[2]):
        a = I3[:, :, c].ravel()
        t = np.sort(T3[:, :, c].ravel())
        cum = np.cumsum(np.bincount(a, minlength=256))
        lut = np.array([t[cum[k] - 1] if cum[k] > 0 else t[0] for k in range(256)], dtype=np.uint8)
        out[:, :, c] = lut[I3[:, :, c]]
    return out if I.ndim == 3 else out[:, :, 0]


def test_hand_example():
    # 2x2 grayscale: I levels {0,0,1,2} (C_I = 2,3,4 at 0,1,2); T levels
    # {10,20,20,30} (C_T = 1,3,4 at 10,20,30): 0 -> min{z: C_T >= 2} = 20,
    # 1 -> min{z: C_T >= 3} = 20, 2 -> min{z: C_T >= 4} = 30
    I = np.array([[0, 0], [1, 2]], np.uint8)
    T = np.array([[10, 20], [20, 30]], np.uint8)
    assert oracle.histogram_match(I, T).tolist() == [[20, 20], [20, 30]]


@pytest.mark.parametrize("fam", ["smooth", "noise", "ties"])
@pytest.mark.parametrize("N,C", [(16, 1), (64, 3), (128, 3), (90, 3)])
def test_matches_sorted_rank_formulation(fam, N, C):
    I, T = synth.make_pair(fam, N, max(N // 8, 1) if N % 8 == 0 else 10, C, seed=N + C)
    assert (oracle.histogram_match(I, T) == _sorted_rank_formulation(I, T)).all()


def test_identical_images_unchanged():
    I, _ = synth.make_pair("smooth", 128, 8, 3, seed=1)
    assert (oracle.histogram_match(I, I) == I).all()


def test_same_histogram_is_identity():
    # I a pixel shuffle of T: equal histograms, so every present level maps to itself
    _, T = synth.make_pair("smooth", 64, 8, 3, seed=2)
    rng = np.random.default_rng(3)
    flat = T.reshape(-1, 3)
    I = flat[rng.permutation(flat.shape[0])].reshape(T.shape)
    assert (oracle.histogram_match(I, T) == I).all()


def test_constant_target():
    I, _ = synth.make_pair("noise", 32, 8, 3, seed=4)
    T = np.full_like(I, 77)
    assert (oracle.histogram_match(I, T) == 77).all()


def test_distinct_levels_reproduce_target_histogram_exactly():
    # 16x16 = 256 pixels per channel, each input level once: C_I takes every
    # value 1..256, so the output's histogram equals the target's exactly
    rng = np.random.default_rng(5)
    I = np.stack([rng.permutation(256).reshape(16, 16) for _ in range(3)], axis=2).astype(np.uint8)
    _, T = synth.make_pair("smooth", 16, 4, 3, seed=6)
    out = oracle.histogram_match(I, T)
    for c in range(3):
        assert (np.bincount(out[:, :, c].ravel(), minlength=256) ==
                np.bincount(T[:, :, c].ravel(), minlength=256)).all()


@pytest.mark.parametrize("seed", [7, 8, 9])
def test_monotone_map_and_cumulative_bound(seed):
    # the map is non-decreasing in the input level (an order-preserving
    # re-levelling), and C_out(z) <= C_T(z) at every level (C_out(z) is the
    # largest C_I(k) not exceeding C_T(z))
    I, T = synth.make_pair("smooth", 64, 8, 3, seed=seed)
    out = oracle.histogram_match(I, T)
    for c in range(3):
        a, o = I[:, :, c].ravel(), out[:, :, c].ravel()
        order = np.argsort(a, kind="stable")
        assert (np.diff(o[order].astype(int)) >= 0).all()
        c_out = np.cumsum(np.bincount(o, minlength=256))
        c_t = np.cumsum(np.bincount(T[:, :, c].ravel(), minlength=256))
        c_i = np.cumsum(np.bincount(a, minlength=256))
        assert (c_out <= c_t).all()
        for z in range(256):
            assert c_out[z] == max([0] + [v for v in c_i if v <= c_t[z]])
