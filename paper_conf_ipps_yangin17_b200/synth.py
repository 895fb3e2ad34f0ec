"""Seeded synthetic input images -- the ONE module shared by the CUDA path's
tests/bench and the oracle's tests.  It holds none of the method's
arithmetic: it only draws u8 images (no tiling of the method, no errors).

The paper's workloads are 8-bit natural photographs from USC-SIPI
(Lena, Sailboat, Airplane, ...), 512^2-2048^2, with the
input histogram-matched to the target.  Those images are not
available, so:

F1 smooth   natural-image-like: per channel, 6 plane-wave cosines
            (frequency U(0.5, 6) cycles/image per axis, amplitude U(0.3, 1),
            phase U(0, 2 pi)) + 8 Gaussian blobs (centre U(0,1)^2,
            sigma U(0.03, 0.2)*N, amplitude U(-2, 2)); min-max to [0, 255];
            + N(0, 6^2) noise; rint; clip; u8.  input seed 2s+1, target 2s+2.
F2 noise    uniform u8.
F3 ties     values in {0, 1, 2} (many equal E entries, Delta = 0 swaps).
F4 identical  T = I.
F5 transposition  T = I with two tiles p, q exchanged.
F6 shuffle  T = a seeded permutation of I's tiles (optimum error 0).

Images are u8 [N][N][C] row-major HWC (C = 3, RGB; reading R2).
"""
from __future__ import annotations

import numpy as np

# BASELINE.json configs: (N, M) with C = 3.  n = (N/M)^2 tiles.
CONFIGS = {
    1: dict(N=128, M=8, C=3),     # 16x16 grid, n = 256
    2: dict(N=512, M=16, C=3),    # 32x32 grid, n = 1024 (Fig. 2 shape)
    3: dict(N=1024, M=16, C=3),   # 64x64 grid, n = 4096
    4: dict(N=2048, M=16, C=3),   # 128x128 grid, n = 16384
    5: dict(N=4096, M=16, C=3),   # 256x256 grid, n = 65536
}

FAMILIES = ("smooth", "noise", "ties", "identical", "transposition", "shuffle")


def _smooth_channel(rng: np.random.Generator, N: int) -> np.ndarray:
    x = (np.arange(N, dtype=np.float64) + 0.5) / N
    img = np.zeros((N, N), dtype=np.float64)
    for _ in range(6):
        fx, fy = rng.uniform(0.5, 6.0, size=2)
        amp = rng.uniform(0.3, 1.0)
        ph = rng.uniform(0.0, 2.0 * np.pi)
        # cos(2pi(fx x + fy y) + ph) = cos(X)cos(Y) - sin(X)sin(Y), X = 2pi fx x + ph
        X = 2.0 * np.pi * fx * x + ph
        Y = 2.0 * np.pi * fy * x
        img += amp * (np.outer(np.cos(Y), np.cos(X)) - np.outer(np.sin(Y), np.sin(X)))
    for _ in range(8):
        cx, cy = rng.uniform(0.0, 1.0, size=2)
        sig = rng.uniform(0.03, 0.2)
        amp = rng.uniform(-2.0, 2.0)
        gx = np.exp(-((x - cx) ** 2) / (2.0 * sig * sig))
        gy = np.exp(-((x - cy) ** 2) / (2.0 * sig * sig))
        img += amp * np.outer(gy, gx)
    lo, hi = img.min(), img.max()
    img = (img - lo) * (255.0 / max(hi - lo, 1e-12))
    img += rng.normal(0.0, 6.0, size=(N, N))
    return np.clip(np.rint(img), 0, 255).astype(np.uint8)


def smooth_image(N: int, C: int, seed: int) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return np.stack([_smooth_channel(rng, N) for _ in range(C)], axis=2)


def _tile_view(img: np.ndarray, M: int) -> np.ndarray:
    """[g, g, M, M, C] view of the raster tile grid (input construction only)."""
    N, _, C = img.shape
    g = N // M
    return img.reshape(g, M, g, M, C).transpose(0, 2, 1, 3, 4)


def make_pair(family: str, N: int, M: int, C: int = 3, seed: int = 0):
    """Return (I, T): u8 [N][N][C] input and target images."""
    if N % M != 0:
        raise ValueError("M must divide N (P:57)")
    if family == "smooth":
        return smooth_image(N, C, 2 * seed + 1), smooth_image(N, C, 2 * seed + 2)
    if family == "noise":
        rng = np.random.default_rng(1000 + seed)
        return (rng.integers(0, 256, size=(N, N, C), dtype=np.uint8),
                rng.integers(0, 256, size=(N, N, C), dtype=np.uint8))
    if family == "ties":
        rng = np.random.default_rng(2000 + seed)
        return (rng.integers(0, 3, size=(N, N, C), dtype=np.uint8),
                rng.integers(0, 3, size=(N, N, C), dtype=np.uint8))
    I = smooth_image(N, C, 2 * seed + 1)
    g = N // M
    S = g * g
    if family == "identical":
        return I, I.copy()
    if family == "transposition":
        rng = np.random.default_rng(3000 + seed)
        p, q = rng.choice(S, size=2, replace=False)
        T = I.copy()
        tv = _tile_view(T, M)
        a = tv[p // g, p % g].copy()
        tv[p // g, p % g] = tv[q // g, q % g]
        tv[q // g, q % g] = a
        return I, T
    if family == "shuffle":
        rng = np.random.default_rng(4000 + seed)
        perm = rng.permutation(S)
        src = _tile_view(I, M).reshape(S, M, M, C)          # copy, raster order
        T = src[perm].reshape(g, g, M, M, C).transpose(0, 2, 1, 3, 4).reshape(N, N, C)
        return I, np.ascontiguousarray(T)
    raise ValueError(f"unknown family {family!r}; one of {FAMILIES}")


def config_pair(cfg: int, family: str = "smooth", seed: int = 0):
    c = CONFIGS[cfg]
    return make_pair(family, c["N"], c["M"], c["C"], seed)
