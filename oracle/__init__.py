"""CPU oracle for the photomosaic hot path (Yang, Ito & Nakano, IPDPS-W 2017).

TEST INFRASTRUCTURE.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference`` arm) may import
this package.  The product path (``paper_conf_ipps_yangin17_b200``) never
imports it and shares no code with it: the C part (``pm_oracle.c``) and this
file were written from the paper, not from the CUDA sources.

``P:<n>`` cites line n of the paper text; "reading Rk" cites the
numbered readings in DESIGN.md where the paper is silent or garbled.

Functions
---------
tiles(img, M)                       Step 1, P:57/P:77            (C loop)
error_matrix(I, T, M, rows=None)    Eq. (1); Step 2 P:79    (C loop nest)
error_entry(I, T, M, u, v)          one entry of Eq. (1)          (C loop nest)
error_matrix_np(I, T, M)            Eq. (1) as one numpy broadcast (second formulation)
num_colors(S), edge_coloring(S)     Theorem 1, groups P:152-203 (C)
local_search(E, r0=None)            Algorithm 2, P:207-223        (C, literal line 5)
local_search_np(E, r0=None)         Algorithm 2, vectorised per group (second formulation)
serial_local_search(E)              Algorithm 1, P:118-129        (C)
cost(E, r)                          Eq. (2), P:63                 (C)
hungarian(E)                        Sec. III, Kuhn-Munkres P:102  (C, with dual certificate)
render(I, M, r)                     the photomosaic image R, P:61/P:247 (C)
histogram_match(I, T)               I's distribution adjusted to T's, reading R12 (C)
brute_force(E)                      Eq. (3), all S! rearrangements (Python, S <= 8)

Pins (tests/test_oracle_*.py) tie each of these to something other than
itself: the printed K_16 groups, closed forms of Eq. (1), brute
force, the LP dual certificate, hand-worked examples and invariants.
"""
from __future__ import annotations

import ctypes
import itertools
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "pm_oracle.c")
_LIB_PATH = os.path.join(_HERE, "libpm_oracle.so")
_lib = None

_I32P = ctypes.POINTER(ctypes.c_int32)
_I64P = ctypes.POINTER(ctypes.c_int64)
_U8P = ctypes.POINTER(ctypes.c_uint8)


def build(force: bool = False) -> str:
    """Compile pm_oracle.c with gcc (-O2 -fopenmp).  Building the checker is
    not using it; ``__graft_entry__.build()`` calls this."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-std=c11", "-o", _LIB_PATH, _SRC]
        subprocess.check_call(cmd)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is not None:
        return _lib
    build()
    lib = ctypes.CDLL(_LIB_PATH)
    lib.or_tiles.argtypes = [_U8P, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, _U8P]
    lib.or_tiles.restype = None
    lib.or_error_entry.argtypes = [_U8P, _U8P, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
                                   ctypes.c_int64, ctypes.c_int64]
    lib.or_error_entry.restype = ctypes.c_int32
    lib.or_error_matrix.argtypes = [_U8P, _U8P, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
                                    ctypes.c_int64, ctypes.c_int64, _I32P]
    lib.or_error_matrix.restype = None
    lib.or_num_colors.argtypes = [ctypes.c_int32]
    lib.or_num_colors.restype = ctypes.c_int32
    lib.or_edge_coloring.argtypes = [ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, _I32P]
    lib.or_edge_coloring.restype = ctypes.c_int32
    lib.or_cost.argtypes = [_I32P, ctypes.c_int64, ctypes.c_int32, _I32P]
    lib.or_cost.restype = ctypes.c_int64
    lib.or_local_search.argtypes = [_I32P, ctypes.c_int64, ctypes.c_int32, _I32P, ctypes.c_int32,
                                    _I32P, _I64P, _I64P, ctypes.c_int32]
    lib.or_local_search.restype = ctypes.c_int32
    lib.or_serial_local_search.argtypes = [_I32P, ctypes.c_int64, ctypes.c_int32, _I32P,
                                           ctypes.c_int32, _I32P, _I64P]
    lib.or_serial_local_search.restype = ctypes.c_int32
    lib.or_hungarian.argtypes = [_I32P, ctypes.c_int64, ctypes.c_int32, _I32P, _I64P, _I64P, _I64P]
    lib.or_hungarian.restype = ctypes.c_int32
    lib.or_render.argtypes = [_U8P, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, _I32P, _U8P]
    lib.or_render.restype = None
    lib.or_histogram_match.argtypes = [_U8P, _U8P, ctypes.c_int32, ctypes.c_int32, _U8P]
    lib.or_histogram_match.restype = None
    lib.or_num_threads.argtypes = []
    lib.or_num_threads.restype = ctypes.c_int32
    lib.or_set_num_threads.argtypes = [ctypes.c_int32]
    lib.or_set_num_threads.restype = None
    _lib = lib
    return lib


def _p(a: np.ndarray, t):
    return a.ctypes.data_as(t)


def _img(img: np.ndarray) -> tuple[np.ndarray, int, int]:
    a = np.ascontiguousarray(img, dtype=np.uint8)
    if a.ndim == 2:
        a = a[:, :, None]
    assert a.ndim == 3 and a.shape[0] == a.shape[1], "N x N x C image expected (P:57)"
    return a, a.shape[0], a.shape[2]


def set_num_threads(t: int) -> None:
    _load().or_set_num_threads(int(t))


def num_threads() -> int:
    return int(_load().or_num_threads())


# ---------------------------------------------------------------- Step 1 ---
def tiles(img: np.ndarray, M: int) -> np.ndarray:
    """Step 1: u8 [S][M*M*C], tile u = raster grid cell."""
    a, N, C = _img(img)
    assert N % M == 0
    S = (N // M) ** 2
    out = np.empty((S, M * M * C), dtype=np.uint8)
    _load().or_tiles(_p(a, _U8P), N, M, C, _p(out, _U8P))
    return out


# ---------------------------------------------------------------- Eq. (1) --
def error_entry(I: np.ndarray, T: np.ndarray, M: int, u: int, v: int) -> int:
    """E(I_u, T_v), Eq. (1), one pixel at a time."""
    a, N, C = _img(I)
    b, N2, C2 = _img(T)
    assert (N, C) == (N2, C2) and N % M == 0
    return int(_load().or_error_entry(_p(a, _U8P), _p(b, _U8P), N, M, C, int(u), int(v)))


def error_matrix(I: np.ndarray, T: np.ndarray, M: int, rows: tuple[int, int] | None = None) -> np.ndarray:
    """Step 2: int32 E[u][v] = E(I_u, T_v) (w_{u,v}) for u in rows."""
    a, N, C = _img(I)
    b, N2, C2 = _img(T)
    assert (N, C) == (N2, C2) and N % M == 0
    S = (N // M) ** 2
    r0, r1 = (0, S) if rows is None else rows
    E = np.empty((r1 - r0, S), dtype=np.int32)
    _load().or_error_matrix(_p(a, _U8P), _p(b, _U8P), N, M, C, r0, r1, _p(E, _I32P))
    return E


def error_matrix_np(I: np.ndarray, T: np.ndarray, M: int) -> np.ndarray:
    """Eq. (1) as a numpy broadcast over (u, v, pixel): a second formulation
    written independently of the C loop nest (tile extraction by reshape)."""
    a, N, C = _img(I)
    b, _, _ = _img(T)
    g = N // M

    def cut(x):  # [g, M, g, M, C] -> [g*g, M*M*C], raster tile order
        return x.reshape(g, M, g, M, C).transpose(0, 2, 1, 3, 4).reshape(g * g, M * M * C).astype(np.int32)

    A, B = cut(a), cut(b)
    return np.abs(A[:, None, :] - B[None, :, :]).sum(axis=2).astype(np.int32)


# ---------------------------------------------------------------- Thm 1 ----
def num_colors(S: int) -> int:
    """Theorem 1: S-1 groups for even S, S for odd S."""
    return int(_load().or_num_colors(int(S)))


def edge_coloring(S: int) -> np.ndarray:
    """Edge groups P_1..P_m as int32 [m][S//2][2], 0-indexed,
    (u < v), pairs by increasing smaller index; odd S pads with (-1,-1)."""
    m = num_colors(S)
    out = np.empty((m, S // 2, 2), dtype=np.int32)
    if m:
        rc = _load().or_edge_coloring(int(S), 0, m, _p(out, _I32P))
        assert rc == 0
    return out


# ---------------------------------------------------------------- Eq. (2) --
def cost(E: np.ndarray, r: np.ndarray) -> int:
    """Error(R, T) = sum_u E(r(I_u), T_u), Eq. (2), int64."""
    E = np.ascontiguousarray(E, dtype=np.int32)
    r = np.ascontiguousarray(r, dtype=np.int32)
    S = E.shape[0]
    return int(_load().or_cost(_p(E, _I32P), E.shape[1], S, _p(r, _I32P)))


# ---------------------------------------------------------------- Alg. 2 ---
def local_search(E: np.ndarray, r0: np.ndarray | None = None, max_rounds: int = 0):
    """Algorithm 2, serial replay of the colour-group rounds.

    Returns (r, rounds, swaps, swaps_per_round, status); status 0 = converged,
    3 = max_rounds reached first."""
    E = np.ascontiguousarray(E, dtype=np.int32)
    S = E.shape[0]
    r = np.arange(S, dtype=np.int32) if r0 is None else np.array(r0, dtype=np.int32, copy=True)
    rounds = ctypes.c_int32(0)
    swaps = ctypes.c_int64(0)
    cap = max_rounds if max_rounds > 0 else 4096
    per = np.zeros(cap, dtype=np.int64)
    st = _load().or_local_search(_p(E, _I32P), E.shape[1], S, _p(r, _I32P), int(max_rounds),
                                 ctypes.byref(rounds), ctypes.byref(swaps), _p(per, _I64P), cap)
    return r, int(rounds.value), int(swaps.value), per[: min(rounds.value, cap)].copy(), int(st)


def local_search_np(E: np.ndarray, r0: np.ndarray | None = None, max_rounds: int = 0):
    """Algorithm 2 again, vectorised: all pairs of one group P_i evaluated at
    once (they are disjoint), groups in order.  Second formulation for
    cross-checking the C replay; uses the C colouring (pinned separately)."""
    E = np.asarray(E, dtype=np.int64)
    S = E.shape[0]
    r = np.arange(S, dtype=np.int64) if r0 is None else np.array(r0, dtype=np.int64)
    groups = edge_coloring(S)
    rounds = 0
    total = 0
    per = []
    while True:
        if max_rounds and rounds >= max_rounds:
            return r.astype(np.int32), rounds, total, np.array(per, dtype=np.int64), 3
        sw = 0
        for g in groups:
            g = g[g[:, 0] >= 0]
            u, v = g[:, 0], g[:, 1]
            a, b = r[u], r[v]
            fire = E[a, u] + E[b, v] > E[b, u] + E[a, v]
            r[u[fire]], r[v[fire]] = b[fire], a[fire]
            sw += int(fire.sum())
        rounds += 1
        total += sw
        per.append(sw)
        if sw == 0:
            return r.astype(np.int32), rounds, total, np.array(per, dtype=np.int64), 0


def serial_local_search(E: np.ndarray, r0: np.ndarray | None = None, max_rounds: int = 0):
    """Algorithm 1.  Returns (r, rounds, swaps, status)."""
    E = np.ascontiguousarray(E, dtype=np.int32)
    S = E.shape[0]
    r = np.arange(S, dtype=np.int32) if r0 is None else np.array(r0, dtype=np.int32, copy=True)
    rounds = ctypes.c_int32(0)
    swaps = ctypes.c_int64(0)
    st = _load().or_serial_local_search(_p(E, _I32P), E.shape[1], S, _p(r, _I32P), int(max_rounds),
                                        ctypes.byref(rounds), ctypes.byref(swaps))
    return r, int(rounds.value), int(swaps.value), int(st)


# ---------------------------------------------------------------- render ---
def render(I: np.ndarray, M: int, r: np.ndarray) -> np.ndarray:
    """The photomosaic R: slot u shows input tile r[u]."""
    a, N, C = _img(I)
    r = np.ascontiguousarray(r, dtype=np.int32)
    out = np.empty_like(a)
    _load().or_render(_p(a, _U8P), N, M, C, _p(r, _I32P), _p(out, _U8P))
    return out if np.asarray(I).ndim == 3 else out[:, :, 0]


# ---------------------------------------------------------------- P:84 -----
def histogram_match(I: np.ndarray, T: np.ndarray) -> np.ndarray:
    """I's intensity distribution adjusted to T's (Sec. II; reading
    R12): per channel, level k -> the smallest level z with C_T(z) >= C_I(k)
    (cumulative pixel counts).  Returns a new u8 image shaped like I."""
    a, N, C = _img(I)
    b, N2, C2 = _img(T)
    assert (N, C) == (N2, C2)
    out = np.empty_like(a)
    _load().or_histogram_match(_p(a, _U8P), _p(b, _U8P), N, C, _p(out, _U8P))
    return out if np.asarray(I).ndim == 3 else out[:, :, 0]


# ---------------------------------------------------------------- Sec. III -
def hungarian(E: np.ndarray):
    """Minimum-weight perfect matching by Kuhn-Munkres.

    Returns (r, cost, p, q): r[v] = input tile at slot v; p, q the LP dual."""
    E = np.ascontiguousarray(E, dtype=np.int32)
    S = E.shape[0]
    r = np.empty(S, dtype=np.int32)
    c = ctypes.c_int64(0)
    p = np.empty(S, dtype=np.int64)
    q = np.empty(S, dtype=np.int64)
    st = _load().or_hungarian(_p(E, _I32P), E.shape[1], S, _p(r, _I32P), ctypes.byref(c),
                              _p(p, _I64P), _p(q, _I64P))
    assert st == 0
    return r, int(c.value), p, q


def brute_force(E: np.ndarray):
    """Eq. (3): evaluate Error(R, T) for all S! rearrangements.
    Pure Python, S <= 8.  Returns (min cost, one argmin r)."""
    E = np.asarray(E, dtype=np.int64)
    S = E.shape[0]
    assert S <= 8, "brute force is for tiny S only"
    best, arg = None, None
    for perm in itertools.permutations(range(S)):
        c = sum(int(E[perm[u], u]) for u in range(S))
        if best is None or c < best:
            best, arg = c, perm
    return best, np.array(arg, dtype=np.int32)
