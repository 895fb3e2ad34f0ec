"""Thin ctypes binding of libpm.so (include/pm.h) -- argument marshalling only.

Every step of the hot path runs in the library's CUDA kernels; this module
never computes anything itself and has no CPU fallback: if ``libpm.so`` is
missing it raises, and every compute call requires CUDA tensors.

Names follow the C-ABI: ``error_matrix`` = ``pm_error_matrix`` (Eq. 1),
``local_search`` = ``pm_local_search_ex`` (Algorithm 2), ``cost`` =
``pm_cost`` (Eq. 2), ``edge_coloring`` = ``pm_edge_coloring``
(Theorem 1), ``photomosaic`` = the Sec. V pipeline.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libpm.so")

(PM_OK, PM_ERR_INVALID, PM_ERR_CUDA, PM_ERR_NOT_CONVERGED, PM_ERR_UNSUPPORTED, PM_ERR_NOT_PERMUTATION,
 PM_ERR_TIMEOUT) = range(7)
METHODS = {"auto": 0, "class": 1, "window": 3, "walk": 5, "trap": 6}

_lib = None
_P = ctypes.c_void_p
_I32, _I64 = ctypes.c_int32, ctypes.c_int64

# (name, restype, argtypes) for every function declared in include/pm.h
_SIGS = [
    ("pm_status_string", ctypes.c_char_p, [ctypes.c_int]),
    ("pm_tile_stride", _I64, [_I32, _I32]),
    ("pm_pack_tiles", ctypes.c_int, [_P, _I32, _I32, _I32, _P, _I64, _P]),
    ("pm_error_matrix", ctypes.c_int, [_P, _P, _I32, _I32, _I32, _I32, _I32, _P, _I64, _P]),
    ("pm_error_matrix_tiles", ctypes.c_int, [_P, _P, _I64, _I32, _I32, _I32, _I32, _P, _I64, _P]),
    ("pm_num_colors", _I32, [_I32]),
    ("pm_edge_coloring", ctypes.c_int, [_I32, _I32, _I32, _P]),
    ("pm_local_search", ctypes.c_int, [_P, _I64, _I32, _P, _I32, _P, _P, _P]),
    ("pm_local_search_ex", ctypes.c_int, [_P, _I64, _I32, _P, _I32, _I32, _P, _P, _P, _I32, _P]),
    ("pm_local_search_async", ctypes.c_int, [_P, _I64, _I32, _P, _I32, _I32, _P, _P]),
    ("pm_sigma_copy_bytes", ctypes.c_size_t, [_I32]),
    ("pm_local_search_ep_async", ctypes.c_int, [_P, _I64, _I32, _P, _I32, _I32, _P, ctypes.c_size_t, _P, _P]),
    ("pm_error_matrix_sigma", ctypes.c_int, [_P, _P, _I32, _I32, _I32, _P, _I64, _P, ctypes.c_size_t, _P]),
    ("pm_local_search_sigma_async", ctypes.c_int, [_P, _I64, _I32, _P, _I32, _I32, _P, ctypes.c_size_t, _P, _P]),
    ("pm_ls_auto_method", _I32, [_I32]),
    ("pm_init_identity", ctypes.c_int, [_P, _I32, _P]),
    ("pm_cost", ctypes.c_int, [_P, _I64, _I32, _P, _P, _P]),
    ("pm_cost_async", ctypes.c_int, [_P, _I64, _I32, _P, _P, _P]),
    ("pm_photomosaic", ctypes.c_int, [_P, _P, _I32, _I32, _I32, _P, _I64, _P, _I32, _P, _P, _P, _P]),
    ("pm_photomosaic_async", ctypes.c_int, [_P, _P, _I32, _I32, _I32, _P, _I64, _P, _I32, _P, _P]),
    ("pm_photomosaic_host", ctypes.c_int, [_P, _P, _I32, _I32, _I32, _I32, _P, _P, _P, _P, _P]),
    ("pm_render", ctypes.c_int, [_P, _I32, _I32, _I32, _P, _P, _P]),
    ("pm_optimal_assignment", ctypes.c_int, [_P, _I64, _I32, _P, _P, _P, _P, _P]),
    ("pm_histogram_match", ctypes.c_int, [_P, _P, _I32, _I32, _P, _P]),
    ("pm_launch_count", _I64, []),
    ("pm_trap_workspace_bytes", ctypes.c_size_t, [_I32]),
    ("pm_trap_workspace_reset", ctypes.c_int, [_P, _I32, _P]),
    ("pm_local_search_multi_async", ctypes.c_int, [_P, _I64, _I32, _P, _P, _I32, _I32, _I32, _P, _P]),
    ("pm_local_search_multi_emulated", ctypes.c_int, [_P, _I64, _I32, _P, _I32, _I32, _P, _P, _P]),
    ("pm_trap_workspace_bytes_sharded", ctypes.c_size_t, [_I32, _I32]),
    ("pm_local_search_sharded_async", ctypes.c_int, [_P, _P, _I64, _I32, _P, _P, _I32, _I32, _I32, _P, _P]),
    ("pm_cost_sharded_async", ctypes.c_int, [_P, _P, _I32, _I64, _I32, _P, _P, _P]),
    ("pm_local_search_sharded_emulated", ctypes.c_int, [_P, _I64, _I32, _P, _I32, _I32, _P, _P, _P]),
    ("pm_tuning_set", ctypes.c_int, [ctypes.c_char_p, _I32]),
    ("pm_tuning_reset", None, []),
    ("pm_scratch_trim", ctypes.c_int, []),
    ("pm_scratch_reserved_bytes", ctypes.c_size_t, []),
]


class PMError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        super().__init__(f"{where}: {status_string(status)}")


def lib():
    """Load libpm.so (raises if it has not been built: there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} not found: run `python -c 'import __graft_entry__ as g; g.build()'` "
                               "or `make` (the CUDA path has no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        for name, res, args in _SIGS:
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def status_string(s: int) -> str:
    return lib().pm_status_string(int(s)).decode()


def _check(status: int, where: str, ok=(PM_OK,)):
    if status not in ok:
        raise PMError(status, where)
    return status


def _torch():
    import torch
    return torch


def _stream(stream=None):
    torch = _torch()
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream)


def _dev_u8_image(x):
    torch = _torch()
    if not (isinstance(x, torch.Tensor) and x.is_cuda and x.dtype == torch.uint8):
        raise TypeError("expected a CUDA uint8 tensor [N][N][C] (or [N][N])")
    if x.dim() == 2:
        x = x.unsqueeze(-1)
    if x.dim() != 3 or x.shape[0] != x.shape[1]:
        raise ValueError("expected an N x N x C image (P:57)")
    return x.contiguous()


def _dev(x, dtype):
    torch = _torch()
    if not (isinstance(x, torch.Tensor) and x.is_cuda and x.dtype == dtype):
        raise TypeError(f"expected a CUDA {dtype} tensor")
    return x


# ----------------------------------------------------------------- Step 1 --
def tile_stride(M: int, C: int) -> int:
    return int(lib().pm_tile_stride(M, C))


def pack_tiles(img, M: int, stream=None):
    """pm_pack_tiles: u8 [S][tile_stride] tiles."""
    torch = _torch()
    img = _dev_u8_image(img)
    N, C = img.shape[0], img.shape[2]
    S = (N // M) ** 2 if M > 0 and N % M == 0 else 0
    ld = tile_stride(M, C)
    out = torch.empty((max(S, 1), max(ld, 16)), dtype=torch.uint8, device=img.device)
    _check(lib().pm_pack_tiles(img.data_ptr(), N, M, C, out.data_ptr(), ld, _stream(stream)), "pm_pack_tiles")
    return out[:, : M * M * C]


# ----------------------------------------------------------------- Step 2 --
def error_matrix(I, T, M: int, rows: tuple[int, int] | None = None, out=None, stream=None):
    """pm_error_matrix: int32 E[u - row_begin][v] = E(I_u, T_v), Eq. (1)."""
    torch = _torch()
    I = _dev_u8_image(I)
    T = _dev_u8_image(T)
    N, C = I.shape[0], I.shape[2]
    if T.shape != I.shape:
        raise ValueError("input and target must have the same shape (P:57)")
    S = (N // M) ** 2 if M > 0 and N % M == 0 else 0
    r0, r1 = (0, S) if rows is None else rows
    if out is None:
        out = torch.empty((max(r1 - r0, 0), S), dtype=torch.int32, device=I.device)
    else:
        _dev(out, torch.int32)
    ld = out.stride(0) if out.dim() == 2 and out.shape[0] > 0 else S
    _check(lib().pm_error_matrix(I.data_ptr(), T.data_ptr(), N, M, C, r0, r1, out.data_ptr(), ld,
                                 _stream(stream)), "pm_error_matrix")
    return out


def error_matrix_tiles(It, Tt, P: int, rows: tuple[int, int] | None = None, out=None, stream=None):
    """pm_error_matrix_tiles on packed tiles from pack_tiles (use their base)."""
    torch = _torch()
    S = Tt.shape[0]
    r0, r1 = (0, S) if rows is None else rows
    if out is None:
        out = torch.empty((r1 - r0, S), dtype=torch.int32, device=Tt.device)
    _check(lib().pm_error_matrix_tiles(It.data_ptr(), Tt.data_ptr(), It.stride(0), S, P, r0, r1, out.data_ptr(),
                                       out.stride(0), _stream(stream)), "pm_error_matrix_tiles")
    return out


# ---------------------------------------------------------------- Thm. 1 ---
def num_colors(S: int) -> int:
    return int(lib().pm_num_colors(S))


def edge_coloring(S: int, class_begin: int = 0, class_end: int | None = None) -> np.ndarray:
    """pm_edge_coloring (host): int32 [classes][S//2][2] edge groups."""
    m = num_colors(S)
    class_end = m if class_end is None else class_end
    out = np.zeros((max(class_end - class_begin, 0), S // 2, 2), dtype=np.int32)
    _check(lib().pm_edge_coloring(S, class_begin, class_end, out.ctypes.data), "pm_edge_coloring")
    return out


# ---------------------------------------------------------------- Alg. 2 ---
def local_search(E, perm=None, max_rounds: int = 0, method: str = "auto", stream=None, log_len: int = 256,
                 allow_not_converged: bool = False):
    """pm_local_search_ex: returns (perm, rounds, swaps, swaps_per_round, status).

    perm (int32 CUDA [S]) is updated in place; None starts from identity."""
    torch = _torch()
    _dev(E, torch.int32)
    S = E.shape[0]
    if perm is None:
        perm = torch.arange(S, dtype=torch.int32, device=E.device)
    _dev(perm, torch.int32)
    rounds = ctypes.c_int32(0)
    swaps = ctypes.c_int64(0)
    per = np.zeros(log_len, dtype=np.int64)
    ok = (PM_OK, PM_ERR_NOT_CONVERGED) if allow_not_converged else (PM_OK,)
    st = _check(lib().pm_local_search_ex(E.data_ptr(), E.stride(0), S, perm.data_ptr(), max_rounds,
                                         METHODS[method], ctypes.byref(rounds), ctypes.byref(swaps),
                                         per.ctypes.data, log_len, _stream(stream)), "pm_local_search_ex", ok)
    n = min(rounds.value, log_len)
    return perm, int(rounds.value), int(swaps.value), per[:n].copy(), st


def local_search_async(E, perm, result, max_rounds: int = 0, method: str = "auto", stream=None):
    """pm_local_search_async: no host sync; result = CUDA int64 [3] {status, rounds, swaps}."""
    _check(lib().pm_local_search_async(E.data_ptr(), E.stride(0), E.shape[0], perm.data_ptr(), max_rounds,
                                       METHODS[method], result.data_ptr(), _stream(stream)),
           "pm_local_search_async")


def sigma_copy_bytes(S: int) -> int:
    """pm_sigma_copy_bytes: size of the caller-owned sigma-permuted copy for S."""
    return int(lib().pm_sigma_copy_bytes(S))


def local_search_ep_async(E, perm, result, Ep, max_rounds: int = 0, method: str = "auto", stream=None):
    """pm_local_search_ep_async: as local_search_async, with TRAP's sigma-permuted
    copy of E built into the caller's buffer Ep (CUDA, >= sigma_copy_bytes(S) bytes)."""
    _check(lib().pm_local_search_ep_async(E.data_ptr(), E.stride(0), E.shape[0], perm.data_ptr(), max_rounds,
                                          METHODS[method], Ep.data_ptr(), Ep.numel() * Ep.element_size(),
                                          result.data_ptr(), _stream(stream)),
           "pm_local_search_ep_async")


def error_matrix_sigma(I, T, M: int, E, Ep, stream=None):
    """pm_error_matrix_sigma: E (all rows) and its sigma-permuted copy Ep in one pass."""
    torch = _torch()
    I = _dev_u8_image(I)
    T = _dev_u8_image(T)
    _dev(E, torch.int32)
    _check(lib().pm_error_matrix_sigma(I.data_ptr(), T.data_ptr(), I.shape[0], M, I.shape[2], E.data_ptr(),
                                       E.stride(0), Ep.data_ptr(), Ep.numel() * Ep.element_size(), _stream(stream)),
           "pm_error_matrix_sigma")
    return E


def local_search_sigma_async(E, perm, result, Ep, max_rounds: int = 0, method: str = "auto", stream=None):
    """pm_local_search_sigma_async: as local_search_async on a prebuilt sigma-permuted copy Ep."""
    _check(lib().pm_local_search_sigma_async(E.data_ptr(), E.stride(0), E.shape[0], perm.data_ptr(), max_rounds,
                                             METHODS[method], Ep.data_ptr(), Ep.numel() * Ep.element_size(),
                                             result.data_ptr(), _stream(stream)),
           "pm_local_search_sigma_async")


def local_search_multi_emulated(E, world: int, perm=None, max_rounds: int = 0, stream=None):
    """pm_local_search_multi_emulated (test hook): the multi-GPU TRAP protocol
    with `world` ranks in one launch on this device.  Returns (perm, rounds, swaps)."""
    torch = _torch()
    _dev(E, torch.int32)
    S = E.shape[0]
    if perm is None:
        perm = torch.arange(S, dtype=torch.int32, device=E.device)
    rounds, swaps = ctypes.c_int32(0), ctypes.c_int64(0)
    _check(lib().pm_local_search_multi_emulated(E.data_ptr(), E.stride(0), S, perm.data_ptr(), world, max_rounds,
                                                ctypes.byref(rounds), ctypes.byref(swaps), _stream(stream)),
           "pm_local_search_multi_emulated", (PM_OK, PM_ERR_NOT_CONVERGED))
    return perm, int(rounds.value), int(swaps.value)


def trap_workspace_bytes(S: int) -> int:
    return int(lib().pm_trap_workspace_bytes(S))


def trap_workspace_reset(ws, S: int, stream=None):
    """pm_trap_workspace_reset on a CUDA byte tensor (async on the stream)."""
    _check(lib().pm_trap_workspace_reset(ws.data_ptr(), S, _stream(stream)), "pm_trap_workspace_reset")


def local_search_multi_async(E, perm_ptrs, ws_ptrs, rank: int, world: int, result, max_rounds: int = 0,
                             stream=None):
    """pm_local_search_multi_async: this rank's part of the multi-GPU search;
    perm_ptrs / ws_ptrs = every rank's perm / workspace device pointers as
    mapped into this process (ints)."""
    P = ctypes.c_void_p * world
    _check(lib().pm_local_search_multi_async(E.data_ptr(), E.stride(0), E.shape[0], P(*perm_ptrs), P(*ws_ptrs),
                                             rank, world, max_rounds, result.data_ptr(), _stream(stream)),
           "pm_local_search_multi_async")


def local_search_sharded_emulated(E, world: int, perm=None, max_rounds: int = 0, stream=None):
    """pm_local_search_sharded_emulated (test hook): the row-sharded multi-GPU
    search with `world` ranks (E split into `world` shard buffers) in one
    launch on this device.  Returns (perm, rounds, swaps)."""
    torch = _torch()
    _dev(E, torch.int32)
    S = E.shape[0]
    if perm is None:
        perm = torch.arange(S, dtype=torch.int32, device=E.device)
    rounds, swaps = ctypes.c_int32(0), ctypes.c_int64(0)
    _check(lib().pm_local_search_sharded_emulated(E.data_ptr(), E.stride(0), S, perm.data_ptr(), world, max_rounds,
                                                  ctypes.byref(rounds), ctypes.byref(swaps), _stream(stream)),
           "pm_local_search_sharded_emulated", (PM_OK, PM_ERR_NOT_CONVERGED))
    return perm, int(rounds.value), int(swaps.value)


def trap_workspace_bytes_sharded(S: int, rows: int) -> int:
    return int(lib().pm_trap_workspace_bytes_sharded(S, rows))


def local_search_sharded_async(E_ptrs, row_begin, ld_E: int, S: int, perm_ptrs, ws_ptrs, rank: int, world: int,
                               result, max_rounds: int = 0, stream=None):
    """pm_local_search_sharded_async: this rank's part of the search over
    row-sharded E; E_ptrs / perm_ptrs / ws_ptrs = every rank's shard / perm /
    workspace device pointers as mapped into this process (ints), row_begin
    the world+1 shard bounds."""
    P = ctypes.c_void_p * world
    RB = ctypes.c_int32 * (world + 1)
    _check(lib().pm_local_search_sharded_async(P(*E_ptrs), RB(*row_begin), ld_E, S, P(*perm_ptrs), P(*ws_ptrs),
                                               rank, world, max_rounds, result.data_ptr(), _stream(stream)),
           "pm_local_search_sharded_async")


def ls_auto_method(S: int) -> str:
    """Name of the method PM_LS_AUTO picks for S on the current device."""
    code = int(lib().pm_ls_auto_method(S))
    return {v: k for k, v in METHODS.items()}[code]


def init_identity(perm, stream=None):
    """pm_init_identity: r := identity (reading R7)."""
    _check(lib().pm_init_identity(perm.data_ptr(), perm.shape[0], _stream(stream)), "pm_init_identity")


# ---------------------------------------------------------------- Eq. (2) --
def cost(E, perm, stream=None) -> int:
    c = ctypes.c_int64(0)
    _check(lib().pm_cost(E.data_ptr(), E.stride(0), E.shape[0], perm.data_ptr(), ctypes.byref(c),
                         _stream(stream)), "pm_cost")
    return int(c.value)


def cost_async(E, perm, out, stream=None):
    _check(lib().pm_cost_async(E.data_ptr(), E.stride(0), E.shape[0], perm.data_ptr(), out.data_ptr(),
                               _stream(stream)), "pm_cost_async")


# ------------------------------------------------------- whole pipeline ----
def cost_sharded_async(E_ptrs, row_begin, ld_E: int, S: int, perm, out, stream=None):
    """pm_cost_sharded_async: Eq. (2) over row-sharded E (peer pointers)."""
    world = len(E_ptrs)
    P = ctypes.c_void_p * world
    RB = ctypes.c_int32 * (world + 1)
    _check(lib().pm_cost_sharded_async(P(*E_ptrs), RB(*row_begin), world, ld_E, S, perm.data_ptr(), out.data_ptr(),
                                       _stream(stream)), "pm_cost_sharded_async")


def photomosaic(I, T, M: int, method: str = "auto", E=None, perm=None, stream=None):
    """pm_photomosaic on device images: returns (perm, rounds, swaps, cost, E)."""
    torch = _torch()
    I = _dev_u8_image(I)
    T = _dev_u8_image(T)
    N, C = I.shape[0], I.shape[2]
    S = (N // M) ** 2
    if E is None:
        E = torch.empty((S, S), dtype=torch.int32, device=I.device)
    if perm is None:
        perm = torch.empty(S, dtype=torch.int32, device=I.device)
    rounds, swaps, c = ctypes.c_int32(0), ctypes.c_int64(0), ctypes.c_int64(0)
    _check(lib().pm_photomosaic(I.data_ptr(), T.data_ptr(), N, M, C, E.data_ptr(), E.stride(0), perm.data_ptr(),
                                METHODS[method], ctypes.byref(rounds), ctypes.byref(swaps), ctypes.byref(c),
                                _stream(stream)), "pm_photomosaic")
    return perm, int(rounds.value), int(swaps.value), int(c.value), E


def photomosaic_async(I, T, M: int, E, perm, result, method: str = "auto", stream=None):
    """pm_photomosaic_async: no host sync; result = CUDA int64 [4] {status, rounds, swaps, cost}."""
    I = _dev_u8_image(I)
    T = _dev_u8_image(T)
    N, C = I.shape[0], I.shape[2]
    _check(lib().pm_photomosaic_async(I.data_ptr(), T.data_ptr(), N, M, C, E.data_ptr(), E.stride(0),
                                      perm.data_ptr(), METHODS[method], result.data_ptr(), _stream(stream)),
           "pm_photomosaic_async")


def photomosaic_host(I: np.ndarray, T: np.ndarray, M: int, method: str = "auto", perm_out: np.ndarray | None = None,
                     stream=None):
    """pm_photomosaic_host: host u8 images in, host r out (end-to-end call).
    Returns (perm, rounds, swaps, cost).  Pass pinned-memory numpy views for
    full-bandwidth copies."""
    if I.ndim == 2:
        I = I[:, :, None]
        T = T[:, :, None]
    assert I.dtype == np.uint8 and T.dtype == np.uint8 and I.shape == T.shape
    assert I.flags.c_contiguous and T.flags.c_contiguous
    N, C = I.shape[0], I.shape[2]
    S = (N // M) ** 2
    if perm_out is None:
        perm_out = np.empty(S, dtype=np.int32)
    rounds, swaps, c = ctypes.c_int32(0), ctypes.c_int64(0), ctypes.c_int64(0)
    _check(lib().pm_photomosaic_host(I.ctypes.data, T.ctypes.data, N, M, C, METHODS[method], perm_out.ctypes.data,
                                     ctypes.byref(rounds), ctypes.byref(swaps), ctypes.byref(c), _stream(stream)),
           "pm_photomosaic_host")
    return perm_out, int(rounds.value), int(swaps.value), int(c.value)


def render(I, M: int, perm, out=None, stream=None):
    """pm_render: the photomosaic image R, slot u showing input tile perm[u]."""
    torch = _torch()
    img = _dev_u8_image(I)
    N, C = img.shape[0], img.shape[2]
    if out is None:
        out = torch.empty_like(img)
    _check(lib().pm_render(img.data_ptr(), N, M, C, perm.data_ptr(), out.data_ptr(), _stream(stream)), "pm_render")
    return out if I.dim() == 3 else out[:, :, 0]


# ------------------------------------------------ histogram ---------
def histogram_match(I, T, out=None, stream=None):
    """pm_histogram_match: I's intensity distribution adjusted to T's (Sec. II,
    P:84; reading R12).  Returns the adjusted image (out, or a new tensor;
    out may be I for in-place)."""
    torch = _torch()
    img = _dev_u8_image(I)
    tgt = _dev_u8_image(T)
    if tgt.shape != img.shape:
        raise ValueError("input and target must have the same shape (P:57)")
    N, C = img.shape[0], img.shape[2]
    if out is None:
        out = torch.empty_like(img)
    elif out.dim() == 2:
        out = out.unsqueeze(-1)
    _check(lib().pm_histogram_match(img.data_ptr(), tgt.data_ptr(), N, C, out.data_ptr(), _stream(stream)),
           "pm_histogram_match")
    return out if I.dim() == 3 else out[:, :, 0]


# ------------------------------------------------- optimum (Sec. III) ------
def optimal_assignment(E, perm=None, price=None, stream=None):
    """pm_optimal_assignment: the best rearrangement R* (Eq. 3) by an exact GPU
    auction.  Returns (perm, cost, rounds, price); price (int64 CUDA [S]) is the
    eps-CS certificate for the costs (S + 1) * E."""
    torch = _torch()
    _dev(E, torch.int32)
    S = E.shape[0]
    if perm is None:
        perm = torch.empty(S, dtype=torch.int32, device=E.device)
    if price is None:
        price = torch.empty(S, dtype=torch.int64, device=E.device)
    rounds, c = ctypes.c_int32(0), ctypes.c_int64(0)
    _check(lib().pm_optimal_assignment(E.data_ptr(), E.stride(0), S, perm.data_ptr(), price.data_ptr(),
                                       ctypes.byref(rounds), ctypes.byref(c), _stream(stream)),
           "pm_optimal_assignment")
    return perm, int(c.value), int(rounds.value), price


def launch_count() -> int:
    return int(lib().pm_launch_count())


# ------------------------------------------------ tuning / scratch (pm.h) ---
def tuning_set(name: str, value: int):
    """pm_tuning_set: override one measured default (tests / dev tools)."""
    _check(lib().pm_tuning_set(name.encode(), int(value)), f"pm_tuning_set({name})")


def tuning_reset():
    lib().pm_tuning_reset()


class tuning:
    """Context manager: ``with pm.tuning(trap_variant=3, ls_sparse=0): ...``
    (every override is dropped on exit)."""

    def __init__(self, **knobs):
        self.knobs = knobs

    def __enter__(self):
        for k, v in self.knobs.items():
            tuning_set(k, v)
        return self

    def __exit__(self, *exc):
        tuning_reset()


def scratch_trim():
    _check(lib().pm_scratch_trim(), "pm_scratch_trim")


def scratch_reserved_bytes() -> int:
    return int(lib().pm_scratch_reserved_bytes())
