"""GPU parity: the CUDA path (through the C-ABI, paper_conf_ipps_yangin17_b200.pm)
against the CPU oracle (oracle/), element by element, on the same seeded
synthetic inputs.  All results are integers, so the bar is bit-exact:
E (Eq. 1), the final rearrangement r, rounds, swaps (per round) and the total
error (Eq. 2).  Full-size configs 4-5 (BASELINE.json) are checked on sampled
E entries the oracle computes one by one, and the local search there via its
closed-form special case (transposition) and properties that hold at any
size (bijection, 2-swap local optimality, cost identity)."""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

DEV = torch.device("cuda:0")
_cache = {}


@pytest.fixture(autouse=True)
def _reset_tuning():
    # overrides set by a test (pm.tuning_set) never leak into the next one
    pm.tuning_reset()
    yield
    pm.tuning_reset()


def pair(fam, N, M, C=3, seed=0):
    key = ("img", fam, N, M, C, seed)
    if key not in _cache:
        _cache[key] = synth.make_pair(fam, N, M, C, seed)
    return _cache[key]


def oracle_E(fam, N, M, C=3, seed=0):
    key = ("E", fam, N, M, C, seed)
    if key not in _cache:
        I, T = pair(fam, N, M, C, seed)
        _cache[key] = oracle.error_matrix(I, T, M)
    return _cache[key]


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).to(DEV)


# shapes: (N, M, C) -- BASELINE configs 1-3 plus ragged / odd-S / grayscale cases
SHAPES = [(128, 8, 3), (512, 16, 3), (90, 10, 3), (42, 6, 3), (200, 5, 1), (48, 16, 3), (64, 64, 1), (30, 10, 3)]


# ------------------------------------------------------------------ Step 1 --
@pytest.mark.parametrize("N,M,C", SHAPES)
def test_pack_tiles_parity(N, M, C):
    I, _ = pair("noise", N, M, C)
    got = pm.pack_tiles(dev(I), M).cpu().numpy()
    assert (got == oracle.tiles(I, M)).all()


# ------------------------------------------------------------------ Step 2 --
@pytest.mark.parametrize("fam", ["smooth", "noise", "ties"])
@pytest.mark.parametrize("N,M,C", SHAPES)
def test_error_matrix_parity(fam, N, M, C):
    I, T = pair(fam, N, M, C)
    E = pm.error_matrix(dev(I), dev(T), M).cpu().numpy()
    assert (E == oracle_E(fam, N, M, C)).all()


@pytest.mark.parametrize("plan", [64001, 64002, 64003, 64004, 128001, 128002, 128003])
@pytest.mark.parametrize("N,M,C,fam", [(512, 16, 3, "noise"), (90, 10, 3, "smooth"), (256, 16, 1, "ties")])
def test_error_matrix_every_tiling_plan(plan, N, M, C, fam):
    # 128 x 128 and 128 x 64 tiles, with and without split-K (exact red.add)
    pm.tuning_set("sad_plan", plan)
    I, T = pair(fam, N, M, C)
    assert (pm.error_matrix(dev(I), dev(T), M).cpu().numpy() == oracle_E(fam, N, M, C)).all()


def test_error_matrix_config3_full():
    # n = 4096, no split-K path, 32 x 32 CTA tiles
    E = pm.error_matrix(*map(dev, pair("smooth", 1024, 16)), 16).cpu().numpy()
    assert (E == oracle_E("smooth", 1024, 16)).all()


@pytest.mark.parametrize("rows", [(0, 1), (5, 77), (128, 256), (255, 256), (40, 40)])
def test_error_matrix_row_shards(rows):
    I, T = pair("smooth", 128, 8)
    part = pm.error_matrix(dev(I), dev(T), 8, rows=rows).cpu().numpy()
    assert (part == oracle_E("smooth", 128, 8)[rows[0]:rows[1]]).all()


def test_error_matrix_padded_ld():
    I, T = pair("smooth", 128, 8)
    big = torch.full((256, 300), -7, dtype=torch.int32, device=DEV)
    pm.error_matrix(dev(I), dev(T), 8, out=big[:, :256])
    got = big.cpu().numpy()
    assert (got[:, :256] == oracle_E("smooth", 128, 8)).all()
    assert (got[:, 256:] == -7).all(), "writes stay inside [0, S) of each row"


def test_error_matrix_extremes():
    # black vs white: every entry 255 * P = 195840 (max, reading R11)
    I = np.zeros((64, 64, 3), np.uint8)
    T = np.full((64, 64, 3), 255, np.uint8)
    E = pm.error_matrix(dev(I), dev(T), 16).cpu().numpy()
    assert (E == 255 * 768).all()


def test_error_matrix_from_tiles():
    I, T = pair("smooth", 512, 16)
    It, Tt = pm.pack_tiles(dev(I), 16), pm.pack_tiles(dev(T), 16)
    E = pm.error_matrix_tiles(It, Tt, 768).cpu().numpy()
    assert (E == oracle_E("smooth", 512, 16)).all()


def _sampled_E_check(I, T, M, Egpu_rows, row0, rng, k):
    n_rows, S = Egpu_rows.shape
    us = rng.integers(0, n_rows, size=k)
    vs = rng.integers(0, S, size=k)
    got = Egpu_rows[torch.from_numpy(us).to(DEV), torch.from_numpy(vs).to(DEV)].cpu().numpy()
    for u, v, g in zip(us, vs, got):
        assert g == oracle.error_entry(I, T, M, row0 + int(u), int(v)), (row0 + u, v)


def test_error_matrix_config4_sampled():
    I, T = pair("smooth", 2048, 16)
    E = pm.error_matrix(dev(I), dev(T), 16)
    rng = np.random.default_rng(4)
    _sampled_E_check(I, T, 16, E, 0, rng, 3000)
    # the four corners and the diagonal ends explicitly
    for u, v in [(0, 0), (0, 16383), (16383, 0), (16383, 16383)]:
        assert int(E[u, v]) == oracle.error_entry(I, T, 16, u, v)


def test_error_matrix_config5_row_chunks_sampled():
    # n = 65536 (16 GiB E): computed in 4096-row shards, as a rank of an 8-GPU
    # job would, each shard sampled against the oracle
    I, T = pair("smooth", 4096, 16)
    dI, dT = dev(I), dev(T)
    rng = np.random.default_rng(5)
    buf = torch.empty((4096, 65536), dtype=torch.int32, device=DEV)
    for r0 in range(0, 65536, 4096):
        pm.error_matrix(dI, dT, 16, rows=(r0, r0 + 4096), out=buf)
        _sampled_E_check(I, T, 16, buf, r0, rng, 150)


# ------------------------------------------------------------------ Alg. 2 --
def _supported(method, S):
    return not (method == "window" and S > 2048) and not (method == "trap" and (S < 256 or S % 2))


def _check_ls(E_np, method, perm0=None, max_rounds=0):
    if not _supported(method, E_np.shape[0]):
        pytest.skip(f"{method} does not take S = {E_np.shape[0]}")
    ref = oracle.local_search(E_np, r0=perm0, max_rounds=max_rounds)
    E = dev(E_np)
    perm = dev(np.arange(E_np.shape[0], dtype=np.int32) if perm0 is None else perm0.astype(np.int32))
    out, rounds, swaps, per, st = pm.local_search(E, perm, max_rounds=max_rounds, method=method,
                                                  allow_not_converged=True)
    assert (out.cpu().numpy() == ref[0]).all(), "final rearrangement r"
    assert (rounds, swaps) == (ref[1], ref[2])
    assert (per == ref[3][: len(per)]).all()
    assert st == ref[4]
    return ref


@pytest.mark.parametrize("method", ["trap", "walk", "window", "class"])
@pytest.mark.parametrize("fam", ["smooth", "noise", "ties", "shuffle", "transposition", "identical"])
def test_local_search_parity_config1(method, fam):
    _check_ls(oracle_E(fam, 128, 8), method)


@pytest.mark.parametrize("method", ["trap", "walk", "window", "class"])
@pytest.mark.parametrize("fam", ["smooth", "noise", "ties"])
def test_local_search_parity_config2(method, fam):
    _check_ls(oracle_E(fam, 512, 16), method)


@pytest.mark.parametrize("method", ["auto", "trap", "walk", "class"])
def test_local_search_parity_config3(method):
    ref = _check_ls(oracle_E("smooth", 1024, 16), method)
    assert ref[1] >= 3


@pytest.mark.parametrize("method", ["trap", "walk", "window", "class"])
@pytest.mark.parametrize("N,M,C", [(90, 10, 3), (42, 6, 3), (200, 5, 1), (48, 16, 3), (30, 10, 3), (64, 64, 1)])
def test_local_search_parity_ragged_and_odd(method, N, M, C):
    # S = 81, 49, 9 are odd (the fixed point idles, reading R9); S = 1 trivial
    _check_ls(oracle_E("smooth", N, M, C), method)


@pytest.mark.parametrize("method", ["trap", "walk", "window", "class"])
def test_local_search_resume_from_any_bijection(method):
    E = oracle_E("noise", 128, 8)
    rng = np.random.default_rng(3)
    _check_ls(E, method, perm0=rng.permutation(256).astype(np.int32))


@pytest.mark.parametrize("method", ["trap", "walk", "window", "class"])
def test_local_search_max_rounds_then_resume(method):
    E_np = oracle_E("smooth", 512, 16)
    ref = _check_ls(E_np, method, max_rounds=2)
    assert ref[4] == pm.PM_ERR_NOT_CONVERGED
    _check_ls(E_np, method, perm0=ref[0])


@pytest.mark.parametrize("method", ["trap", "walk", "window", "class"])
def test_local_search_rejects_non_permutation(method):
    E = dev(oracle_E("smooth", 128, 8))
    bad = torch.arange(256, dtype=torch.int32, device=DEV)
    bad[7] = 3
    with pytest.raises(pm.PMError) as ei:
        pm.local_search(E, bad, method=method)
    assert ei.value.status == pm.PM_ERR_NOT_PERMUTATION
    bad[7] = 999
    with pytest.raises(pm.PMError) as ei:
        pm.local_search(E, bad, method=method)
    assert ei.value.status == pm.PM_ERR_NOT_PERMUTATION


def test_local_search_random_small_matrices():
    # tie-heavy random E for S <= 9 against the oracle replay, every method
    # that takes such S
    rng = np.random.default_rng(0)
    for _ in range(25):
        S = int(rng.integers(1, 10))
        E = rng.integers(0, 4, size=(S, S)).astype(np.int32)
        for method in ("walk", "window", "class"):
            _check_ls(E, method)


@pytest.mark.parametrize("S", [256, 258, 300, 512])
@pytest.mark.parametrize("hi", [2, 4, 50])
def test_trap_tie_heavy_random_E(S, hi):
    # TRAP's smallest S with random E whose entries take only `hi` values:
    # many line-5 ties (strict '>', reading R6), swaps anywhere incl. pair 0
    rng = np.random.default_rng(S * 100 + hi)
    E = rng.integers(0, hi, size=(S, S)).astype(np.int32)
    _check_ls(E, "trap")
    with pm.tuning(ls_sparse=0):
        _check_ls(E, "trap")


def _two_opt_gpu(E, perm):
    F = E.index_select(0, perm.long())                   # F[u][v] = E[r[u]][v]
    d = torch.diagonal(F).to(torch.int64)
    S = F.shape[0]
    for r0 in range(0, S, 2048):
        r1 = min(S, r0 + 2048)
        lhs = d[r0:r1, None] + d[None, :]
        rhs = F[r0:r1].to(torch.int64) + F[:, r0:r1].T.to(torch.int64)
        if bool((lhs > rhs).any()):
            return False
    return True


def test_local_search_config4_properties_and_closed_form():
    # n = 16384 (E = 1 GiB, beyond L2): transposition closed form (1 swap,
    # 2 rounds, cost 0) and, on the smooth family, bijection + 2-opt + cost.
    I, T = pair("transposition", 2048, 16)
    E = pm.error_matrix(dev(I), dev(T), 16)
    moved = torch.nonzero(torch.diagonal(E)).flatten().cpu().numpy()
    assert len(moved) == 2
    perm, rounds, swaps, per, st = pm.local_search(E)
    expect = np.arange(16384)
    expect[moved[0]], expect[moved[1]] = moved[1], moved[0]
    assert (perm.cpu().numpy() == expect).all() and (rounds, swaps) == (2, 1)
    assert pm.cost(E, perm) == 0

    I, T = pair("smooth", 2048, 16)
    E = pm.error_matrix(dev(I), dev(T), 16)
    perm, rounds, swaps, per, st = pm.local_search(E)
    p = perm.cpu().numpy()
    assert sorted(p.tolist()) == list(range(16384))
    assert per[-1] == 0 and per.sum() == swaps
    assert _two_opt_gpu(E, perm)
    assert pm.cost(E, perm) == int(E[perm.long(), torch.arange(16384, device=DEV)].to(torch.int64).sum())


def test_local_search_config5_properties_and_closed_form():
    # n = 65536 (E = 16 GiB): transposition closed form (1 swap, 2 rounds,
    # cost 0) and, on the smooth family, bijection + 2-opt + cost identity
    I, T = pair("transposition", 4096, 16)
    E = pm.error_matrix(dev(I), dev(T), 16)
    moved = torch.nonzero(torch.diagonal(E)).flatten().cpu().numpy()
    assert len(moved) == 2
    perm, rounds, swaps, per, st = pm.local_search(E)
    expect = np.arange(65536)
    expect[moved[0]], expect[moved[1]] = moved[1], moved[0]
    assert (perm.cpu().numpy() == expect).all() and (rounds, swaps) == (2, 1)
    assert pm.cost(E, perm) == 0
    del E
    I, T = pair("smooth", 4096, 16)
    E = pm.error_matrix(dev(I), dev(T), 16)
    perm, rounds, swaps, per, st = pm.local_search(E)
    assert sorted(perm.cpu().numpy().tolist()) == list(range(65536))
    assert per[-1] == 0 and per.sum() == swaps
    assert _two_opt_gpu(E, perm)
    assert pm.cost(E, perm) == int(E[perm.long(), torch.arange(65536, device=DEV)].to(torch.int64).sum())


# ------------------------------------------------------------------ Eq. (2) -
@pytest.mark.parametrize("N,M,C", [(128, 8, 3), (512, 16, 3), (90, 10, 3)])
def test_cost_parity(N, M, C):
    E_np = oracle_E("smooth", N, M, C)
    S = E_np.shape[0]
    rng = np.random.default_rng(S)
    for perm in (np.arange(S), rng.permutation(S)):
        perm = perm.astype(np.int32)
        assert pm.cost(dev(E_np), dev(perm)) == oracle.cost(E_np, perm)


def test_cost_int64():
    S = 64
    E = torch.full((S, S), 2**31 - 1, dtype=torch.int32, device=DEV)
    assert pm.cost(E, torch.arange(S, dtype=torch.int32, device=DEV)) == S * (2**31 - 1)


# -------------------------------------------------------------- pipeline ----
@pytest.mark.parametrize("method", ["auto", "trap", "window", "class"])
def test_photomosaic_pipeline_config2(method):
    I, T = pair("smooth", 512, 16)
    E_np = oracle_E("smooth", 512, 16)
    ref = oracle.local_search(E_np)
    perm, rounds, swaps, c, E = pm.photomosaic(dev(I), dev(T), 16, method=method)
    assert (E.cpu().numpy() == E_np).all()
    assert (perm.cpu().numpy() == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])
    assert c == oracle.cost(E_np, ref[0])


def test_photomosaic_host_config1():
    I, T = pair("smooth", 128, 8)
    E_np = oracle_E("smooth", 128, 8)
    ref = oracle.local_search(E_np)
    perm, rounds, swaps, c = pm.photomosaic_host(I, T, 8)
    assert (perm == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])
    assert c == oracle.cost(E_np, ref[0])


# ------------------------------------------------------------ error paths ---
def test_invalid_arguments_launch_nothing():
    L = pm.lib()
    I = torch.zeros((64, 64, 3), dtype=torch.uint8, device=DEV)
    E = torch.zeros((16, 16), dtype=torch.int32, device=DEV)
    n0 = pm.launch_count()
    assert L.pm_error_matrix(I.data_ptr(), I.data_ptr(), 64, 15, 3, 0, 16, E.data_ptr(), 16, None) == pm.PM_ERR_INVALID
    assert L.pm_error_matrix(I.data_ptr(), I.data_ptr(), 64, 16, 3, 0, 17, E.data_ptr(), 16, None) == pm.PM_ERR_INVALID
    assert L.pm_error_matrix(I.data_ptr(), I.data_ptr(), 64, 16, 3, 0, 16, E.data_ptr(), 15, None) == pm.PM_ERR_INVALID
    assert L.pm_error_matrix(None, I.data_ptr(), 64, 16, 3, 0, 16, E.data_ptr(), 16, None) == pm.PM_ERR_INVALID
    # 255 * P must fit int32 (reading R11)
    assert L.pm_error_matrix(I.data_ptr(), I.data_ptr(), 8192, 4096, 1, 0, 4, E.data_ptr(), 16,
                             None) == pm.PM_ERR_INVALID
    assert L.pm_local_search(E.data_ptr(), 15, 16, E.data_ptr(), 0, None, None, None) == pm.PM_ERR_INVALID
    assert L.pm_local_search_ex(E.data_ptr(), 16, 16, E.data_ptr(), 0, 9, None, None, None, 0,
                                None) == pm.PM_ERR_INVALID
    assert L.pm_cost(E.data_ptr(), 16, 0, E.data_ptr(), None, None) == pm.PM_ERR_INVALID
    assert pm.launch_count() == n0


def test_launch_count_increments():
    I, T = pair("smooth", 128, 8)
    n0 = pm.launch_count()
    pm.photomosaic(dev(I), dev(T), 8, method="class")
    assert pm.launch_count() - n0 >= 5   # 2 pack + E + iota + search + cost


@pytest.mark.parametrize("method", ["window"])
@pytest.mark.parametrize("N,M", [(1600, 40), (1152, 32), (1440, 32), (224, 32), (280, 40)])
def test_local_search_window_sizes(N, M, method):
    # S = 1600, 1296, 2025 (the second window tier, S in (1024, 2048]), 49, 49 -- grayscale noise
    _check_ls(oracle_E("noise", N, M, 1), method)


@pytest.mark.parametrize("method", ["window"])
@pytest.mark.parametrize("S_side", [7, 31, 33, 45])
def test_local_search_window_odd_mid(S_side, method):
    # odd S around the window tiers (49, 961, 1089, 2025)
    _check_ls(oracle_E("smooth", S_side * 4, 4, 3), method)


def test_local_search_window_rejects_large_S():
    E = torch.zeros((2116, 2116), dtype=torch.int32, device=DEV)
    with pytest.raises(pm.PMError) as ei:
        pm.local_search(E, method="window")
    assert ei.value.status == pm.PM_ERR_UNSUPPORTED


# ------------------------------------------------------- fused Step 1 path --
@pytest.mark.parametrize("N,M,C,rows", [(512, 16, 3, (100, 900)), (256, 16, 1, None), (192, 32, 1, (3, 30)),
                                        (320, 16, 3, (0, 400))])
def test_error_matrix_fused_loader_parity(N, M, C, rows):
    # M*C % 16 == 0 and P % 64 == 0: the E kernel reads tiles straight from the images
    I, T = pair("noise", N, M, C)
    E = pm.error_matrix(dev(I), dev(T), M, rows=rows).cpu().numpy()
    ref = oracle_E("noise", N, M, C)
    assert (E == (ref if rows is None else ref[rows[0]:rows[1]])).all()


def test_error_matrix_unaligned_images_fall_back_to_packing():
    # image base pointers not 16-byte aligned -> packed path, same result
    I, T = pair("smooth", 512, 16)
    bufI = torch.empty(I.size + 16, dtype=torch.uint8, device=DEV)
    bufT = torch.empty(T.size + 16, dtype=torch.uint8, device=DEV)
    dI = bufI[1:1 + I.size].view(512, 512, 3)
    dT = bufT[3:3 + T.size].view(512, 512, 3)
    dI.copy_(dev(I))
    dT.copy_(dev(T))
    E = pm.error_matrix(dI, dT, 16).cpu().numpy()
    assert (E == oracle_E("smooth", 512, 16)).all()


def test_error_matrix_simulated_8_shards_config4():
    # the row shards an 8-GPU job computes (dist.shard_rows) reassemble E exactly
    from paper_conf_ipps_yangin17_b200 import dist as pdist
    I, T = pair("smooth", 2048, 16)
    dI, dT = dev(I), dev(T)
    full = pm.error_matrix(dI, dT, 16)
    for g in range(8):
        b, e = pdist.shard_rows(16384, 8, g)
        part = pm.error_matrix(dI, dT, 16, rows=(b, e))
        assert torch.equal(part, full[b:e])


# ------------------------------------------- NEXT-1: the paper's grayscale grid
@pytest.mark.parametrize("N,g", [(512, 16), (512, 32), (512, 64), (1024, 16), (1024, 32), (1024, 64),
                                 (2048, 16), (2048, 32), (2048, 64)])
def test_paper_grid_grayscale_parity(N, g):
    # all nine Tables II-IV shapes, C = 1: grids 16^2 / 32^2 / 64^2
    # (S = 256 / 1024 / 4096), tile sides 8..128 px, P up to 16384 bytes --
    # E, r, rounds, swaps and cost against the oracle
    M = N // g
    I, T = pair("smooth", N, M, 1)
    Eg = pm.error_matrix(dev(I), dev(T), M)
    E = oracle_E("smooth", N, M, 1)
    assert (Eg.cpu().numpy() == E).all()
    ref = oracle.local_search(E)
    perm, rounds, swaps, per, st = pm.local_search(Eg)
    assert (perm.cpu().numpy() == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])
    assert (per == ref[3]).all()
    assert pm.cost(Eg, perm) == oracle.cost(E, ref[0])


# ------------------------------------------------- NEXT-3: render R --
@pytest.mark.parametrize("N,M,C", [(128, 8, 3), (90, 10, 3), (200, 5, 1)])
def test_render_parity(N, M, C):
    I, T = pair("noise", N, M, C)
    S = (N // M) ** 2
    perm = np.random.default_rng(S).permutation(S).astype(np.int32)
    R = pm.render(dev(I), M, dev(perm)).cpu().numpy()
    assert R.shape == I.shape and (R == oracle.render(I, M, perm)).all()


def test_render_transposition_reproduces_target():
    # closed form: Alg. 2 solves a transposition exactly, so R == T bit for bit
    I, T = pair("transposition", 512, 16)
    perm, rounds, swaps, cost, E = pm.photomosaic(dev(I), dev(T), 16)
    assert cost == 0 and (pm.render(dev(I), 16, perm).cpu().numpy() == T).all()


# ------------------------------------------- sparse rounds (k_sparse.cu) ---
# The dense stage (WINDOW / CLASS) hands over to exact sparse rounds after a
# round with <= PM_LS_SPARSE_T swaps; every hand-over point must reproduce the
# oracle bit for bit (r, rounds, swaps per round).
@pytest.mark.parametrize("cwalk", ["0", "1"])
@pytest.mark.parametrize("method", ["window", "class"])
@pytest.mark.parametrize("T", ["0", "1", "40", "1000000000"])
@pytest.mark.parametrize("shape,fam", [((128, 8, 3), "smooth"), ((512, 16, 3), "smooth"), ((90, 10, 3), "smooth"),
                                       ((200, 5, 1), "noise"), ((128, 8, 3), "ties"), ((42, 6, 3), "transposition")])
def test_sparse_rounds_parity(cwalk, method, T, shape, fam):
    pm.tuning_set("ls_cwalk", int(cwalk))
    pm.tuning_set("ls_sparse_T", int(T))
    _check_ls(oracle_E(fam, *shape), method)


@pytest.mark.parametrize("cwalk", ["0", "1"])
@pytest.mark.parametrize("gmem", ["0", "1"])
def test_sparse_rounds_global_arrays_and_resume(gmem, cwalk):
    """Walk arrays in global memory (the S > 17K layout, forced), a resumed
    search and a max_rounds cut that lands inside the sparse stage."""
    pm.tuning_set("ls_sparse_gmem", int(gmem))
    pm.tuning_set("ls_cwalk", int(cwalk))
    pm.tuning_set("ls_sparse_T", 1000000000)
    E_np = oracle_E("smooth", 512, 16)
    _check_ls(E_np, "walk")
    for mr in (1, 2, 4):
        _check_ls(E_np, "walk", max_rounds=mr)
    _check_ls(E_np, "class")
    _check_ls(E_np, "window")
    for mr in (1, 2, 3, 5):
        _check_ls(E_np, "window", max_rounds=mr)
        _check_ls(E_np, "class", max_rounds=mr)
    rng = np.random.default_rng(5)
    _check_ls(E_np, "window", perm0=rng.permutation(E_np.shape[0]))


def test_sparse_rounds_disabled_matches():
    pm.tuning_set("ls_sparse", 0)
    _check_ls(oracle_E("smooth", 512, 16), "window")
    _check_ls(oracle_E("smooth", 128, 8), "class")


# ---------------------------------- cluster walk (k_cwalk.cu), all rounds ---
@pytest.mark.parametrize("fam", ["smooth", "noise", "ties", "transposition", "identical", "shuffle"])
@pytest.mark.parametrize("N,M,C", [(128, 8, 3), (512, 16, 3), (90, 10, 3), (200, 5, 1), (1152, 32, 1), (1440, 32, 1)])
def test_walk_all_rounds_parity(fam, N, M, C):
    # S = 256, 1024, 81 (odd), 1600, 1296, 2025 (odd): every round as scan + cluster walk
    _check_ls(oracle_E(fam, N, M, C), "walk")


@pytest.mark.parametrize("C", [8, 16])
@pytest.mark.parametrize("N,M,C_img,fam", [(512, 16, 3, "smooth"), (1440, 32, 1, "noise"), (128, 8, 3, "ties")])
def test_walk_cluster_sizes(C, N, M, C_img, fam):
    # the cluster walk on 8 (portable) or 16 (non-portable) CTAs
    pm.tuning_set("ls_cwalk_c", C)
    pm.tuning_set("ls_cwalk", 1)
    _check_ls(oracle_E(fam, N, M, C_img), "walk")


def test_walk_mailbox_overflow_falls_back_exactly():
    # T = I with the tiles of 63 pairs of the first colour class exchanged: from
    # the identity all 63 fire in that class, more than one CTA's mailbox holds
    # (k_cwalk.cu), so every CTA re-tests the class in full
    I, _ = pair("smooth", 512, 16)
    g, M = 32, 16
    groups = oracle.edge_coloring(g * g)          # [class][pair][2]
    Tt = I.copy()
    for a, b in groups[0][:63]:
        ya, xa, yb, xb = (a // g) * M, (a % g) * M, (b // g) * M, (b % g) * M
        ta = Tt[ya:ya + M, xa:xa + M].copy()
        Tt[ya:ya + M, xa:xa + M] = Tt[yb:yb + M, xb:xb + M]
        Tt[yb:yb + M, xb:xb + M] = ta
    E_np = oracle.error_matrix(I, Tt, M)
    ref = _check_ls(E_np, "walk")
    assert ref[3][0] >= 63


def _check_trap(E_np, cluster_forced=False):
    # the cluster mode is unsupported (PM_ERR_UNSUPPORTED) when the chunks do
    # not fit one cluster; every other outcome must match the oracle
    try:
        _check_ls(E_np, "trap")
    except pm.PMError as e:
        if e.status != pm.PM_ERR_UNSUPPORTED or not cluster_forced:
            raise
        pytest.skip("chunks do not fit one cluster")


# ---- PM_LS_TRAP: every round on the temporal-blocked kernel (sparse hand-over
# off), every compiled (pairs-per-lane, T) variant, chunk widths that do not
# divide S/2, grid-barrier and cluster (DSMEM) modes.
@pytest.mark.parametrize("variant", [0, 1, 2, 3, 4, 5, 6, 7])
@pytest.mark.parametrize("N,M,fam,W", [(128, 8, "smooth", 0), (512, 16, "smooth", 0), (512, 16, "ties", 7),
                                       (240, 8, "noise", 0), (336, 8, "smooth", 21), (128, 8, "transposition", 19)])
@pytest.mark.parametrize("mode", ["0", "1"])
def test_trap_every_round(variant, N, M, fam, W, mode):
    pm.tuning_set("trap_variant", int(variant))
    pm.tuning_set("trap_cluster", int(mode))
    pm.tuning_set("ls_sparse", 0)
    pm.tuning_set("trap_W", int(W))
    _check_trap(oracle_E(fam, N, M), mode == "1")


@pytest.mark.parametrize("spec", [0, 1, 2])
@pytest.mark.parametrize("variant", [0, 1, 3, 5, 6, 7])
@pytest.mark.parametrize("N,M,fam", [(512, 16, "smooth"), (512, 16, "ties"), (336, 8, "smooth"), (1024, 16, "smooth")])
@pytest.mark.parametrize("mode", ["0", "1"])
def test_trap_speculative_steps(spec, variant, N, M, fam, mode):
    # speculative class steps (batches of classes tested on the state of the
    # batch start, first firing class applied exactly): off, after quiet
    # rounds (default), every round -- with and without sparse rounds after
    pm.tuning_set("trap_spec", spec)
    pm.tuning_set("trap_variant", variant)
    pm.tuning_set("trap_cluster", int(mode))
    E_np = oracle_E(fam, N, M)
    _check_trap(E_np, mode == "1")
    pm.tuning_set("ls_sparse", 0)
    _check_trap(E_np, mode == "1")


@pytest.mark.parametrize("cpc,variant", [(1, 0), (2, 0), (3, 1), (1, 3), (2, 4), (4, 2), (8, 1)])
@pytest.mark.parametrize("mode", ["0", "1"])
def test_trap_chunks_per_cta(cpc, variant, mode):
    pm.tuning_set("trap_cluster", int(mode))
    pm.tuning_set("trap_cpc", int(cpc))
    pm.tuning_set("trap_variant", int(variant))
    pm.tuning_set("ls_sparse", 0)
    # cluster mode holds every chunk in <= 16 CTAs: S = 1024 (16-64 chunks)
    _check_trap(oracle_E("noise", 1024 if mode == "0" else 512, 16), mode == "1")


@pytest.mark.parametrize("method", ["trap", "class", "window"])
def test_local_search_padded_leading_dimension(method):
    # E as the left S columns of a wider matrix (ld_E = S + 3): TRAP's
    # 16-byte row pieces need ld_E % 4 == 0 and take the entry-wise path here
    E_np = oracle_E("smooth", 512, 16)
    S = E_np.shape[0]
    ref = oracle.local_search(E_np)
    big = torch.full((S, S + 3), -1, dtype=torch.int32, device=DEV)
    big[:, :S] = dev(E_np)
    out, rounds, swaps, per, st = pm.local_search(big[:, :S], method=method)
    assert (out.cpu().numpy() == ref[0]).all()
    assert (rounds, swaps) == (ref[1], ref[2])


@pytest.mark.parametrize("variant,mode,vec", [("0", "0", "1"), ("0", "0", "0"), ("1", "1", "1"), ("3", "0", "1"), ("5", "0", "0")])
def test_trap_every_round_config3(variant, mode, vec):
    # S = 4096 with P = 768: pair-0 swaps at every u0 mod 4 (the 16-byte span offsets)
    pm.tuning_set("trap_variant", int(variant))
    pm.tuning_set("trap_cluster", int(mode))
    pm.tuning_set("trap_vec", int(vec))
    pm.tuning_set("ls_sparse", 0)
    _check_trap(oracle_E("smooth", 1024, 16), mode == "1")


# ---- multi-GPU TRAP protocol (pm_local_search_multi_*): every rank of a world
# emulated in one launch on this GPU -- chunk ranges per rank, halo slots and
# phase flags to the neighbour ranks' workspaces, per-round cross-rank swap
# totals and barrier, the final r on every rank -- against the oracle.
@pytest.mark.parametrize("N,M,fam,world", [(128, 8, "smooth", 2), (128, 8, "noise", 4), (512, 16, "smooth", 1),
                                           (512, 16, "smooth", 2), (512, 16, "ties", 3), (512, 16, "smooth", 8),
                                           (1024, 16, "smooth", 4), (336, 8, "transposition", 5)])
def test_multi_rank_trap_emulated(N, M, fam, world):
    E_np = oracle_E(fam, N, M)
    ref = oracle.local_search(E_np)
    out, rounds, swaps = pm.local_search_multi_emulated(dev(E_np), world)
    assert (out.cpu().numpy() == ref[0]).all()
    assert (rounds, swaps) == (ref[1], ref[2])


@pytest.mark.parametrize("variant", ["0", "5", "6"])
def test_multi_rank_trap_geometries(variant):
    pm.tuning_set("trap_variant", int(variant))
    E_np = oracle_E("smooth", 1024, 16)
    ref = oracle.local_search(E_np)
    out, rounds, swaps = pm.local_search_multi_emulated(dev(E_np), 3)
    assert (out.cpu().numpy() == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])


def test_multi_rank_trap_max_rounds_then_resume():
    E_np = oracle_E("smooth", 512, 16)
    ref = oracle.local_search(E_np, max_rounds=2)
    out, rounds, swaps = pm.local_search_multi_emulated(dev(E_np), 3, max_rounds=2)
    assert (out.cpu().numpy() == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])
    ref2 = oracle.local_search(E_np, r0=ref[0])
    out2, rounds2, swaps2 = pm.local_search_multi_emulated(dev(E_np), 3, perm=out)
    assert (out2.cpu().numpy() == ref2[0]).all() and (rounds2, swaps2) == (ref2[1], ref2[2])


def test_multi_rank_trap_symmetric_memory_world1():
    # the multi-process plumbing (torch symmetric memory, peer pointer table,
    # workspace reset + barrier) through pm_local_search_multi_async, at one rank
    import torch.distributed as tdist

    from paper_conf_ipps_yangin17_b200 import dist as pdist
    E_np = oracle_E("smooth", 512, 16)
    ref = oracle.local_search(E_np)
    own = not tdist.is_initialized()
    if own:
        tdist.init_process_group("nccl", init_method="tcp://127.0.0.1:29513", rank=0, world_size=1,
                                 device_id=torch.device(DEV))
    try:
        try:
            out, rounds, swaps = pdist.local_search_multi(dev(E_np))
        except (RuntimeError, AttributeError) as e:
            pytest.skip(f"symmetric memory unavailable here: {e}")
        assert (out.cpu().numpy() == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])
    finally:
        if own:
            tdist.destroy_process_group()


# ---- the same protocol over ROW-SHARDED E (pm_local_search_sharded_*): E's
# rows split into `world` separate shard buffers, each rank's permuted rows in
# its own workspace, every TRAP tile reading the owner's shard
@pytest.mark.parametrize("N,M,fam,world", [(128, 8, "smooth", 2), (128, 8, "noise", 4), (512, 16, "smooth", 1),
                                           (512, 16, "smooth", 2), (512, 16, "ties", 3), (512, 16, "smooth", 8),
                                           (1024, 16, "smooth", 4), (1024, 16, "noise", 7),
                                           (336, 8, "transposition", 5)])
def test_sharded_trap_emulated(N, M, fam, world):
    E_np = oracle_E(fam, N, M)
    ref = oracle.local_search(E_np)
    out, rounds, swaps = pm.local_search_sharded_emulated(dev(E_np), world)
    assert (out.cpu().numpy() == ref[0]).all()
    assert (rounds, swaps) == (ref[1], ref[2])


@pytest.mark.parametrize("variant", ["0", "5", "6"])
def test_sharded_trap_geometries(variant):
    pm.tuning_set("trap_variant", int(variant))
    E_np = oracle_E("smooth", 1024, 16)
    ref = oracle.local_search(E_np)
    out, rounds, swaps = pm.local_search_sharded_emulated(dev(E_np), 3)
    assert (out.cpu().numpy() == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])


def test_sharded_trap_padded_ld_max_rounds_then_resume():
    E_np = oracle_E("smooth", 512, 16)
    S = E_np.shape[0]
    big = torch.full((S, S + 5), -7, dtype=torch.int32, device=DEV)
    big[:, :S] = dev(E_np)
    ref = oracle.local_search(E_np, max_rounds=2)
    out, rounds, swaps = pm.local_search_sharded_emulated(big[:, :S], 3, max_rounds=2)
    assert (out.cpu().numpy() == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])
    ref2 = oracle.local_search(E_np, r0=ref[0])
    out2, rounds2, swaps2 = pm.local_search_sharded_emulated(big[:, :S], 3, perm=out)
    assert (out2.cpu().numpy() == ref2[0]).all() and (rounds2, swaps2) == (ref2[1], ref2[2])


@pytest.mark.parametrize("bounds", ["even", "empty_first"])
def test_sharded_async_one_process(bounds):
    # pm_local_search_sharded_async itself at world 1 (own shard = all of E),
    # and at world 2 with rank 1 owning every row while rank 0 holds none --
    # rank 0 alone cannot finish, so that case is run as the bounded-wait
    # failure path: PM_ERR_TIMEOUT, nothing hangs
    E_np = oracle_E("smooth", 512, 16)
    S = E_np.shape[0]
    E = dev(E_np)
    ref = oracle.local_search(E_np)
    res = torch.zeros(3, dtype=torch.int64, device=DEV)
    if bounds == "even":
        wsb = pm.trap_workspace_bytes_sharded(S, S)
        ws = torch.zeros(wsb, dtype=torch.uint8, device=DEV)
        perm = torch.arange(S, dtype=torch.int32, device=DEV)
        pm.local_search_sharded_async([E.data_ptr()], [0, S], E.stride(0), S, [perm.data_ptr()], [ws.data_ptr()],
                                      0, 1, res)
        torch.cuda.synchronize()
        assert int(res[0]) == pm.PM_OK
        assert (perm.cpu().numpy() == ref[0]).all() and (int(res[1]), int(res[2])) == (ref[1], ref[2])
    else:
        wss = [torch.zeros(pm.trap_workspace_bytes_sharded(S, n), dtype=torch.uint8, device=DEV) for n in (0, S)]
        perms = [torch.arange(S, dtype=torch.int32, device=DEV) for _ in range(2)]
        with pm.tuning(trap_wait_ms=300):
            pm.local_search_sharded_async([0, E.data_ptr()], [0, 0, S], E.stride(0), S,
                                          [p_.data_ptr() for p_ in perms], [w.data_ptr() for w in wss], 0, 2, res)
            torch.cuda.synchronize()
        assert int(res[0]) == pm.PM_ERR_TIMEOUT
        _check_ls(E_np, "trap")


def test_sharded_symmetric_memory_world1():
    # dist.photomosaic_sharded / local_search_sharded (symmetric-memory shard,
    # workspace and perm; pm_error_matrix straight into the shard) at one rank
    import torch.distributed as tdist

    from paper_conf_ipps_yangin17_b200 import dist as pdist
    I, T = pair("smooth", 512, 16)
    E_np = oracle.error_matrix(I, T, 16)
    ref = oracle.local_search(E_np)
    own = not tdist.is_initialized()
    if own:
        tdist.init_process_group("nccl", init_method="tcp://127.0.0.1:29514", rank=0, world_size=1,
                                 device_id=torch.device(DEV))
    try:
        try:
            out, rounds, swaps = pdist.photomosaic_sharded(dev(I), dev(T), 16)
        except (RuntimeError, AttributeError) as e:
            pytest.skip(f"symmetric memory unavailable here: {e}")
        assert (out.cpu().numpy() == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])
        out2, rounds2, swaps2 = pdist.local_search_sharded(dev(E_np), E_np.shape[0])
        assert (out2.cpu().numpy() == ref[0]).all() and (rounds2, swaps2) == (ref[1], ref[2])
    finally:
        if own:
            tdist.destroy_process_group()


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_cost_sharded(world):
    # Eq. (2) with E split into `world` separate shard buffers (uneven bounds)
    E_np = oracle_E("noise", 512, 16)
    S = E_np.shape[0]
    rng = np.random.default_rng(world)
    r = rng.permutation(S).astype(np.int32)
    cuts = sorted(rng.integers(0, S + 1, size=world - 1).tolist())
    rb = [0] + cuts + [S]
    shards = [dev(E_np[rb[o]:rb[o + 1]]) if rb[o + 1] > rb[o] else None for o in range(world)]
    out = torch.full((1,), -1, dtype=torch.int64, device=DEV)
    pm.cost_sharded_async([0 if t is None else t.data_ptr() for t in shards], rb, S, S, dev(r), out)
    assert int(out.item()) == oracle.cost(E_np, r)


@pytest.mark.parametrize("coal", [0, 1])
@pytest.mark.parametrize("ep,mode", [("0", "1"), ("0", "0"), ("1", "0"), ("1", "1")])
def test_trap_sigma_permuted_and_plain_row_staging(ep, mode, coal):
    # runs staged from the sigma-permuted copy of E (default while E is
    # L2-resident), warp-cooperatively or one thread per tile, or from E's rows
    # directly: identical results
    pm.tuning_set("trap_ep", int(ep))
    pm.tuning_set("trap_cluster", int(mode))
    pm.tuning_set("trap_coal", coal)
    pm.tuning_set("ls_sparse", 0)
    _check_trap(oracle_E("smooth", 512, 16), mode == "1")
    _check_trap(oracle_E("ties", 128, 8), mode == "1")


# ------------------------------------------------------- failure paths -----
def test_multi_rank_timeout_when_a_peer_never_runs():
    # rank 0 of a world of 2 on this GPU; rank 1 is never launched.  Every
    # cross-rank wait is bounded: rank 0 stops with PM_ERR_TIMEOUT instead of
    # hanging, and the sparse rounds after it do not run
    S = 1024
    E = dev(oracle_E("smooth", 512, 16))
    wsb = (pm.trap_workspace_bytes(S) + 255) // 256 * 256
    bufs = [torch.zeros(wsb + 4 * S, dtype=torch.uint8, device=DEV) for _ in range(2)]
    perms = [b[wsb:].view(torch.int32) for b in bufs]
    for p_ in perms:
        pm.init_identity(p_)
    res = torch.zeros(3, dtype=torch.int64, device=DEV)
    with pm.tuning(trap_wait_ms=300):
        pm.local_search_multi_async(E, [p_.data_ptr() for p_ in perms], [b.data_ptr() for b in bufs], 0, 2, res)
        torch.cuda.synchronize()
    assert int(res[0]) == pm.PM_ERR_TIMEOUT
    # the device is still usable: a normal search right after is exact
    _check_ls(oracle_E("smooth", 512, 16), "trap")


def test_multi_rank_rejects_unsupported_before_enqueue():
    E = torch.zeros((258, 258), dtype=torch.int32, device=DEV)
    res = torch.full((3,), -5, dtype=torch.int64, device=DEV)
    n0 = pm.launch_count()
    with pytest.raises(pm.PMError) as ei:      # 129 pairs -> 5 chunks < world 8
        pm.local_search_multi_async(E, [E.data_ptr()] * 8, [E.data_ptr()] * 8, 0, 8, res)
    assert ei.value.status == pm.PM_ERR_UNSUPPORTED
    assert int(res[0]) == -5 and pm.launch_count() == n0     # nothing enqueued


def test_photomosaic_trap_odd_S_rejected_before_error_matrix():
    I, T = pair("smooth", 90, 10)              # S = 81 (odd): TRAP does not take it
    n0 = pm.launch_count()
    with pytest.raises(pm.PMError) as ei:
        pm.photomosaic(dev(I), dev(T), 10, method="trap")
    assert ei.value.status == pm.PM_ERR_UNSUPPORTED and pm.launch_count() == n0


def test_scratch_pool_trim():
    E = dev(oracle_E("smooth", 512, 16))
    pm.local_search(E)
    torch.cuda.synchronize()
    assert pm.scratch_reserved_bytes() > 0
    pm.scratch_trim()
    assert pm.scratch_reserved_bytes() == 0
    _check_ls(oracle_E("smooth", 512, 16), "trap")           # the pool refills on demand


# ---- pm_local_search_ep_async: TRAP's sigma-permuted copy in a caller-owned
# buffer (allocated once, reused across searches) -- same result as the oracle
@pytest.mark.parametrize("N,M,fam,method", [(128, 8, "smooth", "auto"), (512, 16, "ties", "trap"),
                                            (512, 16, "smooth", "auto"), (240, 8, "noise", "window"),
                                            (200, 10, "smooth", "class")])
def test_local_search_caller_owned_sigma_copy(N, M, fam, method):
    E_np = oracle_E(fam, N, M)
    S = E_np.shape[0]
    if not _supported(method, S):
        pytest.skip(f"{method} does not take S = {S}")
    ref = oracle.local_search(E_np)
    E = dev(E_np)
    nbytes = pm.sigma_copy_bytes(S)
    assert nbytes == 4 * S * (((S - 1 + 48 + 31) // 32) * 32)
    Ep = torch.full((nbytes // 4,), -7, dtype=torch.int32, device=DEV)
    res = torch.zeros(3, dtype=torch.int64, device=DEV)
    for _ in range(2):   # the same buffer twice
        perm = torch.arange(S, dtype=torch.int32, device=DEV)
        pm.local_search_ep_async(E, perm, res, Ep, method=method)
        torch.cuda.synchronize()
        assert res.cpu().tolist() == [ref[4], ref[1], ref[2]]
        assert (perm.cpu().numpy() == ref[0]).all()
    if method in ("auto", "trap"):   # the copy itself: Ep[t][q] = E[t][2q mod m], q < m + 48 cyclic
        m, ld = S - 1, nbytes // 4 // S
        q = np.arange(m + 48)
        assert (Ep.view(S, ld)[:, : m + 48].cpu().numpy() == E_np[:, (2 * q) % m]).all()


def test_local_search_caller_owned_sigma_copy_too_small_rejected():
    E_np = oracle_E("smooth", 128, 8)
    S = E_np.shape[0]
    E = dev(E_np)
    Ep = torch.empty(pm.sigma_copy_bytes(S) // 4 - 4, dtype=torch.int32, device=DEV)
    perm = torch.arange(S, dtype=torch.int32, device=DEV)
    res = torch.zeros(3, dtype=torch.int64, device=DEV)
    with pytest.raises(pm.PMError) as e:
        pm.local_search_ep_async(E, perm, res, Ep, method="trap")
    assert e.value.status == pm.PM_ERR_INVALID


# ---- pm_error_matrix_sigma: E and its sigma-permuted copy in one pass (the
# E kernel's epilogue writes both), and pm_local_search_sigma_async on it
def _sigma_ref(E_np):
    S = E_np.shape[0]
    m = S - 1
    q = np.arange(m + 48)
    return E_np[:, (2 * q) % m]


@pytest.mark.parametrize("N,M,C,fam,plan", [(128, 8, 3, "smooth", 0), (512, 16, 3, "noise", 0), (1024, 16, 3, "smooth", 0),
                                            (512, 16, 3, "smooth", 128002), (512, 16, 3, "ties", 64003),
                                            (256, 16, 1, "smooth", 0), (160, 10, 3, "noise", 0),
                                            (48, 8, 3, "noise", 0), (32, 8, 1, "smooth", 0)])   # m < 48: the extension wraps twice
def test_error_matrix_sigma_parity(N, M, C, fam, plan):
    # plan: sad_plan override (split-K plans accumulate E atomically, so the
    # copy is permuted from E afterwards instead of in the epilogue)
    if plan:
        pm.tuning_set("sad_plan", plan)
    I, T = pair(fam, N, M, C)
    E_np = oracle_E(fam, N, M, C)
    S = E_np.shape[0]
    nbytes = pm.sigma_copy_bytes(S)
    E = torch.full((S, S), -1, dtype=torch.int32, device=DEV)
    Ep = torch.full((nbytes // 4,), -7, dtype=torch.int32, device=DEV)
    pm.error_matrix_sigma(dev(I), dev(T), M, E, Ep)
    torch.cuda.synchronize()
    assert (E.cpu().numpy() == E_np).all()
    ld = nbytes // 4 // S
    assert (Ep.view(S, ld)[:, : S - 1 + 48].cpu().numpy() == _sigma_ref(E_np)).all()
    # the search on the prebuilt copy gives the oracle's replay
    ref = oracle.local_search(E_np)
    perm = torch.arange(S, dtype=torch.int32, device=DEV)
    res = torch.zeros(3, dtype=torch.int64, device=DEV)
    pm.local_search_sigma_async(E, perm, res, Ep)
    torch.cuda.synchronize()
    assert res.cpu().tolist() == [ref[4], ref[1], ref[2]]
    assert (perm.cpu().numpy() == ref[0]).all()


def test_error_matrix_sigma_odd_S_unsupported():
    I, T = pair("smooth", 90, 10, 3)   # S = 81
    S = 81
    E = torch.empty((S, S), dtype=torch.int32, device=DEV)
    Ep = torch.empty(max(pm.sigma_copy_bytes(S) // 4, 1), dtype=torch.int32, device=DEV)
    with pytest.raises(pm.PMError) as e:
        pm.error_matrix_sigma(dev(I), dev(T), 10, E, Ep)
    assert e.value.status == pm.PM_ERR_UNSUPPORTED


def test_sigma_copy_misaligned_rejected():
    E_np = oracle_E("smooth", 128, 8)
    S = E_np.shape[0]
    E = dev(E_np)
    buf = torch.empty(pm.sigma_copy_bytes(S) // 4 + 4, dtype=torch.int32, device=DEV)
    Ep = buf[1:1 + pm.sigma_copy_bytes(S) // 4]   # 4-byte offset: not 16-byte aligned
    perm = torch.arange(S, dtype=torch.int32, device=DEV)
    res = torch.zeros(3, dtype=torch.int64, device=DEV)
    for call in (lambda: pm.local_search_ep_async(E, perm, res, Ep), lambda: pm.local_search_sigma_async(E, perm, res, Ep)):
        with pytest.raises(pm.PMError) as e:
            call()
        assert e.value.status == pm.PM_ERR_INVALID
