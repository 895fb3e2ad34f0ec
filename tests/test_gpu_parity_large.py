"""GPU parity at BASELINE.json's full sizes: configs 4 (S = 16384, E = 1 GiB,
the bench workload) and 5 (S = 65536, E = 16 GiB), against the CPU oracle run
on the same seeded images, element by element.

* Eq. 1: the whole GPU E equals oracle.error_matrix -- every entry, at
  config 4 and at config 5 (compared in 4096-row chunks).
* Alg. 2: the GPU search on its E gives the oracle replay's r
  (all S slots), rounds, per-round swaps, status and Eq. 2 cost.  The
  GPU's E is bit-identical to the oracle's (asserted first), so the search
  input is the oracle's own.  Config 4: AUTO (TRAP dense rounds + sparse
  rounds, the bench path), TRAP on every round, CLASS (the paper's launch
  structure), the multi-rank protocol emulated at world 8, a max_rounds cut
  + resume, and the host-buffer pipeline.  Config 5: the first five rounds
  (TRAP grid mode from HBM, the hand-over, the first sparse round) from the
  identity, single-GPU and emulated world 8, then every remaining round to
  convergence (the oracle resumes from its own round-5 state: resumption is
  exact, tests/test_oracle_search.py).  Oracle cost on the 16-core GPU host:
  config 4 E 8 s + search 3 s; config 5 E 127 s + ~6.5 s per round.
"""
import time

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import oracle  # noqa: E402
from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

DEV = torch.device("cuda:0")


def dev(x):
    return torch.from_numpy(np.ascontiguousarray(x)).to(DEV)


def _log(msg):
    print(f"[large parity] {msg}", flush=True)


@pytest.fixture(autouse=True)
def _reset_tuning():
    pm.tuning_reset()
    yield
    pm.tuning_reset()


def _assert_E_equal(E_gpu, E_or, chunk=4096):
    S = E_or.shape[0]
    for r0 in range(0, S, chunk):
        r1 = min(S, r0 + chunk)
        got = E_gpu[r0:r1].cpu().numpy()
        bad = np.argwhere(got != E_or[r0:r1])
        assert bad.size == 0, f"E differs at {len(bad)} entries, first (u, v) = {tuple(bad[0] + [r0, 0])}"


def _assert_search(got, ref, E_or, what):
    perm, rounds, swaps, per, st = got
    r_ref, k_ref, s_ref, per_ref, st_ref = ref
    p = perm.cpu().numpy() if hasattr(perm, "cpu") else perm
    assert (p == r_ref).all(), f"{what}: final r differs at {int((p != r_ref).sum())} slots"
    assert (rounds, swaps, st) == (k_ref, s_ref, st_ref), (what, (rounds, swaps, st), (k_ref, s_ref, st_ref))
    if per is not None:
        assert (np.asarray(per) == per_ref[: len(per)]).all(), (what, per, per_ref)


# --------------------------------------------------------------- config 4 --
@pytest.fixture(scope="module")
def cfg4():
    I, T = synth.config_pair(4, "smooth", 0)
    t = time.perf_counter()
    E_or = oracle.error_matrix(I, T, 16)
    _log(f"config 4 oracle E {time.perf_counter() - t:.1f} s")
    E_gpu = pm.error_matrix(dev(I), dev(T), 16)
    t = time.perf_counter()
    ref = oracle.local_search(E_or)
    _log(f"config 4 oracle Alg. 2 {time.perf_counter() - t:.1f} s: rounds {ref[1]} swaps {ref[2]}")
    yield I, T, E_or, E_gpu, ref
    del E_gpu
    torch.cuda.empty_cache()


def test_cfg4_error_matrix_every_entry(cfg4):
    I, T, E_or, E_gpu, ref = cfg4
    _assert_E_equal(E_gpu, E_or)


@pytest.mark.parametrize("method", ["auto", "trap", "class"])
def test_cfg4_local_search(cfg4, method):
    I, T, E_or, E_gpu, ref = cfg4
    got = pm.local_search(E_gpu, method=method)
    _assert_search(got, ref, E_or, f"config 4 {method}")
    assert pm.cost(E_gpu, got[0]) == oracle.cost(E_or, ref[0])


def test_cfg4_caller_owned_sigma_copy(cfg4):
    # pm_local_search_ep_async: the 1 GiB sigma-permuted copy in a torch buffer
    I, T, E_or, E_gpu, ref = cfg4
    S = E_gpu.shape[0]
    Ep = torch.empty(pm.sigma_copy_bytes(S) // 4, dtype=torch.int32, device=DEV)
    res = torch.zeros(3, dtype=torch.int64, device=DEV)
    perm = torch.arange(S, dtype=torch.int32, device=DEV)
    pm.local_search_ep_async(E_gpu, perm, res, Ep)
    st, rounds, swaps = res.cpu().tolist()
    _assert_search((perm, rounds, swaps, None, st), ref, E_or, "config 4 auto, caller-owned sigma copy")


def test_cfg4_error_matrix_sigma(cfg4):
    # E and its sigma-permuted copy in one pass (the bench's Step 2), then the
    # search on that copy: E equal to the oracle's, the copy equal to its
    # permutation, the search equal to the oracle's replay
    I, T, E_or, E_gpu, ref = cfg4
    S = E_or.shape[0]
    nbytes = pm.sigma_copy_bytes(S)
    E = torch.empty((S, S), dtype=torch.int32, device=DEV)
    Ep = torch.empty(nbytes // 4, dtype=torch.int32, device=DEV)
    pm.error_matrix_sigma(dev(I), dev(T), 16, E, Ep)
    _assert_E_equal(E, E_or)
    ld = nbytes // 4 // S
    q = np.arange(S - 1 + 48)
    cols = (2 * q) % (S - 1)
    Epv = Ep.view(S, ld)
    for r0 in range(0, S, 4096):
        assert (Epv[r0:r0 + 4096, : S - 1 + 48].cpu().numpy() == E_or[r0:r0 + 4096][:, cols]).all()
    res = torch.zeros(3, dtype=torch.int64, device=DEV)
    perm = torch.arange(S, dtype=torch.int32, device=DEV)
    pm.local_search_sigma_async(E, perm, res, Ep)
    st, rounds, swaps = res.cpu().tolist()
    _assert_search((perm, rounds, swaps, None, st), ref, E_or, "config 4 auto on the fused sigma copy")
    del E, Ep
    torch.cuda.empty_cache()


def test_cfg4_trap_every_round(cfg4):
    # the sparse hand-over off: every round (incl. the quiet ones) on TRAP
    I, T, E_or, E_gpu, ref = cfg4
    with pm.tuning(ls_sparse=0):
        got = pm.local_search(E_gpu, method="trap")
    _assert_search(got, ref, E_or, "config 4 trap, no sparse rounds")


def test_cfg4_multi_rank_emulated_world8(cfg4):
    I, T, E_or, E_gpu, ref = cfg4
    out, rounds, swaps = pm.local_search_multi_emulated(E_gpu, 8)
    _assert_search((out, rounds, swaps, None, 0), ref, E_or, "config 4 world 8 (emulated)")


def test_cfg4_sharded_emulated_world8(cfg4):
    # E row-sharded over 8 ranks (separate shard buffers), read through the
    # owner's shard: the whole search on TRAP rounds, same result
    I, T, E_or, E_gpu, ref = cfg4
    out, rounds, swaps = pm.local_search_sharded_emulated(E_gpu, 8)
    _assert_search((out, rounds, swaps, None, 0), ref, E_or, "config 4 world 8 row-sharded (emulated)")


def test_cfg4_max_rounds_then_resume(cfg4):
    I, T, E_or, E_gpu, ref = cfg4
    cut = oracle.local_search(E_or, max_rounds=3)
    got = pm.local_search(E_gpu, max_rounds=3, allow_not_converged=True)
    _assert_search(got, cut, E_or, "config 4 first 3 rounds")
    rest = oracle.local_search(E_or, r0=cut[0])
    got2 = pm.local_search(E_gpu, perm=got[0])
    _assert_search(got2, rest, E_or, "config 4 resumed after 3 rounds")
    assert (got2[0].cpu().numpy() == ref[0]).all()


def test_cfg4_photomosaic_host(cfg4):
    # the end-to-end call the bench's e2e number uses (host images -> host r)
    I, T, E_or, E_gpu, ref = cfg4
    perm, rounds, swaps, c = pm.photomosaic_host(I, T, 16)
    assert (perm == ref[0]).all() and (rounds, swaps) == (ref[1], ref[2])
    assert c == oracle.cost(E_or, ref[0])


# --------------------------------------------------------------- config 5 --
@pytest.fixture(scope="module")
def cfg5():
    I, T = synth.config_pair(5, "smooth", 0)
    t = time.perf_counter()
    E_or = oracle.error_matrix(I, T, 16)                      # 16 GiB on the host
    _log(f"config 5 oracle E {time.perf_counter() - t:.1f} s")
    E_gpu = pm.error_matrix(dev(I), dev(T), 16)
    t = time.perf_counter()
    ref5 = oracle.local_search(E_or, max_rounds=5)
    _log(f"config 5 oracle Alg. 2, 5 rounds {time.perf_counter() - t:.1f} s: per round {ref5[3].tolist()}")
    yield I, T, E_or, E_gpu, ref5
    del E_gpu
    torch.cuda.empty_cache()


def test_cfg5_error_matrix_every_entry(cfg5):
    I, T, E_or, E_gpu, ref5 = cfg5
    _assert_E_equal(E_gpu, E_or)


def test_cfg5_local_search_first_rounds(cfg5):
    # rounds 0-3 dense (TRAP, grid mode, E from HBM), hand-over, round 4 sparse
    I, T, E_or, E_gpu, ref5 = cfg5
    got = pm.local_search(E_gpu, max_rounds=5, allow_not_converged=True)
    _assert_search(got, ref5, E_or, "config 5 first 5 rounds")


def test_cfg5_multi_rank_emulated_world8_first_rounds(cfg5):
    I, T, E_or, E_gpu, ref5 = cfg5
    out, rounds, swaps = pm.local_search_multi_emulated(E_gpu, 8, max_rounds=5)
    _assert_search((out, rounds, swaps, None, 3), ref5, E_or, "config 5 world 8 (emulated), 5 rounds")


def test_cfg5_sharded_emulated_world8_first_rounds(cfg5):
    # config 5's E (16 GiB) in 8 row shards of 2 GiB + their permuted copies
    I, T, E_or, E_gpu, ref5 = cfg5
    out, rounds, swaps = pm.local_search_sharded_emulated(E_gpu, 8, max_rounds=5)
    _assert_search((out, rounds, swaps, None, 3), ref5, E_or, "config 5 world 8 row-sharded (emulated), 5 rounds")


def test_cfg5_local_search_to_convergence(cfg5):
    I, T, E_or, E_gpu, ref5 = cfg5
    t = time.perf_counter()
    rest = oracle.local_search(E_or, r0=ref5[0])
    _log(f"config 5 oracle Alg. 2 rounds 5.. {time.perf_counter() - t:.1f} s: per round {rest[3].tolist()}")
    got = pm.local_search(E_gpu)
    per_all = np.concatenate([ref5[3], rest[3]])
    ref_all = (rest[0], ref5[1] + rest[1], ref5[2] + rest[2], per_all, rest[4])
    _assert_search(got, ref_all, E_or, "config 5 all rounds")
    assert pm.cost(E_gpu, got[0]) == oracle.cost(E_or, rest[0])
    out, rounds, swaps = pm.local_search_multi_emulated(E_gpu, 8)
    _assert_search((out, rounds, swaps, None, 0), ref_all, E_or, "config 5 world 8 (emulated), all rounds")
