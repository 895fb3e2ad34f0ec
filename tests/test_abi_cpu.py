"""CPU-side checks of the C-ABI boundary (no GPU needed, no compute calls):
libpm.so loads, exports every function include/pm.h declares, and its
host-only entry points (pm_num_colors, pm_edge_coloring, pm_tile_stride,
pm_status_string) behave -- the edge groups checked against the paper's
printed K_16 table and against the oracle's colouring."""
import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "pm.h")


def _declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(pm_[A-Za-z0-9_]+)\s*\(", src)))


@pytest.fixture(scope="module")
def pm():
    from paper_conf_ipps_yangin17_b200 import pm as _pm
    if not os.path.exists(_pm.LIB_PATH):
        import __graft_entry__
        __graft_entry__.build()
    return _pm


def test_header_declares_the_boundary():
    names = _declared_functions()
    for required in ("pm_error_matrix", "pm_edge_coloring", "pm_local_search", "pm_cost"):
        assert required in names


def test_library_exports_every_declared_symbol(pm):
    L = pm.lib()
    missing = [n for n in _declared_functions() if not hasattr(L, n)]
    assert not missing, f"declared in pm.h but not exported: {missing}"
    out = subprocess.run(["nm", "-D", "--defined-only", pm.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (pm_[A-Za-z0-9_]+)$", out, flags=re.M))
    assert set(_declared_functions()) <= exported
    # the python binding covers the whole ABI
    assert {n for n, _, _ in pm._SIGS} == set(_declared_functions())


def test_library_is_sm100a(pm):
    out = subprocess.run(["cuobjdump", "--list-elf", pm.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_status_strings(pm):
    for s in range(7):
        assert pm.status_string(s).startswith("PM_")
    assert "TIMEOUT" in pm.status_string(pm.PM_ERR_TIMEOUT)


def test_tuning_overrides_are_explicit(pm):
    # development overrides go through the ABI only (never the environment):
    # unknown names are rejected, known ones accepted, reset restores defaults
    L = pm.lib()
    assert L.pm_tuning_set(b"no_such_knob", 1) == pm.PM_ERR_INVALID
    assert L.pm_tuning_set(None, 1) == pm.PM_ERR_INVALID
    for name in ("trap_variant", "trap_cluster", "ls_sparse_T", "ls_cwalk", "auction_gs"):
        assert L.pm_tuning_set(name.encode(), 1) == pm.PM_OK
    pm.tuning_reset()
    with pytest.raises(pm.PMError):
        pm.tuning_set("PM_TRAP_V", 3)      # the round-1 environment names are gone


def test_release_library_reads_no_environment():
    # the library's own sources never read the environment: behaviour cannot
    # depend on the caller's environment (tuning overrides are explicit ABI
    # calls; the static CUDA runtime still reads its own CUDA_* variables)
    csrc = os.path.join(ROOT, "paper_conf_ipps_yangin17_b200", "csrc")
    for f in os.listdir(csrc):
        src = open(os.path.join(csrc, f)).read()
        assert "getenv(" not in src and "std::getenv" not in src, f


def test_retired_methods_rejected(pm):
    # PM_LS_* 2 and 4 (round-1 single-CTA / pair-window methods) are retired
    assert set(pm.METHODS.values()) == {0, 1, 3, 5, 6}


def test_tile_stride(pm):
    assert pm.tile_stride(16, 3) == 768
    assert pm.tile_stride(8, 3) == 192
    assert pm.tile_stride(5, 1) == 64
    assert pm.tile_stride(0, 3) == 0


def test_edge_coloring_matches_printed_k16(pm, golden_dir):
    from tests.test_oracle_coloring import _read_golden
    gold = _read_golden(os.path.join(golden_dir, "k16_groups.txt"))
    got = pm.edge_coloring(16)
    assert pm.num_colors(16) == 15 and got.shape == (15, 8, 2)
    for i in range(1, 16):
        assert [tuple(map(int, p)) for p in got[i - 1]] == gold[i], f"P_{i}"


@pytest.mark.parametrize("S", [2, 3, 4, 5, 16, 17, 64, 255, 256, 1024])
def test_edge_coloring_matches_oracle(pm, S):
    import oracle
    assert pm.num_colors(S) == oracle.num_colors(S)
    assert (pm.edge_coloring(S) == oracle.edge_coloring(S)).all()


def test_edge_coloring_rejects_bad_ranges(pm):
    out = np.zeros(16, dtype=np.int32)
    assert pm.lib().pm_edge_coloring(1, 0, 0, out.ctypes.data) == pm.PM_ERR_INVALID
    assert pm.lib().pm_edge_coloring(16, 3, 2, out.ctypes.data) == pm.PM_ERR_INVALID
    assert pm.lib().pm_edge_coloring(16, 0, 16, out.ctypes.data) == pm.PM_ERR_INVALID
    part = pm.edge_coloring(16, 4, 6)
    assert (part == pm.edge_coloring(16)[4:6]).all()


def test_multi_rank_entry_points_validate_before_any_launch(pm):
    # host-side checks of the multi-GPU boundary (no device needed)
    import ctypes
    L = pm.lib()
    S = 1024
    ws = pm.trap_workspace_bytes(S)
    assert ws >= 5 * 4 * S and pm.trap_workspace_bytes(1) == 0
    assert pm.trap_workspace_bytes(4 * S) > ws
    P2 = ctypes.c_void_p * 2
    fake = 0x1000
    # null E / tables / result, rank outside the world, ld_E < S
    assert L.pm_local_search_multi_async(None, S, S, P2(fake, fake), P2(fake, fake), 0, 2, 0, fake, None) == pm.PM_ERR_INVALID
    assert L.pm_local_search_multi_async(fake, S, S, None, P2(fake, fake), 0, 2, 0, fake, None) == pm.PM_ERR_INVALID
    assert L.pm_local_search_multi_async(fake, S, S, P2(fake, fake), P2(fake, fake), 2, 2, 0, fake, None) == pm.PM_ERR_INVALID
    assert L.pm_local_search_multi_async(fake, S - 1, S, P2(fake, fake), P2(fake, fake), 0, 2, 0, fake, None) == pm.PM_ERR_INVALID
    assert L.pm_local_search_multi_async(fake, S, S, P2(fake, None), P2(fake, fake), 0, 2, 0, fake, None) == pm.PM_ERR_INVALID
    assert L.pm_trap_workspace_reset(None, S, None) == pm.PM_ERR_INVALID
    assert L.pm_local_search_multi_emulated(None, S, S, fake, 2, 0, None, None, None) == pm.PM_ERR_INVALID


def test_sharded_entry_points_validate_before_any_launch(pm):
    # host-side checks of the row-sharded multi-GPU boundary (no device needed)
    import ctypes
    L = pm.lib()
    S = 1024
    full = pm.trap_workspace_bytes(S)
    half = pm.trap_workspace_bytes_sharded(S, S // 2)
    assert half >= full + 4 * (S // 2) * (S - 1)          # + this rank's permuted rows
    assert pm.trap_workspace_bytes_sharded(S, S) > half
    assert pm.trap_workspace_bytes_sharded(S, S + 1) == 0 and pm.trap_workspace_bytes_sharded(S, -1) == 0
    P2 = ctypes.c_void_p * 2
    RB = ctypes.c_int32 * 3
    fake = 0x1000
    ok = (P2(fake, fake), RB(0, S // 2, S), S, S, P2(fake, fake), P2(fake, fake), 0, 2, 0, fake, None)

    def call(**kw):
        a = list(ok)
        for i, v in kw.items():
            a[int(i[1:])] = v
        return L.pm_local_search_sharded_async(*a)

    assert call(a0=None) == pm.PM_ERR_INVALID                       # no shard table
    assert call(a1=None) == pm.PM_ERR_INVALID                       # no row bounds
    assert call(a1=RB(0, S // 2, S - 2)) == pm.PM_ERR_INVALID       # bounds do not end at S
    assert call(a1=RB(1, S // 2, S)) == pm.PM_ERR_INVALID           # ... nor start at 0
    assert call(a1=RB(0, S, S // 2)) == pm.PM_ERR_INVALID           # decreasing
    assert call(a0=P2(fake, None)) == pm.PM_ERR_INVALID             # non-empty shard without a pointer
    assert call(a2=S - 1) == pm.PM_ERR_INVALID                      # ld_E < S
    assert call(a6=2) == pm.PM_ERR_INVALID                          # rank outside the world
    assert call(a5=P2(fake, None)) == pm.PM_ERR_INVALID             # missing workspace
    assert call(a9=None) == pm.PM_ERR_INVALID                       # no result
    assert L.pm_local_search_sharded_emulated(None, S, S, fake, 2, 0, None, None, None) == pm.PM_ERR_INVALID
    assert L.pm_local_search_sharded_emulated(fake, S, S, fake, 9, 0, None, None, None) == pm.PM_ERR_INVALID
    C2 = ctypes.c_void_p * 2
    assert L.pm_cost_sharded_async(None, RB(0, S // 2, S), 2, S, S, fake, fake, None) == pm.PM_ERR_INVALID
    assert L.pm_cost_sharded_async(C2(fake, fake), RB(0, S // 2, S - 1), 2, S, S, fake, fake, None) == pm.PM_ERR_INVALID
    assert L.pm_cost_sharded_async(C2(fake, None), RB(0, S // 2, S), 2, S, S, fake, fake, None) == pm.PM_ERR_INVALID
    assert L.pm_cost_sharded_async(C2(fake, fake), RB(0, S // 2, S), 2, S - 1, S, fake, fake, None) == pm.PM_ERR_INVALID
    assert L.pm_cost_sharded_async(C2(fake, fake), RB(0, S // 2, S), 9, S, S, fake, fake, None) == pm.PM_ERR_INVALID

