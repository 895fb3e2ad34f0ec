"""Per-round breakdown of PM_LS_PAIRWIN (needs tools/libpm_prof.so built with -DPM_LS_PROFILE)."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_yangin17_b200 import pm, synth
pm.LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libpm_prof.so")
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
c = synth.CONFIGS[cfg]
I, T = synth.config_pair(cfg, "smooth", 0)
E = pm.error_matrix(torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda(), c["M"])
S = E.shape[0]
L = pm.lib()
for rep in range(2):
    full = np.zeros(1024, dtype=np.int64)
    perm = torch.arange(S, dtype=torch.int32, device="cuda")
    r_, s_ = ctypes.c_int32(0), ctypes.c_int64(0)
    L.pm_local_search_ex(E.data_ptr(), E.stride(0), S, perm.data_ptr(), 0, 4, ctypes.byref(r_), ctypes.byref(s_), full.ctypes.data, 1024, pm._stream())
rounds = r_.value
prev_end = None
for r in range(rounds):
    gs, ge = full[768 + r], full[832 + r]
    gap = (gs - prev_end) / 1e3 if prev_end else float('nan')
    prev_end = ge
    print(f"round {r}: swaps={full[r]:5d} cta_cycles={full[512+r]:9d} patch={full[576+r]:8d} classes={full[640+r]:9d} wait={full[704+r]:7d} "
          f"cta_us={(ge-gs)/1e3:8.1f} gap_before_us={gap:6.1f}")
