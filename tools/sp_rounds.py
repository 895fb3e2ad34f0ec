import sys
import os
"""Per-round timing of the sparse rounds (needs tools/libpm_prof.so built
with -DPM_LS_PROFILE).  Development probe: python tools/sp_rounds.py cfg method"""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_ipps_yangin17_b200 import pm, synth
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import _devknobs  # noqa: E402
_devknobs.apply(pm)
pm.LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), os.environ.get("PMLIB", "libpm_prof.so"))
cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
method = sys.argv[2] if len(sys.argv) > 2 else "window"
c = synth.CONFIGS[cfg]
I, T = synth.config_pair(cfg, "smooth", 0)
E = pm.error_matrix(torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda(), c["M"])
S = E.shape[0]
L = pm.lib()
for rep in range(3):
    full = np.zeros(1024, dtype=np.int64)
    perm = torch.arange(S, dtype=torch.int32, device="cuda")
    r_, s_ = ctypes.c_int32(0), ctypes.c_int64(0)
    torch.cuda.synchronize()
    L.pm_local_search_ex(E.data_ptr(), E.stride(0), S, perm.data_ptr(), 0, pm.METHODS[method], ctypes.byref(r_),
                         ctypes.byref(s_), full.ctypes.data, 1024, pm._stream())
rounds = r_.value
prev_end = None
for r in range(rounds):
    dur = full[512 + r]
    if full[832 + r] == 0:
        print(f"round {r}: swaps={full[r]} (dense stage)")
        continue
    gap = (full[832 + r] - prev_end) if prev_end else (full[832 + r] - full[1023] if full[1023] else 0)
    prev_end = full[896 + r]
    print(f"round {r}: swaps={full[r]:6d} walk={dur/1e3:8.1f} us gap-before(scan+launch)={gap/1e3:7.1f} us "
          f"windows={full[576 + r]} applies={full[640 + r]} dirty_end={full[704 + r]} stamped={full[768 + r]} "
          f"| t0 cycles: prologue={full[960 + r]} eval={full[448 + r]} barrier={full[384 + r]} apply={full[320 + r]} [dirty-issue={full[256 + r]} stamped-issue={full[192 + r]} dirty-wait={full[128 + r]}]")
