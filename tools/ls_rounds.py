import sys
import os
"""Per-round cycle breakdown of the WINDOW search (needs tools/libpm_prof.so,
built with -DPM_LS_PROFILE).  Development probe."""
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
for rep in range(2):
    perm = torch.arange(S, dtype=torch.int32, device="cuda")
    _, rounds, swaps, per, st = pm.local_search(E, perm, method=method, log_len=1024)
full = np.zeros(1024, dtype=np.int64)
L = pm.lib()
perm = torch.arange(S, dtype=torch.int32, device="cuda")
r_, s_ = ctypes.c_int32(0), ctypes.c_int64(0)
L.pm_local_search_ex(E.data_ptr(), E.stride(0), S, perm.data_ptr(), 0, pm.METHODS[method], ctypes.byref(r_), ctypes.byref(s_), full.ctypes.data, 1024, pm._stream())
tot = full[512:512 + rounds].sum()
for r in range(rounds):
    cyc = full[512 + r]
    print(f"round {r}: swaps={full[r]:6d} cycles={cyc:9d} ({100*cyc/tot:4.1f}%) apply_steps={full[640+r]:5d} spec_batches={full[768+r]:5d} cyc/class={cyc/(S-1):7.0f} fill={full[896+r]} spec={full[928+r]} apply(incl spec)={full[960+r]}")
for r in range(rounds):
    print(f"  round {r}: warp1 eval+swap={full[256+r]} exch={full[272+r]} barrier={full[288+r]} | thread0 eval+swap={full[320+r]} exch={full[336+r]} barrier={full[352+r]}")
print("total cycles", tot, "=", tot / 1.965e9 * 1e3, "ms at 1965 MHz")
