"""TRAP phase profile of QUIET rounds only: run the first R rounds, then
profile TRAP (trap_prof, no sparse hand-over) resumed from that state.
Development probe.  Usage: python tools/trap_quiet_prof.py cfg R [knob=value ...]"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402

cfg, R = int(sys.argv[1]), int(sys.argv[2])
c = synth.CONFIGS[cfg]
I, T = synth.config_pair(cfg, "smooth", 0)
E = pm.error_matrix(torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda(), c["M"])
S = E.shape[0]
perm0, *_ = pm.local_search(E, max_rounds=R, allow_not_converged=True)
pm.tuning_set("trap_prof", 1)
for kv in sys.argv[3:]:
    k, v = kv.split("=")
    pm.tuning_set(k, int(v))
pm.tuning_set("ls_sparse", 0)
for rep in range(2):
    perm = perm0.clone()
    per = np.zeros(256, dtype=np.int64)
    r, sw = ctypes.c_int32(0), ctypes.c_int64(0)
    st = pm.lib().pm_local_search_ex(E.data_ptr(), E.stride(0), S, perm.data_ptr(), 0, pm.METHODS["trap"],
                                     ctypes.byref(r), ctypes.byref(sw), per.ctypes.data, 256, None)
ld, stp, bar, nph, pub, t0 = per[192:198]
nph = max(int(nph), 1)
ends = [int(x) for x in per[224:256] if x > 0]
rt = np.diff([int(t0)] + ends) / 1e3
print(f"cfg{cfg} resumed after {R} rounds {sys.argv[3:]}: rounds={r.value} phases={nph} per phase: stage+wait {(ld-stp)/nph:.0f} ns, "
      f"steps {stp/nph:.0f} ns, pub+barrier {bar/nph:.0f} ns; TRAP rounds (us) {np.round(rt, 1).tolist()} swaps {per[:len(rt)].tolist()}",
      flush=True)
