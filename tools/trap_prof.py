"""TRAP phase profile (trap_prof=1): block 0 / warp 0 time split per phase
into staging (state + E runs), class steps, write-back + grid barrier, and
the duration of every TRAP round.  Development probe.
Usage: PM_TRAP_PROF=1 [PM_TRAP_SPEC=0|1|2] python tools/trap_prof.py [cfgs]"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import _devknobs  # noqa: E402
if os.environ.get("PM_LIB"):   # a development build of the library (knockout experiments)
    pm.LIB_PATH = os.environ["PM_LIB"]
_devknobs.apply(pm)

pm.tuning_set("trap_prof", int(os.environ.get("PM_TRAP_PROF", "1")))
cfgs = [int(c) for c in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["1", "2", "3"])]
for cfg in cfgs:
    c = synth.CONFIGS[cfg]
    I, T = synth.config_pair(cfg, "smooth", 0)
    E = pm.error_matrix(torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda(), c["M"])
    S = E.shape[0]
    for rep in range(2):
        perm = torch.arange(S, dtype=torch.int32, device="cuda")
        per = np.zeros(256, dtype=np.int64)
        r, sw = ctypes.c_int32(0), ctypes.c_int64(0)
        st = pm.lib().pm_local_search_ex(E.data_ptr(), E.stride(0), S, perm.data_ptr(), int(os.environ.get("PM_MAX_ROUNDS", "0")), pm.METHODS["trap"],
                                         ctypes.byref(r), ctypes.byref(sw), per.ctypes.data, 256, None)
    ld, stp, bar, nph, pub, t0 = per[192:198]
    fw, iss, cpw = per[198:201]
    nph = max(int(nph), 1)
    ends = [int(x) for x in per[224:256] if x > 0]
    rt = np.diff([int(t0)] + ends) / 1e3
    print(f"cfg{cfg} S={S} st={st} rounds={r.value} phases={nph} per phase: stage {ld/nph:.0f} ns, "
          f"[flag wait {fw/nph:.0f}, state+issue {iss/nph:.0f}, copy wait {cpw/nph:.0f}] steps {stp/nph:.0f} ns, publish {pub/nph:.0f} ns, publish+barrier {bar/nph:.0f} ns; total "
          f"{(ld+stp+bar)/1e6:.3f} ms; TRAP rounds (us) {np.round(rt, 1).tolist()} swaps {per[:len(rt)].tolist()}",
          flush=True)
