"""Whole-search timing with the library's scratch copy vs a caller-owned
sigma-permuted copy (pm_local_search_ep_async).  Development probe:
python tools/ep_bench.py [cfg]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 5
c = synth.CONFIGS[cfg]
I, T = synth.config_pair(cfg, "smooth", 0)
E = pm.error_matrix(torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda(), c["M"])
S = E.shape[0]
Ep = torch.empty(pm.sigma_copy_bytes(S) // 4, dtype=torch.int32, device="cuda")
res = torch.zeros(3, dtype=torch.int64, device="cuda")
for variant in ("scratch", "caller"):
    ts = []
    for r in range(5):
        perm = torch.arange(S, dtype=torch.int32, device="cuda")
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        if variant == "scratch":
            pm.local_search_async(E, perm, res)
        else:
            pm.local_search_ep_async(E, perm, res, Ep)
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b))
    print(f"cfg{cfg} S={S} {variant:8s} ms per search {[round(t, 1) for t in ts]} result {res.cpu().tolist()}", flush=True)
