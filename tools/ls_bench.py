"""Quick timing of the local-search methods (device-resident E) per config.
Not the contract bench -- a development probe.  Usage: python tools/ls_bench.py [cfgs] [methods]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import _devknobs  # noqa: E402
if os.environ.get("PM_LIB"):   # a development build of the library
    pm.LIB_PATH = os.environ["PM_LIB"]
_devknobs.apply(pm)

cfgs = [int(c) for c in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["1", "2", "3"])]
methods = sys.argv[2].split(",") if len(sys.argv) > 2 else ["trap", "window"]
reps = max(1, int(os.environ.get("REPS", "5")))
for cfg in cfgs:
    c = synth.CONFIGS[cfg]
    I, T = synth.config_pair(cfg, "smooth", 0)
    E = pm.error_matrix(torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda(), c["M"])
    S = E.shape[0]
    ref = None
    for m in methods:
        ts = []
        res_t = torch.zeros(3, dtype=torch.int64, device="cuda")
        for r in range(reps + 1):
            perm = torch.arange(S, dtype=torch.int32, device="cuda")
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            pm.local_search_async(E, perm, res_t, method=m)
            b.record()
            b.synchronize()
            if r:
                ts.append(a.elapsed_time(b))
        perm = torch.arange(S, dtype=torch.int32, device="cuda")
        _, rounds, swaps, per, st = pm.local_search(E, perm, method=m)
        res = (rounds, swaps, perm.cpu().numpy().tobytes())
        same = "" if ref is None else ("same" if res == ref else "DIFFERENT")
        ref = ref or res
        ts.sort()
        print(f"cfg{cfg} S={S} {m:7s} {ts[len(ts)//2]:9.3f} ms [min {ts[0]:.3f} max {ts[-1]:.3f}] rounds={rounds} swaps={swaps} "
              f"ns/class-step={ts[len(ts)//2]*1e6/(rounds*(S-1)):.0f} per_round={per.tolist()} {same}", flush=True)
