"""Time pm_optimal_assignment (GPU eps-scaling auction) on the BASELINE
configs; compare its cost with Algorithm 2's (the paper's Table III/IV
comparison of the optimization and approximation algorithms)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import _devknobs  # noqa: E402
_devknobs.apply(pm)

cfgs = [int(x) for x in (sys.argv[1:] or ["1", "2", "3"])]
fams = os.environ.get("FAMS", "smooth").split(",")
for cfg in cfgs:
    for fam in fams:
        c = synth.CONFIGS[cfg]
        I, T = synth.config_pair(cfg, fam, seed=0)
        Id, Td = torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda()
        E = pm.error_matrix(Id, Td, c["M"])
        S = E.shape[0]
        perm, rounds_ls, swaps, _, _ = pm.local_search(E)
        c_ls = pm.cost(E, perm)
        times = []
        for rep in range(int(os.environ.get("REPS", "3"))):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            p2, c_opt, rounds, price = pm.optimal_assignment(E)
            torch.cuda.synchronize()
            times.append(time.perf_counter() - t0)
        print(json.dumps({"cfg": cfg, "fam": fam, "S": S, "auction_s": min(times), "bid_rounds": rounds,
                          "cost_opt": c_opt, "cost_ls": c_ls, "ls_over_opt": c_ls / max(c_opt, 1),
                          "env": {k: v for k, v in os.environ.items() if k.startswith("PM_AUCTION")}}),
              flush=True)
