"""Cost of the multi-GPU TRAP protocol on one GPU: pm_local_search_multi_emulated
with every rank of a world in one launch (the GPU's SMs split among the ranks),
against world = 1.  Development probe.  Usage:
python tools/multi_emul_bench.py [cfgs] [worlds] [multi|sharded]
(sharded: pm_local_search_sharded_emulated, E split into row-shard buffers;
its time includes the shard copies and the permuted-row builds)"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import _devknobs  # noqa: E402
_devknobs.apply(pm)

cfgs = [int(c) for c in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["3", "4"])]
worlds = [int(w) for w in (sys.argv[2].split(",") if len(sys.argv) > 2 else ["1", "2", "4", "8"])]
mode = sys.argv[3] if len(sys.argv) > 3 else "multi"
run = pm.local_search_sharded_emulated if mode == "sharded" else pm.local_search_multi_emulated
for cfg in cfgs:
    c = synth.CONFIGS[cfg]
    I, T = synth.config_pair(cfg, "smooth", 0)
    E = pm.error_matrix(torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda(), c["M"])
    S = E.shape[0]
    for w in worlds:
        ts = []
        for rep in range(3):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            perm, rounds, swaps = run(E, w)
            torch.cuda.synchronize()
            ts.append(time.perf_counter() - t0)
        print(f"{mode} cfg{cfg} S={S} world={w} {min(ts) * 1e3:9.3f} ms rounds={rounds} swaps={swaps}", flush=True)
