"""Small workload for compute-sanitizer: every kernel of libpm once (config 1
and a ragged odd shape), results checked against the oracle.  Tuning knobs
from the environment (tools/_devknobs.py); METHODS, MULTI select the search
paths.  Usage: compute-sanitizer --tool memcheck python tools/sanitize_run.py"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import _devknobs  # noqa: E402
_devknobs.apply(pm)

for (N, M, C) in [(128, 8, 3), (90, 10, 3)]:
    I, T = synth.make_pair("smooth", N, M, C, seed=1)
    dI, dT = torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda()
    assert (pm.histogram_match(dI, dT).cpu().numpy() == oracle.histogram_match(I, T)).all()
    E = pm.error_matrix(dI, dT, M)
    Er = oracle.error_matrix(I, T, M)
    assert (E.cpu().numpy() == Er).all()
    ref = oracle.local_search(Er)
    methods = os.environ.get("METHODS", "trap,window,class,walk").split(",")
    perm = None
    for meth in methods:
        if meth == "trap" and (E.shape[0] < 256 or E.shape[0] % 2):
            continue
        if meth == "window" and E.shape[0] > 2048:
            continue
        perm, rounds, swaps, per, st = pm.local_search(E, method=meth)
        assert (perm.cpu().numpy() == ref[0]).all() and rounds == ref[1], meth
    if os.environ.get("MULTI") and E.shape[0] >= 256 and E.shape[0] % 2 == 0:
        out, rounds, swaps = pm.local_search_multi_emulated(E, int(os.environ["MULTI"]))
        assert (out.cpu().numpy() == ref[0]).all() and rounds == ref[1], "multi"
    if perm is None:
        continue
    c = pm.cost(E, perm)
    R = pm.render(dI, M, perm)
    t = pm.pack_tiles(dI, M)
torch.cuda.synchronize()
print("sanitize workload ok")
