import sys
"""Small workload for compute-sanitizer: every kernel of libpm once (configs 1
and a ragged odd shape), results checked against the oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle
from paper_conf_ipps_yangin17_b200 import pm, synth
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import _devknobs  # noqa: E402
_devknobs.apply(pm)
for (N, M, C) in [(128, 8, 3), (90, 10, 3)]:
    I, T = synth.make_pair("smooth", N, M, C, seed=1)
    dI, dT = torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda()
    E = pm.error_matrix(dI, dT, M)
    Er = oracle.error_matrix(I, T, M)
    assert (E.cpu().numpy() == Er).all()
    ref = oracle.local_search(Er)
    methods = os.environ.get("METHODS", "trap,window,class,walk").split(",")
    perm = None
    for meth in methods:
        if (meth == "trap" and (E.shape[0] < 256 or E.shape[0] % 2)):
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
print("sanitize workload ok")
