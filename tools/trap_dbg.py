"""TRAP parity sweep over sizes/variants against the oracle (development probe)."""
import itertools
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_ipps_yangin17_b200 import pm, synth  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import _devknobs  # noqa: E402
_devknobs.apply(pm)

sizes = [(int(a), int(b)) for a, b in (x.split("/") for x in sys.argv[1].split(","))]
for (N, M) in sizes:
    I, T = synth.make_pair("smooth", N, M, 3, seed=0)
    E_np = oracle.error_matrix(I, T, M)
    ref = oracle.local_search(E_np)
    E = torch.from_numpy(E_np).cuda()
    for vec, cm, v in itertools.product(["1", "0"], ["0"], ["0", "1"]):
        os.environ.update(PM_TRAP_VEC=vec, PM_TRAP_CLUSTER=cm, PM_TRAP_V=v, PM_LS_SPARSE="0")
        out, r, sw, per, st = pm.local_search(E, method="trap")
        ok = (out.cpu().numpy() == ref[0]).all() and (r, sw) == (ref[1], ref[2])
        print(N, M, E_np.shape[0], "vec", vec, "v", v, "OK" if ok else f"BAD round0 {per[0]} vs {ref[3][0]}", flush=True)
