import sys
"""NEXT-1 (SURVEY §8(f)): the paper's own workload grid -- grayscale (C = 1)
N in {512, 1024, 2048} x S in {16^2, 32^2, 64^2} (Tables II-IV, P:346-422) --
timed on this GPU with the same kernels: Step 2 (E) and Step 3 (Alg. 2, AUTO
method), device-resident synthetic 'smooth' images, CUDA events, median of 3.
Prints a markdown table with the paper's K40 times beside ours (context: the
paper used histogram-matched SIPI photographs; round counts differ)."""
import os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_yangin17_b200 import pm, synth
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import _devknobs  # noqa: E402
_devknobs.apply(pm)

# Table II (E, GPU s), Table III (approx. rearrangement, GPU s), Table IV (approx total, GPU s)
PAPER = {(512, 16): (0.005, 0.012, 0.017), (512, 32): (0.017, 0.063, 0.081), (512, 64): (0.107, 0.343, 0.450),
         (1024, 16): (0.020, 0.011, 0.033), (1024, 32): (0.077, 0.069, 0.148), (1024, 64): (0.269, 0.372, 0.643),
         (2048, 16): (0.079, 0.014, 0.098), (2048, 32): (0.316, 0.065, 0.386), (2048, 64): (1.230, 0.352, 1.587)}
print("| N | grid | tile px | E ours | E K40 (Tab. II) | Alg. 2 ours (method, rounds) | Alg. 2 K40 (Tab. III) | total ours | total K40 (Tab. IV) |")
print("|---|---|---|---|---|---|---|---|---|")
for (N, g), (pe, pls, ptot) in PAPER.items():
    M = N // g
    S = g * g
    I, T = synth.make_pair("smooth", N, M, 1, seed=0)
    dI, dT = torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda()
    E = torch.empty((S, S), dtype=torch.int32, device="cuda")
    te, tl = [], []
    for rep in range(4):
        perm = torch.arange(S, dtype=torch.int32, device="cuda")
        res = torch.zeros(3, dtype=torch.int64, device="cuda")
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        torch.cuda.synchronize()
        ev[0].record()
        pm.error_matrix(dI, dT, M, out=E)
        ev[1].record()
        pm.local_search_async(E, perm, res)
        ev[2].record()
        ev[2].synchronize()
        if rep:
            te.append(ev[0].elapsed_time(ev[1]))
            tl.append(ev[1].elapsed_time(ev[2]))
    st, rounds, swaps = res.cpu().tolist()
    assert st == 0
    e, l = statistics.median(te), statistics.median(tl)
    print(f"| {N} | {g}x{g} | {M}x{M} | {e:.3f} ms | {pe*1e3:.0f} ms | {l:.3f} ms ({pm.ls_auto_method(S)}, {rounds}) | "
          f"{pls*1e3:.0f} ms | {e+l:.3f} ms | {ptot*1e3:.0f} ms |", flush=True)
