import sys
"""E-kernel (Step 2, Eq. 1) timing per BASELINE config: device-resident images,
CUDA events, median of reps.  Development probe (the contract bench is bench.py)."""
import os, statistics, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_ipps_yangin17_b200 import pm, synth
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import _devknobs  # noqa: E402
if os.environ.get("PM_LIB"):   # a development build of the library
    pm.LIB_PATH = os.environ["PM_LIB"]
_devknobs.apply(pm)

PEAK = 148 * 64 * 4 * 1.965e9          # VABSDIFF4.U8.ACC: 64 /clk/SM, 4 byte-absdiffs each
cfgs = [int(c) for c in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["1", "2", "3", "4", "5"])]
for cfg in cfgs:
    c = synth.CONFIGS[cfg]
    N, M, C = c["N"], c["M"], c["C"]
    S, P = (N // M) ** 2, M * M * C
    I, T = synth.config_pair(cfg, "smooth", 0)
    dI, dT = torch.from_numpy(I).cuda(), torch.from_numpy(T).cuda()
    E = torch.empty((S, S), dtype=torch.int32, device="cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    Ep = torch.empty(pm.sigma_copy_bytes(S) // 4, dtype=torch.int32, device="cuda") if S % 2 == 0 else None
    for variant in ("fused", "packed", "sigma"):
        if variant == "sigma" and Ep is None:
            continue
        ts = []
        It = Tt = None
        if variant == "packed":
            It, Tt = pm.pack_tiles(dI, M), pm.pack_tiles(dT, M)
        for r in range(6 if cfg >= 4 else 12):
            flush.fill_(r)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            if variant == "fused":
                pm.error_matrix(dI, dT, M, out=E)
            elif variant == "sigma":   # E + the sigma-permuted copy in one pass
                pm.error_matrix_sigma(dI, dT, M, E, Ep)
            else:
                pm.error_matrix_tiles(It, Tt, P, out=E)
            b.record()
            b.synchronize()
            if r >= 2:
                ts.append(a.elapsed_time(b))
        ms = statistics.median(ts)
        ops = S * S * P / (ms * 1e-3)
        print(f"cfg{cfg} S={S:6d} P={P} {variant:6s} {ms:9.3f} ms  {S*S/(ms*1e-3)/1e9:8.2f} Gpairs/s  "
              f"{ops/1e12:6.2f} T absdiff/s = {100*ops/PEAK:5.1f}% of ALU peak @1965MHz", flush=True)
    del E, Ep
    torch.cuda.empty_cache()
