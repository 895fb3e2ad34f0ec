#!/usr/bin/env python
"""Benchmark of the photomosaic hot path (Yang, Ito & Nakano, IPDPS-W 2017).

One STEP = one pass of the whole hot path over one synthetic photomosaic:
Step 1 (tile packing), Step 2 (the all-pairs error matrix E, Eq. 1), r :=
identity, Step 3 (Algorithm 2, colour-class local search to convergence) and
Eq. 2 (total error) -- the paper's approximation pipeline (Sec. V).

Workload (N=1): BASELINE.json configs[3] -- 2048x2048 RGB, 128x128 grid of
16x16-px tiles (S = 16384, E = 1 GiB), family "smooth", seed 0: the largest
configuration that fits one GPU and the 1-GPU point of north_star's
"1/2/4/8 B200" curve.  (configs[0..2] and configs[4] are parity-test cases.)
Multi-GPU (N > 1, torchrun): ONE photomosaic for the whole job (strong
scaling): rank g computes rows shard_rows(S, N, g) of E, NCCL all-gathers E,
and Algorithm 2 runs across the ranks (pm_local_search_multi_async: chunk
ranges per rank, halo slots by NVLink peer stores).  --independent runs N
independent photomosaics instead (weak scaling).

metric: tile-pair errors/s (Gpairs/s) + end-to-end local-search photomosaic ms
  value        = S^2 / (max-over-ranks device time per step)      [Gpairs/s]
                 (x N for --independent)
  ms_per_step  = the end-to-end local-search photomosaic time (device-resident)
  gpairs_per_s_error_matrix = S^2 / t_E (Step 1+2 alone, SURVEY 8(d)'s n^2/t_E)
  e2e          = the same metric through pm_photomosaic_host (HOST images in,
                 HOST r out, H2D/D2H inside the timed region)

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config 4] [--method auto]
  python bench.py --impl reference ...   # the CPU oracle as the reference arm
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "tile-pair errors/s (Gpairs/s) + end-to-end local-search photomosaic ms"
UNIT = "Gpairs/s"
DEFAULT_CONFIG = 4
L2_FLUSH_BYTES = 512 << 20          # > 126 MB L2
# VABSDIFF4.U8.ACC issue rate, measured (tools/ubench_alu.cu,
# profiles/r01_ubench_alu.txt): 1.83e13 instr/s on 148 SMs = 64 per clock per
# SM (half the IADD3 rate, ~124/clk/SM, measured in the same run)
ALU_VABSDIFF4_PER_CLK_PER_SM = 64


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=DEFAULT_CONFIG)
    ap.add_argument("--family", default="smooth")
    ap.add_argument("--method", default="auto", choices=["auto", "trap", "class", "window", "walk"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-oracle", action="store_true", help="skip the oracle entirely (profiling runs)")
    ap.add_argument("--cpu-1t-rows", type=int, default=96,
                    help="rows of E in the one-thread oracle sample (extrapolated to S rows)")
    ap.add_argument("--ref-rows", type=int, default=1024,
                    help="--impl reference: rows of E per step (extrapolated to S rows)")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--independent", action="store_true",
                    help="N > 1: N independent photomosaics (weak scaling) instead of one sharded one")
    ap.add_argument("--sharded", action="store_true", help="N = 1: force the sharded code path")
    ap.add_argument("--e-layout", default="gathered", choices=["gathered", "rows"],
                    help="one photomosaic over N ranks: E all-gathered onto every rank (default), or left "
                         "row-sharded in symmetric memory and read over NVLink (pm_local_search_sharded_async)")
    return ap.parse_args()


def workload_desc(cfg, fam, seeds):
    from paper_conf_ipps_yangin17_b200 import synth
    c = synth.CONFIGS[cfg]
    g = c["N"] // c["M"]
    return {"workload": f"config{cfg}: {c['N']}x{c['N']} RGB, {g}x{g} grid of {c['M']}x{c['M']}-px tiles "
                        f"(S={g * g}), synthetic family '{fam}'",
            "N": c["N"], "M": c["M"], "C": c["C"], "S": g * g, "family": fam, "seeds": seeds}


def host_info():
    import platform
    model = platform.processor() or ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"cpu_model": model, "host_cores": len(os.sched_getaffinity(0))}


def peaks_and_alu(sm_max_mhz):
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except (OSError, ValueError):
        pass
    hbm_peak = peaks.get("hbm_gbs", 6650.0)
    hbm_src = "measured (MEASURED_PEAKS.json hbm_gbs)" if "hbm_gbs" in peaks else "fallback (B200_PROFILING.md)"
    alu_peak = 148 * ALU_VABSDIFF4_PER_CLK_PER_SM * 4 * sm_max_mhz * 1e6 / 1e12   # T byte-absdiff/s
    return hbm_peak, hbm_src, alu_peak


def ncu_traffic(name, cfg):
    """dram read+write bytes per launch of kernel `name` from the committed ncu
    --set full capture of this workload (profiles/traffic.json), or None."""
    try:
        t = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
    except (OSError, ValueError):
        return None
    e = t.get(f"config{cfg}", {}).get(name)
    return None if not e else e["dram_read_bytes"] + e["dram_write_bytes"]


# ------------------------------------------------------------- CPU oracle --
def oracle_full(I, T, M):
    """The oracle as it stands (E loop nest, OpenMP over rows; Alg. 2 serial
    replay, OpenMP inside each class; Eq. 2) on the whole workload, all host
    threads.  Returns timings and the result."""
    import oracle
    oracle.build()
    t0 = time.perf_counter()
    E = oracle.error_matrix(I, T, M)
    t1 = time.perf_counter()
    r, rounds, swaps, per, st = oracle.local_search(E)
    t2 = time.perf_counter()
    c = oracle.cost(E, r)
    t3 = time.perf_counter()
    return E, dict(r=r, rounds=rounds, swaps=swaps, cost=c, status=st), dict(E=t1 - t0, ls=t2 - t1, cost=t3 - t2)


def oracle_one_thread_sample(I, T, M, E, rounds, rows):
    """One host thread (the paper's CPU convention): E rows [0, rows)
    and one round of Alg. 2 on the full E, each timed and extrapolated (E is
    row-independent work; every oracle round evaluates all S(S-1)/2 pairs)."""
    import oracle
    S = E.shape[0]
    nt = oracle.num_threads()
    oracle.set_num_threads(1)
    try:
        t0 = time.perf_counter()
        oracle.error_matrix(I, T, M, rows=(0, rows))
        t1 = time.perf_counter()
        oracle.local_search(E, max_rounds=1)
        t2 = time.perf_counter()
    finally:
        oracle.set_num_threads(nt)
    t_E = (t1 - t0) * S / rows
    t_ls = (t2 - t1) * rounds
    return {"value": S * S / (t_E + t_ls) / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"one thread: E rows [0, {rows}) ({t1 - t0:.2f} s, x{S / rows:.0f}) + one Alg. 2 round "
                      f"({t2 - t1:.2f} s, x{rounds} rounds), extrapolated",
            "ms_per_photomosaic_extrapolated": (t_E + t_ls) * 1e3}


# ---------------------------------------------------------------- clocks ---
class ClockSampler:
    """nvidia-smi-equivalent sampling (NVML) of SM clock and throttle reasons
    during the timed region."""

    def __init__(self, dev_index=0, period=0.01):
        self.samples = []
        self.reasons = set()
        self.period = period
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:  # pragma: no cover
            self.max_mhz = None
        self._stop = threading.Event()

    def _run(self):
        nv = self.nv
        names = {
            "gpu_idle": 0x1, "applications_clocks_setting": 0x2, "sw_power_cap": 0x4, "hw_slowdown": 0x8,
            "sync_boost": 0x10, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
            "hw_power_brake_slowdown": 0x80, "display_clock_setting": 0x100,
        }
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                mask = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for k, bit in names.items():
                    if mask & bit and k != "gpu_idle":
                        self.reasons.add(k)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def rooflines(cfg, S, P, rounds, ls_ms, e_ms, e_rows, sm_max, method_used, sigma_fused=False):
    """Dominant-kernel roofline objects: Alg. 2 against HBM
    with its algorithmic 8 bytes per pair evaluation, the E kernel against
    the VABSDIFF4 ALU peak with P byte-absdiffs per pair."""
    hbm_peak, hbm_src, alu_peak = peaks_and_alu(sm_max)
    ls_bytes = rounds * (S * (S - 1) // 2) * 8
    ls_gbs = ls_bytes / (ls_ms * 1e-3) / 1e9
    e_tops = e_rows * S * P / (e_ms * 1e-3) / 1e12
    ls_kernel = {"trap": "k_ls_trap (dense rounds) + k_sp_scan/k_sp_cwalk (sparse rounds)",
                 "window": "k_ls_window + sparse rounds", "class": "k_ls_class x (S-1) per round + sparse rounds",
                 "walk": "k_sp_scan + k_sp_cwalk rounds"}[method_used]
    roof_ls = {"kernel": f"Alg. 2, all rounds: {ls_kernel}", "bound": "hbm", "achieved": ls_gbs,
               "peak": hbm_peak, "unit": "GB/s", "frac": ls_gbs / hbm_peak,
               "traffic": ncu_traffic("k_ls_trap", cfg) if method_used == "trap" else None,
               "peak_source": hbm_src, "algorithmic_bytes": ls_bytes,
               "timing": "CUDA events around the local-search call on its stream, mean over the timed steps",
               "note": "latency-bound chain of S-1 dependent class steps per round; "
                       "algorithmic bytes = rounds * S(S-1)/2 * 8 (2 int32 E gathers per pair evaluation)"}
    roof_e = {"kernel": "k_sad (Eq. 1 SAD-GEMM, VABSDIFF4) + k_pack (Step 1)"
                        + (", whose epilogue also writes the sigma-permuted copy of E (1 more int32 store per entry; "
                           "the search then skips k_permute_cols)" if sigma_fused else ""), "bound": "alu",
              "achieved": e_tops, "peak": alu_peak, "unit": "T byte-absdiff/s", "frac": e_tops / alu_peak,
              "traffic": ncu_traffic("k_sad", cfg),
              "peak_source": f"derived: 148 SM x {ALU_VABSDIFF4_PER_CLK_PER_SM} VABSDIFF4/clk (measured issue "
                             f"rate) x 4 byte-absdiffs x {sm_max} MHz",
              "algorithmic_ops": e_rows * S * P}
    return (roof_ls, roof_e) if ls_ms >= e_ms else (roof_e, roof_ls)


# ------------------------------------------------------------ one GPU ------
def bench_single(args, rank, world, local_rank):
    import torch

    from paper_conf_ipps_yangin17_b200 import pm, synth
    from paper_conf_ipps_yangin17_b200 import dist as pdist

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    cfg = synth.CONFIGS[args.config]
    N, M, C = cfg["N"], cfg["M"], cfg["C"]
    S = (N // M) ** 2
    P = M * M * C
    seed = rank if args.independent else 0
    I_np, T_np = synth.make_pair(args.family, N, M, C, seed=seed)
    dI = torch.from_numpy(I_np).to(dev)
    dT = torch.from_numpy(T_np).to(dev)
    E = torch.empty((S, S), dtype=torch.int32, device=dev)
    perm = torch.empty(S, dtype=torch.int32, device=dev)
    res = torch.zeros(4, dtype=torch.int64, device=dev)       # {status, rounds, swaps, cost}
    flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    # TRAP stages from the sigma-permuted copy of E: write it in the E pass
    # (pm_error_matrix_sigma) into a buffer allocated once, as
    # pm_photomosaic_async does internally
    use_sigma = (pm.ls_auto_method(S) if args.method == "auto" else args.method) == "trap"
    Ep = torch.empty(pm.sigma_copy_bytes(S) // 4 if use_sigma else 1, dtype=torch.int32, device=dev)

    def step(evs=None):
        # the public ABI pieces of pm_photomosaic_async, with events between them
        if evs: evs[0].record(stream)
        if use_sigma:
            pm.error_matrix_sigma(dI, dT, M, E, Ep)            # Step 1 + Step 2 (+ the sigma copy)
        else:
            pm.error_matrix(dI, dT, M, out=E)                  # Step 1 + Step 2
        if evs: evs[1].record(stream)
        pm.init_identity(perm)
        if use_sigma:
            pm.local_search_sigma_async(E, perm, res[:3], Ep, method=args.method)
        else:
            pm.local_search_async(E, perm, res[:3], method=args.method)
        if evs: evs[2].record(stream)
        pm.cost_async(E, perm, res[3:])
        if evs: evs[3].record(stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    ref_res = res.cpu().tolist()

    K = args.steps
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in range(K)]
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    torch.cuda.synchronize()
    n0 = pm.launch_count()
    with ClockSampler(local_rank) as clk:
        t_wall0 = time.perf_counter()
        for i in range(K):
            flush.fill_(i & 0xFF)                              # L2 flush, outside the step events
            step(evs[i])
        torch.cuda.synchronize()
        t_wall = time.perf_counter() - t_wall0
    launches = pm.launch_count() - n0
    if world > 1:
        dist.barrier()
    step_ms = [e[0].elapsed_time(e[3]) for e in evs]
    e_ms = [e[0].elapsed_time(e[1]) for e in evs]
    ls_ms = [e[1].elapsed_time(e[2]) for e in evs]
    cost_ms = [e[2].elapsed_time(e[3]) for e in evs]
    out_res = res.cpu().tolist()
    assert out_res == ref_res, "non-deterministic result across steps"
    assert out_res[0] == 0, f"search status {out_res[0]}"
    max_tot_ms = pdist.max_over_ranks(sum(step_ms), device=dev)
    ms_per_step = max_tot_ms / K
    value = S * S * world / (ms_per_step * 1e-3) / 1e9
    mean_e, mean_ls = statistics.mean(e_ms), statistics.mean(ls_ms)

    # -------- e2e: HOST images -> pm_photomosaic_host -> HOST r (pinned) ------
    hI = torch.from_numpy(I_np).pin_memory()
    hT = torch.from_numpy(T_np).pin_memory()
    hperm = torch.empty(S, dtype=torch.int32).pin_memory()
    pm.photomosaic_host(hI.numpy(), hT.numpy(), M, method=args.method, perm_out=hperm.numpy())
    torch.cuda.synchronize()
    e2e_ms = []
    for i in range(args.e2e_steps):
        flush.fill_(i & 0xFF)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        _, rounds_h, swaps_h, cost_h = pm.photomosaic_host(hI.numpy(), hT.numpy(), M, method=args.method,
                                                          perm_out=hperm.numpy())
        b.record(stream)
        b.synchronize()
        e2e_ms.append(a.elapsed_time(b))
    assert [0, rounds_h, swaps_h, cost_h] == out_res
    assert (hperm.numpy() == perm.cpu().numpy()).all()
    e2e_max_ms = pdist.max_over_ranks(statistics.mean(e2e_ms), device=dev)
    e2e_val = S * S * world / (e2e_max_ms * 1e-3) / 1e9

    rounds = out_res[1]
    sm_max = clk.max_mhz or 1965
    used = pm.ls_auto_method(S) if args.method == "auto" else args.method
    dominant, other = rooflines(args.config, S, P, rounds, mean_ls, mean_e, S, sm_max, used, use_sigma)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K, "warmup": args.warmup,
        "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "u8->int32", "data": "synthetic",
        "config": dict(workload_desc(args.config, args.family, [seed] if world == 1 else list(range(world))),
                       l2="flushed between steps (512 MiB write outside the per-step CUDA events)",
                       method=args.method,
                       parallelism="1 GPU" if world == 1 else f"{world} independent photomosaics (one per rank)"),
        "gpairs_per_s_error_matrix": S * S / (mean_e * 1e-3) / 1e9,
        "e2e": {"value": e2e_val, "unit": UNIT, "ms": e2e_max_ms,
                "h2d_bytes_per_step": 2 * N * N * C, "d2h_bytes_per_step": 4 * S + 8 * 4,
                "api": "pm_photomosaic_host (pinned host images -> host r)"},
        "gpu_launches": launches,
        "roofline": dominant, "roofline_other": other,
        "breakdown_ms": {"pack+error_matrix": mean_e, "local_search": mean_ls, "cost": statistics.mean(cost_ms),
                         "note": ("the E pass also writes TRAP's sigma-permuted copy of E (pm_error_matrix_sigma); "
                                  "the search runs on it (pm_local_search_sigma_async)") if use_sigma else ""},
        "local_search": {"method": used, "rounds": rounds, "class_steps": rounds * max(S - 1, 1),
                         "ns_per_class_step": mean_ls * 1e6 / (rounds * max(S - 1, 1))},
        "result": {"rounds": rounds, "swaps": out_res[2], "cost": out_res[3]},
        "wall_s_timed_region": t_wall,
        "clocks": clk.summary(),
    }
    return line, (I_np, T_np, M, S, perm.cpu().numpy(), out_res)


# ------------------------------------------------- one photomosaic, N GPUs --
def bench_sharded(args, rank, world, local_rank):
    """One photomosaic for the whole job: every rank computes its row shard of
    E (pm_error_matrix rows), NCCL all-gathers E, and Algorithm 2 runs across
    the ranks (pm_local_search_multi_async).  value = S^2 / step time.
    --e-layout rows: E is never gathered -- each rank's rows stay in its
    symmetric-memory shard and pm_local_search_sharded_async /
    pm_cost_sharded_async read every row from its owner over NVLink."""
    import torch
    import torch.distributed as dist
    import torch.distributed._symmetric_memory as symm_mem

    from paper_conf_ipps_yangin17_b200 import dist as pdist
    from paper_conf_ipps_yangin17_b200 import pm, synth

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world == 1 and not dist.is_initialized():
        dist.init_process_group("nccl", init_method="tcp://127.0.0.1:29517", rank=0, world_size=1, device_id=dev)
    cfg = synth.CONFIGS[args.config]
    N, M, C = cfg["N"], cfg["M"], cfg["C"]
    S = (N // M) ** 2
    P = M * M * C
    I_np, T_np = synth.make_pair(args.family, N, M, C, seed=0)       # the same photomosaic on every rank
    hI = torch.from_numpy(I_np).pin_memory()
    hT = torch.from_numpy(T_np).pin_memory()
    dI = hI.to(dev)
    dT = hT.to(dev)
    b, e = pdist.shard_rows(S, world, rank)
    sizes = [pdist.shard_rows(S, world, g) for g in range(world)]
    rows_max = max(se - sb for sb, se in sizes)
    rows_layout = args.e_layout == "rows"
    pb = (4 * S + 255) // 256 * 256
    if rows_layout:
        rb = [sb for sb, _ in sizes] + [S]
        ws_bytes = (pm.trap_workspace_bytes_sharded(S, rows_max) + 255) // 256 * 256
        buf = symm_mem.empty(ws_bytes + pb + 4 * rows_max * S, dtype=torch.uint8, device=dev)
        part = buf[ws_bytes + pb:].view(torch.int32).view(rows_max, S)     # this rank's shard, peer-mapped
    else:
        parts = torch.zeros((world, rows_max, S), dtype=torch.int32, device=dev)
        part = parts[rank]                                               # in-place all-gather
        contiguous = all(se - sb == rows_max for sb, se in sizes)
        E_full = parts.view(world * rows_max, S) if contiguous else torch.empty((S, S), dtype=torch.int32, device=dev)
        ws_bytes = (pm.trap_workspace_bytes(S) + 255) // 256 * 256
        buf = symm_mem.empty(ws_bytes + pb, dtype=torch.uint8, device=dev)
    hdl = symm_mem.rendezvous(buf, dist.group.WORLD.group_name)
    ptrs = [int(p) for p in hdl.buffer_ptrs]
    my_perm = buf[ws_bytes:ws_bytes + 4 * S].view(torch.int32)
    e_ptrs = [p + ws_bytes + pb for p in ptrs]
    res = torch.zeros(3, dtype=torch.int64, device=dev)
    cost = torch.zeros(1, dtype=torch.int64, device=dev)
    token = torch.zeros(1, dtype=torch.int32, device=dev)
    hperm = torch.empty(S, dtype=torch.int32).pin_memory()
    stream = torch.cuda.current_stream()
    flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)

    def step(evs=None, host=False):
        if host:                                                           # e2e: host images in
            dI.copy_(hI, non_blocking=True)
            dT.copy_(hT, non_blocking=True)
        if evs: evs[0].record(stream)
        pm.error_matrix(dI, dT, M, rows=(b, e), out=part[: e - b])        # Step 1+2, this rank's rows
        if evs: evs[1].record(stream)
        if world > 1 and not rows_layout:
            dist.all_gather_into_tensor(parts.view(world * rows_max, S), part)
            if not contiguous:
                for g, (sb, se) in enumerate(sizes):
                    E_full[sb:se].copy_(parts[g, : se - sb])
        if evs: evs[2].record(stream)
        pm.init_identity(my_perm)
        pm.trap_workspace_reset(buf, S)
        dist.all_reduce(token)                             # every workspace reset, every shard written (device order)
        if rows_layout:
            pm.local_search_sharded_async(e_ptrs, rb, S, S, [p + ws_bytes for p in ptrs], ptrs, rank, world, res)
        else:
            pm.local_search_multi_async(E_full, [p + ws_bytes for p in ptrs], ptrs, rank, world, res)
        if evs: evs[3].record(stream)
        if rows_layout:
            pm.cost_sharded_async(e_ptrs, rb, S, S, my_perm, cost)
        else:
            pm.cost_async(E_full, my_perm, cost)
        if evs: evs[4].record(stream)
        if host:                                                           # e2e: host r out
            hperm.copy_(my_perm, non_blocking=True)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    ref = res.cpu().tolist() + cost.cpu().tolist()
    K = args.steps
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(5)] for _ in range(K)]
    dist.barrier()
    torch.cuda.synchronize()
    n0 = pm.launch_count()
    with ClockSampler(local_rank) as clk:
        for i in range(K):
            flush.fill_(i & 0xFF)
            step(evs[i])
        torch.cuda.synchronize()
    launches = pm.launch_count() - n0
    dist.barrier()
    out = res.cpu().tolist() + cost.cpu().tolist()
    assert out == ref and out[0] == 0, f"sharded search {out} vs {ref}"
    tot = [ev[0].elapsed_time(ev[4]) for ev in evs]
    ms = pdist.max_over_ranks(statistics.mean(tot), device=dev)
    part_ms = {k: statistics.mean([ev[i].elapsed_time(ev[i + 1]) for ev in evs])
               for k, i in (("error_matrix_shard", 0), ("all_gather", 1), ("local_search_multi", 2), ("cost", 3))}
    # e2e: pinned host images -> ... -> host r, every step
    e2e = []
    for i in range(args.e2e_steps):
        flush.fill_(i & 0xFF)
        a, z = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        step(host=True)
        z.record(stream)
        z.synchronize()
        e2e.append(a.elapsed_time(z))
    assert (hperm.numpy() == my_perm.cpu().numpy()).all()
    e2e_ms = pdist.max_over_ranks(statistics.mean(e2e), device=dev)
    sm_max = clk.max_mhz or 1965
    dominant, other = rooflines(args.config, S, P, out[1], part_ms["local_search_multi"],
                                part_ms["error_matrix_shard"], e - b, sm_max, "trap")
    line = {
        "metric": METRIC, "value": S * S / (ms * 1e-3) / 1e9, "unit": UNIT, "n_gpus": world, "steps": K,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "u8->int32", "data": "synthetic",
        "config": dict(workload_desc(args.config, args.family, [0]),
                       method="trap (multi-rank, row-sharded E)" if rows_layout else "trap (multi-rank)",
                       parallelism=(f"one photomosaic: E rows sharded over {world} ranks, never gathered; Alg. 2 "
                                    f"across the ranks reading E rows from their owner (NVLink peer loads)"
                                    if rows_layout else
                                    f"one photomosaic: E rows sharded over {world} ranks + NCCL all-gather; "
                                    f"Alg. 2 across the ranks (NVLink peer stores of halo slots)"),
                       l2="flushed between steps (512 MiB write outside the per-step CUDA events)"),
        "gpairs_per_s_error_matrix": S * S / (pdist.max_over_ranks(part_ms["error_matrix_shard"], device=dev)
                                              * 1e-3) / 1e9,
        "e2e": {"value": S * S / (e2e_ms * 1e-3) / 1e9, "unit": UNIT, "ms": e2e_ms,
                "h2d_bytes_per_step": 2 * N * N * C, "d2h_bytes_per_step": 4 * S,
                "api": ("per rank: pinned host images -> pm_error_matrix rows -> pm_local_search_sharded_async -> "
                        "pm_cost_sharded_async -> pinned host r" if rows_layout else
                        "per rank: pinned host images -> pm_error_matrix rows -> all-gather -> "
                        "pm_local_search_multi_async -> pm_cost_async -> pinned host r")},
        "gpu_launches": launches,
        "roofline": dominant, "roofline_other": other,
        "breakdown_ms_rank0": part_ms,
        "result": {"rounds": out[1], "swaps": out[2], "cost": out[3]},
        "clocks": clk.summary(),
    }
    return line, (I_np, T_np, M, S, my_perm.cpu().numpy(), [0, out[1], out[2], out[3]])


def attach_oracle(line, extra, args):
    """cpu_baseline (rank 0, N = 1) and parity of this run's result against the
    oracle's full replay of the same workload."""
    I_np, T_np, M, S, perm_np, out_res = extra
    E, ref, t = oracle_full(I_np, T_np, M)
    import oracle
    full_s = t["E"] + t["ls"] + t["cost"]
    line["parity_vs_oracle"] = bool((ref["r"] == perm_np).all() and ref["rounds"] == out_res[1]
                                    and ref["swaps"] == out_res[2] and ref["cost"] == out_res[3])
    line["parity_detail"] = {"compared": "final r (all S slots), rounds, swaps, cost (Eq. 2) vs oracle.local_search "
                                         "on oracle.error_matrix", "oracle_rounds": ref["rounds"],
                             "oracle_swaps": ref["swaps"], "oracle_cost": ref["cost"]}
    if not args.no_cpu_baseline:
        one = oracle_one_thread_sample(I_np, T_np, M, E, ref["rounds"], args.cpu_1t_rows)
        line["cpu_baseline"] = {
            "value": S * S / full_s / 1e9, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
            "sample": f"the full workload once: E {t['E']:.1f} s + Alg. 2 {t['ls']:.1f} s + Eq. 2 on all host "
                      f"threads (OpenMP over E rows / over the pairs of one class)",
            "ms_per_photomosaic": full_s * 1e3, "one_thread": one}


# ------------------------------------------------------------------ main ---
def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return main_reference(args, rank, world)
    import torch
    import torch.distributed as dist
    if world > 1:
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    if (world > 1 and not args.independent) or args.sharded or args.e_layout == "rows":
        line, extra = bench_sharded(args, rank, world, local_rank)
    else:
        line, extra = bench_single(args, rank, world, local_rank)
    if rank == 0 and not args.no_oracle:
        if world == 1:
            attach_oracle(line, extra, args)                 # cpu_baseline + parity
        elif not args.independent:
            args.no_cpu_baseline = True                      # cpu_baseline: rank 0 at N = 1 only
            attach_oracle(line, extra, args)                 # parity of the sharded result
    if rank == 0:
        line["host"] = host_info()
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def main_reference(args, rank, world):
    """The reference arm: the CPU oracle (oracle/), as it stands, on this
    box's host cores, same workload/metric; rank 0 only.  Each step is a
    bounded sample of the workload: E rows [i*R, (i+1)*R) and one round of
    Alg. 2 on the full E, extrapolated to the whole photomosaic (S/R row
    blocks, `rounds` rounds -- the oracle evaluates all pairs every round)."""
    if rank != 0:
        return
    from paper_conf_ipps_yangin17_b200 import synth
    import oracle
    oracle.build()
    cfg = synth.CONFIGS[args.config]
    N, M, C = cfg["N"], cfg["M"], cfg["C"]
    S = (N // M) ** 2
    I, T = synth.make_pair(args.family, N, M, C, seed=0)
    E = oracle.error_matrix(I, T, M)                        # setup (untimed): the full E, and the round count
    rounds = oracle.local_search(E)[1]
    R = min(args.ref_rows, S)
    nblk = max(S // R, 1)

    def one(i):
        r0 = (i % nblk) * R
        t0 = time.perf_counter()
        oracle.error_matrix(I, T, M, rows=(r0, r0 + R))
        t1 = time.perf_counter()
        oracle.local_search(E, max_rounds=1)
        t2 = time.perf_counter()
        return (t1 - t0) * S / R + (t2 - t1) * rounds

    for i in range(min(args.warmup, 3)):
        one(i)
    times = [one(i) for i in range(args.steps)]
    mean = statistics.mean(times)
    value = S * S / mean / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": mean * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u8->int32", "data": "synthetic",
        "config": dict(workload_desc(args.config, args.family, [0]), method="oracle (CPU)"),
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
                         "sample": f"per step: E rows of one {R}-row block (x{S / R:.0f}) + one Alg. 2 round on "
                                   f"the full E (x{rounds} rounds), extrapolated; all host threads"},
        "host": host_info(),
    }
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
