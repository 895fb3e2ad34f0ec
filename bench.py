#!/usr/bin/env python
"""Benchmark of the photomosaic hot path (Yang, Ito & Nakano, IPDPS-W 2017).

One STEP = one pass of the whole hot path over one synthetic photomosaic:
Step 1 (tile packing), Step 2 (the all-pairs error matrix E, Eq. 1), r :=
identity, Step 3 (Algorithm 2, colour-class local search to convergence) and
Eq. 2 (total error) -- the paper's approximation pipeline (Sec. V).

Workload (N=1): BASELINE.json configs[1] -- 512x512 RGB, 32x32 grid of 16x16
tiles (S = 1024, the paper's Fig. 2 shape), family "smooth", seed = rank.
Multi-GPU: one process per GPU, each rank an independent photomosaic
(weak scaling; no data-path collective -- DESIGN.md "Multi-GPU").

metric: tile-pair errors/s (Gpairs/s) + end-to-end local-search photomosaic ms
  value        = S^2 * n_ranks / (max-over-ranks device time per step)   [Gpairs/s]
  ms_per_step  = the end-to-end local-search photomosaic time (device-resident)
  e2e          = the same through pm_photomosaic_host (HOST images in, HOST r
                 out, H2D/D2H inside the timed region)

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config 2] [--method auto]
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
L2_FLUSH_BYTES = 512 << 20          # > 126 MB L2
ALU_VABSDIFF4_PER_CLK_PER_SM = 64    # tools/ubench_alu.cu (same issue rate as IADD3)


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--family", default="smooth")
    ap.add_argument("--method", default="auto", choices=["auto", "trap", "class", "cta", "window", "pairwin", "walk"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0, help="budget of the cpu_baseline sample")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--sharded", action="store_true",
                    help="one photomosaic for the whole job (strong scaling): E row-sharded + all-gathered "
                         "(NCCL), Alg. 2 across the ranks (pm_local_search_multi_async over symmetric memory)")
    return ap.parse_args()


def workload_desc(cfg, fam, rank_seeds):
    from paper_conf_ipps_yangin17_b200 import synth
    c = synth.CONFIGS[cfg]
    g = c["N"] // c["M"]
    return {"workload": f"config{cfg}: {c['N']}x{c['N']} RGB, {g}x{g} grid of {c['M']}x{c['M']}-px tiles "
                        f"(S={g * g}), synthetic family '{fam}', seed=rank",
            "N": c["N"], "M": c["M"], "C": c["C"], "S": g * g, "family": fam, "seeds": rank_seeds}


# ------------------------------------------------------------- CPU oracle --
def run_oracle_once(I, T, M):
    import oracle
    t0 = time.perf_counter()
    E = oracle.error_matrix(I, T, M)
    r, rounds, swaps, per, st = oracle.local_search(E)
    c = oracle.cost(E, r)
    return time.perf_counter() - t0, dict(r=r, rounds=rounds, swaps=swaps, cost=c)


def cpu_baseline(I, T, M, S, budget_s):
    """The oracle as it stands (E loop nest with OpenMP over rows, serial class
    replay with OpenMP inside each class, Eq. 2), repeated on the whole
    workload until `budget_s` of CPU time has been spent (at least once)."""
    import oracle
    oracle.build()
    times, res = [], None
    t_start = time.perf_counter()
    while True:
        t, res = run_oracle_once(I, T, M)
        times.append(t)
        if time.perf_counter() - t_start >= budget_s:
            break
    mean = statistics.mean(times)
    return {"value": S * S / mean / 1e9, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
            "sample": f"the full workload (one 512x512-class photomosaic: E + Alg. 2 + Eq. 2) x {len(times)} "
                      f"repetitions, mean {mean * 1e3:.1f} ms each",
            "ms_per_photomosaic": mean * 1e3}, res


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


# ------------------------------------------------------------------ ours ---
def bench_ours(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist

    from paper_conf_ipps_yangin17_b200 import pm, synth

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    cfg = synth.CONFIGS[args.config]
    N, M, C = cfg["N"], cfg["M"], cfg["C"]
    S = (N // M) ** 2
    P = M * M * C
    I_np, T_np = synth.make_pair(args.family, N, M, C, seed=rank)
    dI = torch.from_numpy(I_np).to(dev)
    dT = torch.from_numpy(T_np).to(dev)
    E = torch.empty((S, S), dtype=torch.int32, device=dev)
    perm = torch.empty(S, dtype=torch.int32, device=dev)
    res = torch.zeros(4, dtype=torch.int64, device=dev)       # {status, rounds, swaps, cost}
    flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    def step(evs=None):
        # the public ABI pieces of pm_photomosaic_async, with events between them
        if evs: evs[0].record(stream)
        pm.error_matrix(dI, dT, M, out=E)                      # pack x2 + E kernel
        if evs: evs[1].record(stream)
        pm.init_identity(perm)
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

    from paper_conf_ipps_yangin17_b200 import dist as pdist
    max_tot_ms = pdist.max_over_ranks(sum(step_ms), device=dev)
    ms_per_step = max_tot_ms / K
    value = S * S * world / (ms_per_step * 1e-3) / 1e9

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

    # -------- roofline of the dominant kernel(s) --------------------------------
    rounds = out_res[1]
    mean_e, mean_ls = statistics.mean(e_ms), statistics.mean(ls_ms)
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except OSError:
        pass
    hbm_peak = peaks.get("hbm_gbs", 6650.0)
    hbm_src = "measured" if "hbm_gbs" in peaks else "fallback"
    sm_max = (clk.max_mhz or 1965)
    alu_peak = 148 * ALU_VABSDIFF4_PER_CLK_PER_SM * 4 * sm_max * 1e6 / 1e12   # T byte-absdiff/s
    ls_bytes = rounds * (S * (S - 1) // 2) * 8          # 2 int32 gathers per pair evaluation
    ls_gbs = ls_bytes / (mean_ls * 1e-3) / 1e9
    e_tops = S * S * P / (mean_e * 1e-3) / 1e12
    used = pm.ls_auto_method(S) if args.method == "auto" else args.method
    ls_kernel = {"trap": "k_ls_trap (temporal-blocked class replay, dense rounds) + sparse rounds",
                 "window": "k_ls_window (+ k_permute_cols) + sparse rounds", "cta": "k_ls_cta",
                 "class": "k_ls_class x (S-1) per round (CUDA graph) + sparse rounds",
                 "pairwin": "k_pw_* rounds", "walk": "k_sp_scan + k_sp_walk rounds"}[used]
    traffic = {}
    try:
        traffic = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
    except (OSError, ValueError):
        pass

    def _traffic(name):
        t = traffic.get(name)
        return None if not t else t["dram_read_bytes"] + t["dram_write_bytes"]

    roof_ls = {"kernel": f"{ls_kernel}: Alg. 2, all rounds", "bound": "hbm", "achieved": ls_gbs,
               "peak": hbm_peak, "unit": "GB/s", "frac": ls_gbs / hbm_peak,
               "traffic": _traffic("k_ls_" + used) if used in ("trap", "window", "cta") else None,
               "peak_source": hbm_src, "algorithmic_bytes": ls_bytes,
               "note": "latency-bound dependency chain of S-1 class steps per round; bytes = rounds*S(S-1)/2*8"}
    roof_e = {"kernel": "k_sad (Eq. 1; Step 1 fused into its loader at S <= 4096)", "bound": "alu",
              "achieved": e_tops, "peak": alu_peak,
              "unit": "T byte-absdiff/s", "frac": e_tops / alu_peak, "traffic": _traffic("k_sad"),
              "peak_source": f"derived: 148 SM x {ALU_VABSDIFF4_PER_CLK_PER_SM} VABSDIFF4/clk x 4 B x {sm_max} MHz",
              "gpairs_per_s": S * S / (mean_e * 1e-3) / 1e9}
    dominant = roof_ls if mean_ls >= mean_e else roof_e
    other = roof_e if dominant is roof_ls else roof_ls

    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": K, "warmup": args.warmup,
        "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
        "dtype": "u8->int32", "data": "synthetic",
        "config": dict(workload_desc(args.config, args.family, list(range(world))),
                       l2="flushed between steps (512 MiB write outside the per-step CUDA events)",
                       method=args.method, parallelism=f"{world} independent photomosaics (one per rank)"),
        "e2e": {"value": e2e_val, "unit": UNIT, "ms": e2e_max_ms,
                "h2d_bytes_per_step": 2 * N * N * C, "d2h_bytes_per_step": 4 * S + 8 * 4,
                "api": "pm_photomosaic_host (pinned host images -> host r)"},
        "gpu_launches": launches,
        "roofline": dominant, "roofline_other": other,
        "breakdown_ms": {"pack+error_matrix": mean_e, "local_search": mean_ls,
                         "cost": statistics.mean(cost_ms)},
        "local_search": {"method": used, "rounds": rounds, "class_steps": rounds * max(S - 1, 1),
                         "ns_per_class_step": mean_ls * 1e6 / (rounds * max(S - 1, 1))},
        "result": {"rounds": rounds, "swaps": out_res[2], "cost": out_res[3]},
        "wall_s_timed_region": t_wall,
        "clocks": clk.summary(),
    }
    return line, (I_np, T_np, M, S, perm.cpu().numpy(), out_res)



def bench_sharded(args, rank, world, local_rank):
    """One photomosaic for the whole job: every rank computes its row shard of
    E (pm_error_matrix rows), NCCL all-gathers E, and Algorithm 2 runs across
    the ranks (pm_local_search_multi_async: per-rank chunk ranges, halo slots
    by NVLink peer stores).  value = S^2 / step time (strong scaling)."""
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
    I_np, T_np = synth.make_pair(args.family, N, M, C, seed=0)       # the same photomosaic on every rank
    dI = torch.from_numpy(I_np).to(dev)
    dT = torch.from_numpy(T_np).to(dev)
    b, e = pdist.shard_rows(S, world, rank)
    rows_max = max(pdist.shard_rows(S, world, g)[1] - pdist.shard_rows(S, world, g)[0] for g in range(world))
    parts = torch.zeros((world, rows_max, S), dtype=torch.int32, device=dev)
    part = parts[rank]                                                   # in-place all-gather
    sizes = [pdist.shard_rows(S, world, g) for g in range(world)]
    contiguous = all(se - sb == rows_max for sb, se in sizes)
    E_full = parts.view(world * rows_max, S) if contiguous else torch.empty((S, S), dtype=torch.int32, device=dev)
    ws_bytes = (pm.trap_workspace_bytes(S) + 255) // 256 * 256
    buf = symm_mem.empty(ws_bytes + 4 * S, dtype=torch.uint8, device=dev)
    hdl = symm_mem.rendezvous(buf, dist.group.WORLD.group_name)
    ptrs = [int(p) for p in hdl.buffer_ptrs]
    my_perm = buf[ws_bytes:].view(torch.int32)
    res = torch.zeros(3, dtype=torch.int64, device=dev)
    cost = torch.zeros(1, dtype=torch.int64, device=dev)
    token = torch.zeros(1, dtype=torch.int32, device=dev)
    stream = torch.cuda.current_stream()

    def step(evs=None):
        if evs: evs[0].record(stream)
        pm.error_matrix(dI, dT, M, rows=(b, e), out=part[: e - b])        # Step 1+2, this rank's rows
        if evs: evs[1].record(stream)
        if world > 1:
            dist.all_gather_into_tensor(parts.view(world * rows_max, S), part)
            if not contiguous:
                for g, (sb, se) in enumerate(sizes):
                    E_full[sb:se].copy_(parts[g, : se - sb])
        if evs: evs[2].record(stream)
        pm.init_identity(my_perm)
        pm.trap_workspace_reset(buf, S)
        dist.all_reduce(token)                                             # every workspace reset (device order)
        pm.local_search_multi_async(E_full, [p + ws_bytes for p in ptrs], ptrs, rank, world, res)
        if evs: evs[3].record(stream)
        pm.cost_async(E_full, my_perm, cost)
        if evs: evs[4].record(stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    ref = res.cpu().tolist() + cost.cpu().tolist()
    K = args.steps
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(5)] for _ in range(K)]
    dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local_rank) as clk:
        for i in range(K):
            step(evs[i])
        torch.cuda.synchronize()
    dist.barrier()
    out = res.cpu().tolist() + cost.cpu().tolist()
    assert out == ref and out[0] == 0, f"sharded search {out} vs {ref}"
    tot = [ev[0].elapsed_time(ev[4]) for ev in evs]
    ms = pdist.max_over_ranks(statistics.mean(tot), device=dev)
    part_ms = {k: statistics.mean([ev[i].elapsed_time(ev[i + 1]) for ev in evs])
               for k, i in (("error_matrix_shard", 0), ("all_gather", 1), ("local_search_multi", 2), ("cost", 3))}
    return {
        "metric": METRIC, "value": S * S / (ms * 1e-3) / 1e9, "unit": UNIT, "n_gpus": world, "steps": K,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "u8->int32", "data": "synthetic",
        "config": dict(workload_desc(args.config, args.family, [0]), method="trap (multi-rank)",
                       parallelism=f"E rows sharded over {world} ranks + all-gather; Alg. 2 across ranks",
                       l2="not flushed (E of the sharded configs exceeds L2)"),
        "breakdown_ms_rank0": part_ms,
        "result": {"rounds": out[1], "swaps": out[2], "cost": out[3]},
        "clocks": clk.summary(),
    }

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
    if args.sharded:
        line = bench_sharded(args, rank, world, local_rank)
        if rank == 0:
            line["host"] = host_info()
            print(json.dumps(line), flush=True)
        if world > 1:
            dist.barrier()
            dist.destroy_process_group()
        return
    line, extra = bench_ours(args, rank, world, local_rank)
    if rank == 0:
        if world == 1 and not args.no_cpu_baseline:
            I_np, T_np, M, S, perm_np, out_res = extra
            cb, ref = cpu_baseline(I_np, T_np, M, S, args.cpu_seconds)
            line["cpu_baseline"] = cb
            line["parity_vs_oracle"] = bool((ref["r"] == perm_np).all() and ref["rounds"] == out_res[1]
                                            and ref["swaps"] == out_res[2] and ref["cost"] == out_res[3])
        line["host"] = host_info()
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def main_reference(args, rank, world):
    """The reference arm: the CPU oracle (oracle/), as it stands, on this
    box's host cores, same workload/metric; rank 0 only."""
    if rank != 0:
        return
    from paper_conf_ipps_yangin17_b200 import synth
    import oracle
    oracle.build()
    cfg = synth.CONFIGS[args.config]
    N, M, C = cfg["N"], cfg["M"], cfg["C"]
    S = (N // M) ** 2
    I, T = synth.make_pair(args.family, N, M, C, seed=0)
    for _ in range(min(args.warmup, 3)):
        run_oracle_once(I, T, M)
    times = [run_oracle_once(I, T, M)[0] for _ in range(args.steps)]
    mean = statistics.mean(times)
    value = S * S / mean / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": mean * 1e3, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u8->int32", "data": "synthetic",
        "config": dict(workload_desc(args.config, args.family, [0]), method="oracle (CPU)"),
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": oracle.num_threads(), "kind": "oracle",
                         "sample": f"the full workload per step x {args.steps} steps"},
        "host": host_info(),
    }
    print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()
