"""Multi-GPU plumbing (one process per GPU, torch.distributed).

Step 2 (the error matrix, Eq. 1) shards naturally by input-tile rows:
rank g computes rows [row_begin, row_end) of E against all S target tiles
(`pm_error_matrix(row_begin, row_end)`, no exchange).  Algorithm 2 does not
shard (every colour class is a global perfect matching), so a
job either

* runs independent photomosaics, one per rank (the benchmark: weak scaling,
  no data-path collective), or
* computes E row-sharded and all-gathers it when every rank needs the full
  matrix (`error_matrix_sharded(..., gather=True)`).

Everything here is host-side marshalling around `pm` calls and
torch.distributed collectives; no compute happens in Python.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard_rows(S: int, world: int, rank: int) -> tuple[int, int]:
    """Balanced contiguous row range of rank `rank` out of `world` (sizes
    differ by at most one row; every row owned exactly once)."""
    if world < 1 or not (0 <= rank < world) or S < 0:
        raise ValueError("bad shard request")
    q, r = divmod(S, world)
    begin = rank * q + min(rank, r)
    return begin, begin + q + (1 if rank < r else 0)


def gather_rows(shard: torch.Tensor, S: int, group=None) -> torch.Tensor:
    """All-gather row shards (rank order, sizes from shard_rows) into the
    full [S, cols] matrix on every rank."""
    world = dist.get_world_size(group)
    sizes = [shard_rows(S, world, g) for g in range(world)]
    rows_max = max(e - b for b, e in sizes)
    cols = shard.shape[1]
    pad = torch.zeros((rows_max, cols), dtype=shard.dtype, device=shard.device)
    pad[: shard.shape[0]] = shard
    parts = [torch.empty_like(pad) for _ in range(world)]
    dist.all_gather(parts, pad, group=group)
    return torch.cat([p[: e - b] for p, (b, e) in zip(parts, sizes)], dim=0)


def error_matrix_sharded(I, T, M: int, gather: bool = False, group=None):
    """Row shard of E for this rank via pm_error_matrix (CUDA); optionally
    all-gathered.  Returns (E_part_or_full, (row_begin, row_end))."""
    from . import pm
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    N = I.shape[0]
    S = (N // M) ** 2
    rows = shard_rows(S, world, rank)
    part = pm.error_matrix(I, T, M, rows=rows)
    if gather and world > 1:
        return gather_rows(part, S, group), rows
    return part, rows


def max_over_ranks(value: float, device=None, group=None) -> float:
    """Max of a per-rank scalar (the benchmark's time: max over ranks)."""
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def sum_over_ranks(value: float, device=None, group=None) -> float:
    if not dist.is_initialized() or dist.get_world_size(group) == 1:
        return float(value)
    t = torch.tensor([float(value)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return float(t.item())


def local_search_multi(E: torch.Tensor, perm: torch.Tensor | None = None, max_rounds: int = 0, group=None):
    """Algorithm 2 across the ranks of `group` (one per GPU of one NVLink box)
    with pm_local_search_multi_async: every rank passes the full E
    (replicated, e.g. from error_matrix_sharded(..., gather=True)) and the
    same initial perm; every rank returns the final r.  The per-rank
    workspaces and perms live in torch symmetric memory, so each rank sees
    the others' as peer pointers.  Returns (perm, rounds, swaps)."""
    import torch.distributed._symmetric_memory as symm_mem

    from . import pm
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    S = E.shape[0]
    ws_bytes = (pm.trap_workspace_bytes(S) + 255) // 256 * 256
    buf = symm_mem.empty(ws_bytes + 4 * S, dtype=torch.uint8, device=E.device)
    name = (group or dist.group.WORLD).group_name
    hdl = symm_mem.rendezvous(buf, name)
    ptrs = [int(p) for p in hdl.buffer_ptrs]
    my_perm = buf[ws_bytes:].view(torch.int32)
    my_perm.copy_(torch.arange(S, dtype=torch.int32, device=E.device) if perm is None else perm)
    buf[:ws_bytes].zero_()
    torch.cuda.synchronize(E.device)
    dist.barrier(group)                                   # every workspace reset before any rank starts
    result = torch.zeros(3, dtype=torch.int64, device=E.device)
    pm.local_search_multi_async(E, [p + ws_bytes for p in ptrs], ptrs, rank, world, result, max_rounds=max_rounds)
    torch.cuda.synchronize(E.device)
    dist.barrier(group)                                   # no rank frees its buffer while peers may write it
    status, rounds, swaps = (int(v) for v in result.tolist())
    if status not in (0, 3):
        raise pm.PMError(status, "pm_local_search_multi_async")
    out = my_perm.clone()
    if perm is not None:
        perm.copy_(out)
        out = perm
    return out, rounds, swaps
