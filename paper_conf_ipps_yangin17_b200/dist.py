"""Multi-GPU plumbing (one process per GPU, torch.distributed).

Step 2 (the error matrix, Eq. 1) shards naturally by input-tile rows:
rank g computes rows [row_begin, row_end) of E against all S target tiles
(`pm_error_matrix(row_begin, row_end)`, no exchange).  Algorithm 2's colour
classes are global perfect matchings, so the search itself is
one job across the ranks, exchanging chunk-boundary slots over peer memory:

* `local_search_multi`: every rank holds all of E (gathered with
  `error_matrix_sharded(..., gather=True)`), sparse rounds included;
* `photomosaic_sharded` / `local_search_sharded`: E stays row-sharded in
  symmetric memory and every rank reads the rows it needs from their owner
  over NVLink (no rank holds all of E: the layout for matrices larger than
  one GPU).

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


def _symm_alloc(nbytes: int, device, group):
    import torch.distributed._symmetric_memory as symm_mem
    buf = symm_mem.empty(nbytes, dtype=torch.uint8, device=device)
    hdl = symm_mem.rendezvous(buf, (group or dist.group.WORLD).group_name)
    return buf, [int(p) for p in hdl.buffer_ptrs]


def _sharded_layout(S: int, world: int):
    from . import pm
    bounds = [shard_rows(S, world, g) for g in range(world)]
    rows_max = max(e - b for b, e in bounds)
    ws = (pm.trap_workspace_bytes_sharded(S, rows_max) + 255) // 256 * 256
    pb = (4 * S + 255) // 256 * 256
    return [b for b, _ in bounds] + [S], rows_max, ws, pb


def _run_sharded(buf, ptrs, S: int, perm, max_rounds: int, group):
    from . import pm
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    rb, rows_max, ws, pb = _sharded_layout(S, world)
    my_perm = buf[ws:ws + 4 * S].view(torch.int32)
    my_perm.copy_(torch.arange(S, dtype=torch.int32, device=buf.device) if perm is None else perm)
    buf[:ws].zero_()
    torch.cuda.synchronize(buf.device)
    dist.barrier(group)                                   # every workspace reset, every shard written
    result = torch.zeros(3, dtype=torch.int64, device=buf.device)
    pm.local_search_sharded_async([p + ws + pb for p in ptrs], rb, S, S, [p + ws for p in ptrs], ptrs, rank, world,
                                  result, max_rounds=max_rounds)
    torch.cuda.synchronize(buf.device)
    dist.barrier(group)                                   # no rank frees its buffer while peers may read it
    status, rounds, swaps = (int(v) for v in result.tolist())
    if status not in (0, 3):
        raise pm.PMError(status, "pm_local_search_sharded_async")
    out = my_perm.clone()
    if perm is not None:
        perm.copy_(out)
        out = perm
    return out, rounds, swaps


def local_search_sharded(E_part: torch.Tensor, S: int, perm: torch.Tensor | None = None, max_rounds: int = 0,
                         group=None):
    """Algorithm 2 across the ranks over ROW-SHARDED E with
    pm_local_search_sharded_async: E_part = this rank's rows
    shard_rows(S, world, rank) of E (e.g. error_matrix_sharded's part).  The
    shard is copied into symmetric memory next to the workspace and perm;
    every rank returns the final r.  Returns (perm, rounds, swaps)."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    rb, rows_max, ws, pb = _sharded_layout(S, world)
    b, e = rb[rank], rb[rank + 1]
    if tuple(E_part.shape) != (e - b, S):
        raise ValueError(f"rank {rank} expects E rows [{b}, {e}) x {S}, got {tuple(E_part.shape)}")
    buf, ptrs = _symm_alloc(ws + pb + 4 * rows_max * S, E_part.device, group)
    buf[ws + pb:ws + pb + 4 * (e - b) * S].view(torch.int32).view(e - b, S).copy_(E_part)
    return _run_sharded(buf, ptrs, S, perm, max_rounds, group)


def photomosaic_sharded(I, T, M: int, perm: torch.Tensor | None = None, max_rounds: int = 0, group=None):
    """Steps 2-3 across the ranks with E never gathered: rank g writes its
    rows of E (pm_error_matrix) straight into its symmetric-memory shard,
    then Algorithm 2 runs over the shards (local_search_sharded).  Returns
    (perm, rounds, swaps)."""
    from . import pm
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    N = I.shape[0]
    S = (N // M) ** 2
    rb, rows_max, ws, pb = _sharded_layout(S, world)
    b, e = rb[rank], rb[rank + 1]
    buf, ptrs = _symm_alloc(ws + pb + 4 * rows_max * S, I.device, group)
    if e > b:
        pm.error_matrix(I, T, M, rows=(b, e), out=buf[ws + pb:ws + pb + 4 * (e - b) * S].view(torch.int32).view(e - b, S))
    return _run_sharded(buf, ptrs, S, perm, max_rounds, group)

