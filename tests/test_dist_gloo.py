"""World-size-2 gloo tests (CPU) of the multi-GPU host logic in
paper_conf_ipps_yangin17_b200/dist.py: row sharding of E (Step 2), the
all-gather of shards, and the max/sum-over-ranks used by bench.py.  Each rank
computes its E shard with the oracle (test infrastructure) so the sharding
and gather logic are checked without a GPU."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_yangin17_b200 import dist as pdist


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("S,world", [(0, 1), (1, 2), (7, 2), (256, 2), (1024, 8), (65536, 8), (13, 5)])
def test_shard_rows_partition(S, world):
    spans = [pdist.shard_rows(S, world, r) for r in range(world)]
    assert spans[0][0] == 0 and spans[-1][1] == S
    for (b0, e0), (b1, e1) in zip(spans, spans[1:]):
        assert e0 == b1
    sizes = [e - b for b, e in spans]
    assert max(sizes) - min(sizes) <= 1


def test_shard_rows_rejects_bad():
    with pytest.raises(ValueError):
        pdist.shard_rows(10, 0, 0)
    with pytest.raises(ValueError):
        pdist.shard_rows(10, 2, 2)


def _worker(rank, world, port, out_dir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ipps_yangin17_b200 import synth
        N, M = 90, 10                      # S = 81: uneven shards (41 + 40)
        I, T = synth.make_pair("smooth", N, M, 3, seed=5)
        S = (N // M) ** 2
        b, e = pdist.shard_rows(S, world, rank)
        part = torch.from_numpy(oracle.error_matrix(I, T, M, rows=(b, e)))
        full = pdist.gather_rows(part, S)
        np.save(os.path.join(out_dir, f"E_{rank}.npy"), full.numpy())
        mx = pdist.max_over_ranks(float(rank + 1) * 1.5)
        sm = pdist.sum_over_ranks(float(rank + 1))
        np.save(os.path.join(out_dir, f"agg_{rank}.npy"), np.array([mx, sm]))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_sharded_error_matrix(tmp_path):
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    import oracle
    from paper_conf_ipps_yangin17_b200 import synth
    I, T = synth.make_pair("smooth", 90, 10, 3, seed=5)
    ref = oracle.error_matrix(I, T, 10)
    for r in range(world):
        assert (np.load(tmp_path / f"E_{r}.npy") == ref).all()
        mx, sm = np.load(tmp_path / f"agg_{r}.npy")
        assert mx == 3.0 and sm == 3.0
