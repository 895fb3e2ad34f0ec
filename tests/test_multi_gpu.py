"""The multi-GPU bench path on real GPUs: one photomosaic across 2 ranks
(torchrun, NCCL, torch symmetric memory, pm_local_search_multi_async over
peer memory, or pm_local_search_sharded_async over row-sharded E) must reproduce the oracle's result.  Runs only where at least
two GPUs are visible (this build's GPU runs have one; the emulated-rank tests
in test_gpu_parity*.py cover the protocol there)."""
import json
import os
import subprocess
import sys

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.skipif(not torch.cuda.is_available() or torch.cuda.device_count() < 2, reason="needs >= 2 GPUs")
@pytest.mark.parametrize("layout", ["gathered", "rows"])
@pytest.mark.parametrize("cfg", [2, 3])
def test_sharded_bench_two_ranks_matches_oracle(cfg, layout):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(29600 + cfg + (10 if layout == "rows" else 0)),
           os.path.join(ROOT, "bench.py"), "--gpus", "2", "--config", str(cfg), "--steps", "3", "--warmup", "3",
           "--e2e-steps", "1", "--e-layout", layout]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads([ln for ln in out.stdout.splitlines() if ln.startswith("{")][-1])
    assert line["n_gpus"] == 2 and line["scaling"] == "strong"
    assert line["parity_vs_oracle"] is True


@pytest.mark.skipif(not torch.cuda.is_available(), reason="needs a GPU")
def test_rows_layout_bench_one_rank_matches_oracle():
    # the row-sharded bench path at N = 1 (symmetric memory, world 1): the
    # same JSON contract and parity against the oracle
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--config", "2", "--steps", "3", "--warmup", "3",
           "--e2e-steps", "1", "--e-layout", "rows", "--no-cpu-baseline"]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads([ln for ln in out.stdout.splitlines() if ln.startswith("{")][-1])
    assert line["n_gpus"] == 1 and line["parity_vs_oracle"] is True
    assert "row-sharded" in line["config"]["method"] and line["gpu_launches"] > 0

