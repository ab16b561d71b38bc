"""Multi-GPU pipeline (a6) over NCCL: bitwise equal to the single-process virtual pipeline.

SURVEY.md 8(c) O7 / 8(e): the P-rank NCCL run (uneven contiguous stages, micro-batched prefill and
decode, last -> first loop-back) must reproduce ``sq_comm_init_local``'s virtual pipeline bit for bit.
Needs >= 2 GPUs (skipped otherwise: gpurun boxes have one).  Also: ``bench.py --gpus N`` without
torchrun must launch N ranks itself or fail loudly -- never measure fewer GPUs than asked for.
"""
from __future__ import annotations

import json
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank: int, world: int, port: int, q) -> None:
    import torch
    import torch.distributed as dist
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(rank)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_cluster_zhaowplw25_b200.selfcheck import pipeline_bitwise_check
    r = pipeline_bitwise_check(rank, world, dist)
    if rank == 0:
        q.put(r)
    dist.barrier()
    dist.destroy_process_group()


def _n_gpus() -> int:
    import torch
    return torch.cuda.device_count() if torch.cuda.is_available() else 0


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 3])
def test_nccl_pipeline_bitwise_equals_virtual(world):
    if _n_gpus() < world:
        pytest.skip(f"needs {world} GPUs")
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    mp.start_processes(_worker, args=(world, _free_port(), q), nprocs=world, join=True, start_method="spawn")
    r = q.get(timeout=10)
    assert r["pipeline_bitwise_ok"], r


def test_bench_gpus_n_never_measures_fewer_gpus():
    """Without enough visible GPUs `bench.py --gpus N` exits non-zero with an error line naming the
    requested and active counts (CPU here: 0 devices)."""
    if _n_gpus() >= 4:
        pytest.skip("enough GPUs: the spawn path would run the real bench")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4", "--steps", "1"],
                       capture_output=True, text=True, timeout=600, env={k: v for k, v in os.environ.items()
                                                                         if k not in ("WORLD_SIZE", "RANK")})
    assert r.returncode != 0
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["n_gpus"] == 4 and line["gpus_active"] < 4 and "error" in line
