"""Experiment: can the NCCL pipeline path (sq_comm_init + sq_pipeline_run with rank >= 0) run with
several ranks on ONE GPU (gpurun boxes have one)?  NCCL normally rejects duplicate devices in one
communicator; this prints what happens.  python tools/dup_gpu_nccl.py [world]"""
import os
import socket
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def worker(rank, world, port):
    import torch
    import torch.distributed as dist
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_cluster_zhaowplw25_b200.selfcheck import pipeline_bitwise_check
    try:
        r = pipeline_bitwise_check(rank, world, dist)
        print(f"rank {rank}: {r}", flush=True)
    except Exception as e:  # noqa: BLE001
        print(f"rank {rank}: FAILED {type(e).__name__}: {e}", flush=True)
        os._exit(3)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    import torch.multiprocessing as mp
    world = int(sys.argv[1]) if len(sys.argv) > 1 else 2
    mp.start_processes(worker, args=(world, _port()), nprocs=world, join=True, start_method="spawn")
