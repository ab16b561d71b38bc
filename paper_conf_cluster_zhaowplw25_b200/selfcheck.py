"""Multi-GPU self-verification of the NCCL pipeline (a6) against the single-process virtual pipeline.

Every kernel of the path is deterministic (fixed-order reductions, fixed launch configurations per
shape), and a stage computes the same micro-batches on the same rows whether its neighbours live on
other GPUs (NCCL point-to-point) or on the same device (``sq_comm_init_local``).  So the P-rank run
must equal the virtual pipeline BITWISE (SURVEY.md 8(c) O7 pin).  This module
runs a configs[0]-sized generation (OPT-125m shapes, 12 layers, mixed bits, micro-batched prefill
and decode, an uneven partition) over the NCCL path on every rank and compares the last rank's
output with the virtual pipeline recomputed on that rank.  It is called by ``bench.py`` before the
timed region at N > 1 and by ``tests/test_gpu_multi.py``; it never touches the oracle.
"""
from __future__ import annotations

import torch

H1, H2, L = 768, 3072, 12


def uneven_partition(n_layers: int, P: int) -> list[int]:
    """Contiguous, deliberately uneven stage sizes (stage 0 one layer short, the last one longer)."""
    base = [n_layers // P] * P
    for i in range(n_layers % P):
        base[P - 1 - i] += 1
    if P > 1 and base[0] > 1:
        base[0] -= 1
        base[-1] += 1
    sol = []
    for s, c in enumerate(base):
        sol += [s] * c
    return sol


def pipeline_bitwise_check(rank: int, world: int, dist, B: int = 5, eta: int = 2, xi: int = 2, s: int = 16,
                           n_dec: int = 3) -> dict:
    """Run on every rank of an initialised torch.distributed group (any backend; only used for the
    NCCL unique-id broadcast and the verdict).  Returns {"pipeline_bitwise_ok": bool, ...} on every rank."""
    import synth
    from . import runtime as R

    assert 1 < world <= L
    bits = [int(b) for b in synth.bits_plan(2, L)]
    sol = uneven_partition(L, world)
    plan = R.Plan(bits, sol, H1, H2, B, eta, xi, s, n_dec)
    R.sq_plan_check(plan)
    mine = plan.layers_of(rank)
    layers = R.build_layers(len(mine), H1, H2, [bits[l] for l in mine], layer_offset=mine[0])
    uid = [R.sq_comm_get_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(uid, src=0)
    comm = R.Comm.nccl(uid[0], world, rank)
    x0 = out = None
    if rank == 0:
        x0 = torch.empty((B, s, H1), dtype=torch.float32, device="cuda")
        synth.device_fill_f32(x0.data_ptr(), 77, 0, x0.numel(), 1.0, False)
    if rank == world - 1:
        out = torch.full((B, 1 + n_dec, H1), float("nan"), dtype=torch.float32, device="cuda")
    ws = R.PipelineWorkspace(plan, layers, rank)
    st = R.sq_pipeline_run(plan, rank, layers, comm, x0, out, ws)
    torch.cuda.synchronize()
    comm.destroy()
    ok, diff = 1, 0.0
    if rank == world - 1:
        every = R.build_layers(L, H1, H2, bits)
        xv = torch.empty((B, s, H1), dtype=torch.float32, device="cuda")
        synth.device_fill_f32(xv.data_ptr(), 77, 0, xv.numel(), 1.0, False)
        ref = torch.full_like(out, float("nan"))
        lc = R.Comm.local(world)
        R.sq_pipeline_run(plan, -1, every, lc, xv, ref, R.PipelineWorkspace(plan, every, -1))
        torch.cuda.synchronize()
        lc.destroy()
        ok = int(torch.equal(out, ref))
        diff = float((out - ref).abs().max().item()) if torch.isfinite(out).all() else float("inf")
    t = torch.tensor([ok], dtype=torch.int32)
    dist.all_reduce(t, op=dist.ReduceOp.MIN)
    return {"pipeline_bitwise_ok": bool(t.item()), "P": world, "stage_sizes": [sol.count(r) for r in range(world)],
            "max_abs_diff_last_rank": diff, "bytes_sent_rank": st["bytes_sent"],
            "case": f"OPT-125m shapes, {L} layers, B={B}, eta={eta}, xi={xi}, prompt {s}, {n_dec} decode steps"}
