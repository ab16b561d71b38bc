"""Host side of the P x tp mesh (intra-node TP inside pipeline stages, P:63, P:236,
P:318 TP2+PP2): the schedule every global rank executes (sq_pipeline_schedule with plan.tp > 1), the
plan checks, and a gloo world-size-4 run (2 stages x TP2) of that schedule with the oracle's arithmetic
and the in-place all-reduce of sq_stage_forward_tp, against the unsharded oracle pipeline O7.
CPU only (libsq loads without a GPU)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest


def R():
    from paper_conf_cluster_zhaowplw25_b200 import runtime as RT
    return RT


def mesh_plan(P, tp, L=6, B=5, eta=3, xi=2, s=3, n_dec=3, h1=256, h2=512, n_heads=0):
    from paper_conf_cluster_zhaowplw25_b200 import plan as PL
    bits = [3, 4, 8, 16, 4, 3][:L]
    sol = PL.partition_layers([1.0] * L, P)
    return R().Plan(bits, sol, h1, h2, B, eta, xi, s, n_dec, n_heads=n_heads, tp=tp)


@pytest.mark.parametrize("P,tp", [(1, 2), (2, 2), (3, 2), (2, 4), (4, 2)])
def test_mesh_schedule_rings(P, tp):
    plan = mesh_plan(P, tp, h1=128 * tp, h2=256 * tp)
    R().sq_plan_check(plan)
    flat = mesh_plan(P, 1, h1=128 * tp, h2=256 * tp)
    for g in range(P * tp):
        p, j = divmod(g, tp)
        sched = R().sq_pipeline_schedule(plan, g)
        ref = R().sq_pipeline_schedule(flat, p)
        # the rank runs its stage's plain-pipeline schedule, with every peer moved onto ring j
        assert len(sched) == len(ref)
        for a, b in zip(sched, ref):
            assert {k: v for k, v in a.items() if k != "peer"} == {k: v for k, v in b.items() if k != "peer"}
            assert a["peer"] == (-1 if b["peer"] < 0 else b["peer"] * tp + j)
    # sends of (p, j) -> (p+1, j) equal the receives of (p+1, j) from (p, j), size for size
    for g in range(P * tp):
        p, j = divmod(g, tp)
        sched = R().sq_pipeline_schedule(plan, g)
        for peer in {o["peer"] for o in sched if o["kind"] in ("SEND_ACT", "SEND_LB")}:
            assert peer % tp == j
            sends = [o["rows"] for o in sched if o["kind"] in ("SEND_ACT", "SEND_LB") and o["peer"] == peer]
            recvs = [o["rows"] for o in R().sq_pipeline_schedule(plan, peer)
                     if o["kind"] in ("RECV_ACT", "RECV_LB") and o["peer"] == g]
            assert sends == recvs
    with pytest.raises(ValueError):
        R().sq_pipeline_schedule(plan, P * tp)


@pytest.mark.parametrize("tp,h1,h2,heads", [(2, 384, 512, 0), (3, 384, 768, 0), (2, 256, 512, 3), (4, 512, 1024, 6)])
def test_plan_check_tp_divisibility(tp, h1, h2, heads):
    # hidden and ffn multiples of 128 tp; n_heads divisible by tp
    from paper_conf_cluster_zhaowplw25_b200 import SQError
    plan = mesh_plan(2, tp, h1=h1, h2=h2, n_heads=heads)
    ok = h1 % (128 * tp) == 0 and h2 % (128 * tp) == 0 and heads % tp == 0
    if heads:
        ok = ok and h1 // heads in (64, 128)
    if ok:
        R().sq_plan_check(plan)
    else:
        with pytest.raises(SQError):
            R().sq_plan_check(plan)


# ---------------------------------------------------------------- gloo world 4 = 2 stages x TP2
def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _oracle_full_and_shards(plan):
    import synth
    from oracle import oracle as O
    h1, h2, T = plan.hidden, plan.ffn, plan.tp
    full, sets = [], [[] for _ in range(T)]
    for l, b in enumerate(plan.bits):
        qf, qs = {}, [{} for _ in range(T)]
        for name, (n, k) in {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}.items():
            seed = synth.weight_seed(l, name)
            w, bias = synth.weight_f16(seed, n, k), synth.bias_f16(seed, n)
            qf[name] = O.QWeight(w, b, bias=bias)
            for r in range(T):
                ws, bs = O.tp_shard(name, w, bias, r, T)
                qs[r][name] = O.QWeight(ws, b, bias=bs)
        full.append(O.Layer(b, 0, qf["qkv"], qf["o"], qf["fc1"], qf["fc2"]))
        for r in range(T):
            sets[r].append(O.Layer(b, 0, qs[r]["qkv"], qs[r]["o"], qs[r]["fc1"], qs[r]["fc2"]))
    x0 = synth.hidden_f32(1, plan.B * plan.prompt_len, h1).reshape(plan.B, plan.prompt_len, h1).astype(np.float64)
    return full, sets, x0


def _mesh_worker(rank, P, tp, port, q):
    import torch
    import torch.distributed as dist
    from oracle import oracle as O
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=P * tp)
    groups = [dist.new_group(list(range(p * tp, (p + 1) * tp))) for p in range(P)]
    plan = mesh_plan(P, tp)
    _, sets, x0 = _oracle_full_and_shards(plan)
    stage, j = divmod(rank, tp)
    mine = [sets[j][l] for l in plan.layers_of(rank)]
    grp = groups[stage]

    def allreduce(a):
        t = torch.from_numpy(np.ascontiguousarray(a))
        dist.all_reduce(t, group=grp)
        return t.numpy().copy()

    def tp_stage(x):
        # sq_stage_forward_tp's order: rank j = 0 contributes x + p_0, the others p_j; one sum per sub-layer
        x = np.array(x, np.float64)
        for Ly in mine:
            hs = Ly.o.k
            p = O.linear(O.linear(O.layernorm(x), Ly.qkv)[:, 2 * hs:3 * hs], Ly.o)
            x = allreduce(x + p if j == 0 else p)
            p = O.linear(np.maximum(O.linear(O.layernorm(x), Ly.fc1), 0.0), Ly.fc2)
            x = allreduce(x + p if j == 0 else p)
        return x

    h1, s, B = plan.hidden, plan.prompt_len, plan.B
    dec_in = np.zeros((B, h1))
    out = np.zeros((B, 1 + plan.n_decode, h1))
    bufs, pending = {}, []
    for o in R().sq_pipeline_schedule(plan, rank):
        k = o["kind"]
        if k == "RECV_LB":
            t = torch.empty((o["nseq"], h1), dtype=torch.float64)
            dist.recv(t, src=o["peer"])
            dec_in[o["seq0"]:o["seq0"] + o["nseq"]] = t.numpy()
        elif k == "RECV_ACT":
            t = torch.empty((o["rows"], h1), dtype=torch.float64)
            dist.recv(t, src=o["peer"])
            bufs[o["slot"]] = t.numpy()
        elif k == "COMPUTE":
            if stage == 0:
                xin = (x0[o["seq0"]:o["seq0"] + o["nseq"]].reshape(-1, h1) if o["phase"] == 0
                       else dec_in[o["seq0"]:o["seq0"] + o["nseq"]])
            else:
                xin = bufs[o["slot"]]
            bufs[o["slot"]] = tp_stage(xin)
        elif k == "SEND_ACT":
            pending.append(dist.isend(torch.from_numpy(np.ascontiguousarray(bufs[o["slot"]])), dst=o["peer"]))
        elif k in ("OUT", "SEND_LB"):
            b = bufs[o["slot"]]
            rows = b.reshape(o["nseq"], s, h1)[:, -1] if o["phase"] == 0 else b
            if k == "OUT":
                out[o["seq0"]:o["seq0"] + o["nseq"], o["t"]] = rows
            else:
                pending.append(dist.isend(torch.from_numpy(np.ascontiguousarray(O.layernorm(rows))), dst=o["peer"]))
    for p_ in pending:
        p_.wait()
    if stage == P - 1:
        q.put((j, out))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_mesh_2x2_matches_unsharded_pipeline():
    import multiprocessing as mp
    from oracle import oracle as O
    P, tp = 2, 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_mesh_worker, args=(r, P, tp, port, q)) for r in range(P * tp)]
    for p_ in procs:
        p_.start()
    outs = dict(q.get(timeout=600) for _ in range(tp))
    for p_ in procs:
        p_.join(timeout=120)
        assert p_.exitcode == 0
    plan = mesh_plan(P, tp)
    full, _, x0 = _oracle_full_and_shards(plan)
    ref = O.pipeline(full, x0, plan.n_decode)
    assert np.array_equal(outs[0], outs[1])     # both TP ranks of the last stage hold the same rows
    assert np.abs(outs[0] - ref).max() / np.abs(ref).max() <= 1e-12
