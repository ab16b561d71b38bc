"""Host-side pipeline schedule (sq_pipeline_schedule, the op list sq_pipeline_run executes):
send/recv matching across ranks and a gloo world-size-2 execution against the oracle.
CPU only (libsq loads without a GPU; compute uses the oracle stage)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest


def R():
    from paper_conf_cluster_zhaowplw25_b200 import runtime as RT
    return RT


def plan_for(P, L=8, B=6, eta=4, xi=4, s=3, n_dec=3, h1=128, h2=512, bits=None):
    from paper_conf_cluster_zhaowplw25_b200 import plan as PL
    bits = bits or [3, 4, 8, 16] * (L // 4)
    sol = PL.partition_layers([1.0 + (b == 16) for b in bits], P)
    return R().Plan(bits, sol, h1, h2, B, eta, xi, s, n_dec)


@pytest.mark.parametrize("P", [2, 3, 4, 5, 8])
@pytest.mark.parametrize("shape", [(6, 4, 4, 3), (32, 8, 32, 5), (7, 3, 2, 1)])
def test_sends_match_receives_in_order(P, shape):
    # every link j -> j+1 (mod P) carries the same sequence of message sizes on both ends,
    # so NCCL point-to-point operations pair up one-to-one (no mismatch, no deadlock)
    B, eta, xi, n_dec = shape
    plan = plan_for(P, B=B, eta=eta, xi=xi, n_dec=n_dec)
    sched = {r: R().sq_pipeline_schedule(plan, r) for r in range(P)}
    for j in range(P):
        nxt = (j + 1) % P
        sends = [(o["rows"]) for o in sched[j] if o["kind"] in ("SEND_ACT", "SEND_LB") and o["peer"] == nxt]
        recvs = [(o["rows"]) for o in sched[nxt] if o["kind"] in ("RECV_ACT", "RECV_LB") and o["peer"] == j]
        assert sends == recvs, (j, sends[:5], recvs[:5])
    # every item is computed exactly once per stage, in the same order everywhere
    items = [[o["item"] for o in sched[r] if o["kind"] == "COMPUTE"] for r in range(P)]
    assert all(it == list(range(len(items[0]))) for it in items)
    mu_pre, mu_dec = -(-B // eta), -(-B // xi)
    assert len(items[0]) == mu_pre + n_dec * mu_dec           # eq. (4): mu_pre + n_dec*mu_dec items
    lb = [o for o in sched[0] if o["kind"] == "RECV_LB"]
    assert len(lb) == mu_pre + (n_dec - 1) * mu_dec           # last step's loop-back is not sent


def test_loopback_received_before_use():
    plan = plan_for(4, B=10, eta=4, xi=3, n_dec=4)
    ready = np.zeros(10, bool)
    for o in R().sq_pipeline_schedule(plan, 0):
        if o["kind"] == "RECV_LB":
            ready[o["seq0"]:o["seq0"] + o["nseq"]] = True
        if o["kind"] == "COMPUTE" and o["phase"] == 1:
            assert ready[o["seq0"]:o["seq0"] + o["nseq"]].all(), o


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    from oracle import oracle as O
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from test_pipeline_schedule import plan_for, oracle_model
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    plan = plan_for(world)
    layers, x0 = oracle_model(plan)
    mine = [layers[l] for l in plan.layers_of(rank)]
    h1, s, B = plan.hidden, plan.prompt_len, plan.B
    dec_in = np.zeros((B, h1))
    out = np.zeros((B, 1 + plan.n_decode, h1))
    bufs = {}
    pending = []
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
            if rank == 0:
                xin = (x0[o["seq0"]:o["seq0"] + o["nseq"]].reshape(-1, h1) if o["phase"] == 0
                       else dec_in[o["seq0"]:o["seq0"] + o["nseq"]])
            else:
                xin = bufs[o["slot"]]
            bufs[o["slot"]], _ = O.stage(mine, xin)
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
    if rank == world - 1:
        q.put(out)
    dist.barrier()
    dist.destroy_process_group()


def oracle_model(plan):
    import synth
    from oracle import oracle as O
    h1, h2 = plan.hidden, plan.ffn
    layers = []
    for l, b in enumerate(plan.bits):
        qs = {}
        for name, (n, k) in {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}.items():
            seed = synth.weight_seed(l, name)
            qs[name] = O.QWeight(synth.weight_f16(seed, n, k), b, bias=synth.bias_f16(seed, n))
        layers.append(O.Layer(b, 0, qs["qkv"], qs["o"], qs["fc1"], qs["fc2"]))
    x0 = synth.hidden_f32(1, plan.B * plan.prompt_len, h1).reshape(plan.B, plan.prompt_len, h1).astype(np.float64)
    return layers, x0


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_world_executes_schedule_like_the_oracle(world):
    """world 2 and an odd stage count (3): the ring's wrap link joins two even ranks."""
    import multiprocessing as mp
    from oracle import oracle as O
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p_ in procs:
        p_.start()
    out = q.get(timeout=600)
    for p_ in procs:
        p_.join(timeout=120)
        assert p_.exitcode == 0
    plan = plan_for(world)
    layers, x0 = oracle_model(plan)
    ref = O.pipeline(layers, x0, plan.n_decode)
    assert np.array_equal(out, ref)   # rows are independent: bitwise, whatever the partition


@pytest.mark.parametrize("P", [1, 2, 3])
@pytest.mark.parametrize("kappa", [2, 4])
def test_chunked_prefill_schedule(P, kappa):
    # P:200 chunked prefill: mu_pre * kappa prefill items of eta sequences x s/kappa tokens; only a
    # micro-batch's last chunk produces its output row / loop-back; links still pair up one-to-one
    B, eta, xi, s, n_dec = 7, 3, 4, 8, 2
    from paper_conf_cluster_zhaowplw25_b200 import plan as PL
    bits = [4, 8, 3, 16] * 2
    sol = PL.partition_layers([1.0] * 8, P)
    plan = R().Plan(bits, sol, 768, 3072, B, eta, xi, s, n_dec, n_heads=12, kappa=kappa)
    R().sq_plan_check(plan)
    sched = {r: R().sq_pipeline_schedule(plan, r) for r in range(P)}
    mu_pre, mu_dec = -(-B // eta), -(-B // xi)
    comp = [o for o in sched[0] if o["kind"] == "COMPUTE"]
    assert len(comp) == mu_pre * kappa + n_dec * mu_dec
    pre = [o for o in comp if o["phase"] == 0]
    assert all(o["rows"] == o["nseq"] * (s // kappa) for o in pre)
    outs = [o for o in sched[P - 1] if o["kind"] == "OUT" and o["phase"] == 0]
    assert [o["item"] % kappa for o in outs] == [kappa - 1] * mu_pre
    for j in range(P if P > 1 else 0):
        nxt = (j + 1) % P
        sends = [o["rows"] for o in sched[j] if o["kind"] in ("SEND_ACT", "SEND_LB") and o["peer"] == nxt]
        recvs = [o["rows"] for o in sched[nxt] if o["kind"] in ("RECV_ACT", "RECV_LB") and o["peer"] == j]
        assert sends == recvs


def test_plan_check_attention_fields():
    import paper_conf_cluster_zhaowplw25_b200 as sq
    bad = [dict(n_heads=0, kappa=2), dict(n_heads=7, kappa=1), dict(n_heads=12, kappa=3), dict(n_heads=-1)]
    for kw in bad:
        plan = R().Plan([4, 4], [0, 0], 768, 3072, 2, 1, 2, 8, 2, **kw)
        with pytest.raises(sq.SQError):
            R().sq_plan_check(plan)
    R().sq_plan_check(R().Plan([4, 4], [0, 0], 768, 3072, 2, 1, 2, 8, 2, n_heads=6, kappa=4))  # dh 128
