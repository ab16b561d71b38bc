"""GPU parity of the tensor-parallel stage (sq_stage_forward_tp, R27)
against the oracle O10 / O6 on the same seeded weights.

Virtual TP (tp_rank -1: all T shard sets on the one GPU of the box, partial products accumulated in
rank order) for T = 2, 3, 4 on configs[0] shapes (OPT-125m), mixed bit-widths, prefill and decode,
stub and real attention; a row-parallel shard that spans a single group (k = 128); an OPT-66B-shaped
TP8 decode step on sampled rows; argument errors.  Tolerance normwise 2e-3 (R10).
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import synth
from oracle import oracle as O

pytestmark = pytest.mark.gpu
TOL = 2e-3


def nw(y, ref):
    y = np.asarray(y, np.float64)
    return float(np.abs(y - ref).max() / max(np.abs(ref).max(), 1e-30))


def sqm():
    import paper_conf_cluster_zhaowplw25_b200 as sq
    from paper_conf_cluster_zhaowplw25_b200 import runtime as R
    return sq, R


def _oracle_sets(L, h1, h2, bits, T, act=0):
    sets = [[] for _ in range(T)]
    for l in range(L):
        q = [{} for _ in range(T)]
        for name, (n, k) in {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}.items():
            seed = synth.weight_seed(l, name)
            w, b = synth.weight_f16(seed, n, k), synth.bias_f16(seed, n)
            for r in range(T):
                ws, bs = O.tp_shard(name, w, b, r, T)
                q[r][name] = O.QWeight(ws, int(bits[l]), bias=bs)
        for r in range(T):
            sets[r].append(O.Layer(int(bits[l]), act, q[r]["qkv"], q[r]["o"], q[r]["fc1"], q[r]["fc2"]))
    return sets


@pytest.mark.parametrize("T", [2, 3, 4])
@pytest.mark.parametrize("phase,tokens", [(0, 70), (1, 1), (1, 13), (1, 32)])
def test_tp_stage_stub(T, phase, tokens):
    sq, R = sqm()
    h1, h2, L = 768, 3072, 4
    if T == 4:
        h1, h2 = 1024, 4096
    bits = [4, 16, 3, 8]
    g = R.build_tp_layers(L, h1, h2, bits, T, act=phase)   # ReLU for prefill, GeLU for decode cases
    o = _oracle_sets(L, h1, h2, bits, T, act=phase)
    x = synth.hidden_f32(40 + tokens, tokens, h1)
    ws = R.TpWorkspace(g, tokens)
    xo = torch.empty((tokens, h1), dtype=torch.float32, device="cuda")
    R.sq_stage_forward_tp(g, phase, torch.from_numpy(x).cuda(), xo, ws, T)
    torch.cuda.synchronize()
    ref = O.stage_tp(o, x.astype(np.float64))
    assert nw(xo.cpu().numpy(), ref) <= TOL
    # in place (x_in aliases x_out) gives the same bits
    xi = torch.from_numpy(x).cuda()
    R.sq_stage_forward_tp(g, phase, xi, xi, ws, T)
    torch.cuda.synchronize()
    assert torch.equal(xi, xo)


def test_tp_equals_unsharded_gpu_stage_to_tolerance():
    # TP2 vs the TP1 (plain sq_stage_forward) run of the same layers: both within R10 of the oracle
    sq, R = sqm()
    h1, h2, L, T, tokens = 768, 3072, 3, 2, 9
    bits = [3, 4, 16]
    g1 = R.build_layers(L, h1, h2, bits)
    g2 = R.build_tp_layers(L, h1, h2, bits, T)
    x = torch.from_numpy(synth.hidden_f32(3, tokens, h1)).cuda()
    y1 = torch.empty_like(x)
    y2 = torch.empty_like(x)
    R.sq_stage_forward(g1, 1, x, y1, R.StageWorkspace(g1, tokens))
    R.sq_stage_forward_tp(g2, 1, x, y2, R.TpWorkspace(g2, tokens), T)
    torch.cuda.synchronize()
    a, b = y1.double().cpu().numpy(), y2.double().cpu().numpy()
    assert nw(b, a) <= 2 * TOL


@pytest.mark.parametrize("T", [2, 3])
def test_tp_stage_attention_prefill_then_decode(T):
    sq, R = sqm()
    h1, h2, L, H, B, s = 768, 3072, 2, 12, 2, 24
    bits = [4, 8]
    g = R.build_tp_layers(L, h1, h2, bits, T)
    o = _oracle_sets(L, h1, h2, bits, T)
    caches = [R.KVCache(L, B, s + 3, h1 // T) for _ in range(T)]
    ocaches = [O.KVCache(L, B, s + 3, h1 // T) for _ in range(T)]
    ws = R.TpWorkspace(g, B * s)
    x = synth.hidden_f32(17, B * s, h1)
    xo = torch.empty((B * s, h1), dtype=torch.float32, device="cuda")
    R.sq_stage_forward_tp(g, 0, torch.from_numpy(x).cuda(), xo, ws, T, caches=caches, n_heads=H, seq0=0, nseq=B,
                          seq_len=s, pos0=0)
    torch.cuda.synchronize()
    ref = O.stage_tp(o, x.astype(np.float64), H, B, s, 0, 0, ocaches)
    assert nw(xo.cpu().numpy(), ref) <= TOL
    for t in range(3):
        e = synth.hidden_f32(30 + t, B, h1)
        xd = torch.empty((B, h1), dtype=torch.float32, device="cuda")
        R.sq_stage_forward_tp(g, 1, torch.from_numpy(e).cuda(), xd, ws, T, caches=caches, n_heads=H, seq0=0,
                              nseq=B, seq_len=1, pos0=s + t)
        torch.cuda.synchronize()
        refd = O.stage_tp(o, e.astype(np.float64), H, B, 1, s + t, 0, ocaches)
        assert nw(xd.cpu().numpy(), refd) <= TOL, (t, nw(xd.cpu().numpy(), refd))


def test_tp_single_group_row_shard():
    # h1 / T = 128: the row-parallel o shard is one quantization group wide (K2 / K2c / K3 k = 128)
    sq, R = sqm()
    h1, h2, L, T = 512, 1024, 2, 4
    bits = [3, 4]
    g = R.build_tp_layers(L, h1, h2, bits, T)
    o = _oracle_sets(L, h1, h2, bits, T)
    for phase, tokens in ((0, 33), (1, 5)):
        x = synth.hidden_f32(50 + tokens, tokens, h1)
        ws = R.TpWorkspace(g, tokens)
        xo = torch.empty((tokens, h1), dtype=torch.float32, device="cuda")
        R.sq_stage_forward_tp(g, phase, torch.from_numpy(x).cuda(), xo, ws, T)
        torch.cuda.synchronize()
        assert nw(xo.cpu().numpy(), O.stage_tp(o, x.astype(np.float64))) <= TOL


def test_tp8_opt66b_layer_decode_sampled():
    # one OPT-66B layer (h1 9216, h2 36864) split TP8, decode micro-batch of 32, INT4;
    # oracle on 3 sampled token rows (rows are independent under the attention stub)
    sq, R = sqm()
    h1, h2, T, m = 9216, 36864, 8, 32
    g = R.build_tp_layers(1, h1, h2, [4], T)
    o = _oracle_sets(1, h1, h2, [4], T)
    x = synth.hidden_f32(60, m, h1)
    ws = R.TpWorkspace(g, m)
    xo = torch.empty((m, h1), dtype=torch.float32, device="cuda")
    R.sq_stage_forward_tp(g, 1, torch.from_numpy(x).cuda(), xo, ws, T)
    torch.cuda.synchronize()
    rows = [0, 17, 31]
    ref = O.stage_tp(o, x[rows].astype(np.float64))
    assert nw(xo.cpu().numpy()[rows], ref) <= TOL


def test_tp_argument_errors():
    sq, R = sqm()
    h1, h2, T = 768, 3072, 2
    g = R.build_tp_layers(1, h1, h2, [4], T)
    ws = R.TpWorkspace(g, 4)
    x = torch.zeros((4, h1), dtype=torch.float32, device="cuda")
    with pytest.raises(sq.SQError):   # shard sets passed for T = 3 (widths do not add up)
        R.sq_stage_forward_tp(g + [g[0]], 1, x, x, ws, 3)
    with pytest.raises(sq.SQError):   # a real TP rank without an NCCL communicator
        R.sq_stage_forward_tp([g[1]], 1, x, x, ws, T, tp_rank=1)
    with pytest.raises(sq.SQError):   # decode with 33 tokens
        x33 = torch.zeros((33, h1), dtype=torch.float32, device="cuda")
        R.sq_stage_forward_tp(g, 1, x33, x33, R.TpWorkspace(g, 33), T)
    # the smallest valid split (h1 / T = 128, h2 / T = 256) runs
    g3 = R.build_tp_layers(1, 384, 768, [4], 3)
    R.sq_stage_forward_tp(g3, 1, torch.zeros((2, 384), device="cuda"), torch.empty((2, 384), device="cuda"),
                          R.TpWorkspace(g3, 2), 3)
    torch.cuda.synchronize()


def _oracle_full(L, h1, h2, bits):
    full = []
    for l in range(L):
        q = {}
        for name, (n, k) in {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}.items():
            seed = synth.weight_seed(l, name)
            q[name] = O.QWeight(synth.weight_f16(seed, n, k), int(bits[l]), bias=synth.bias_f16(seed, n))
        full.append(O.Layer(int(bits[l]), 0, q["qkv"], q["o"], q["fc1"], q["fc2"]))
    return full


@pytest.mark.parametrize("P,tp,heads,kappa", [(2, 2, 0, 1), (1, 3, 0, 1), (2, 2, 12, 2), (3, 3, 12, 1)])
def test_pipeline_mesh_virtual(P, tp, heads, kappa):
    # a P x tp mesh (TP inside every pipeline stage, P:236 / P:318) run whole on one device (rank -1),
    # configs[0] shapes, against the UNSHARDED oracle pipeline (O7, or O7 with attention)
    sq, R = sqm()
    from paper_conf_cluster_zhaowplw25_b200 import plan as PL
    h1, h2, L = 768, 3072, 6
    B, eta, xi, s, n_dec = 3, 2, 2, 16, 4
    bits = [4, 3, 16, 8, 4, 3]
    sol = PL.partition_layers([1.0] * L, P)
    plan = R.Plan(bits, sol, h1, h2, B, eta, xi, s, n_dec, n_heads=heads, kappa=kappa, tp=tp)
    R.sq_plan_check(plan)
    sets = R.build_tp_layers(L, h1, h2, bits, tp)
    comm = R.Comm.local(P)
    ws = R.PipelineWorkspace(plan, sets, -1)
    x0 = synth.hidden_f32(1, B * s, h1).reshape(B, s, h1)
    out = torch.zeros((B, 1 + n_dec, h1), dtype=torch.float32, device="cuda")
    st = R.sq_pipeline_run(plan, -1, sets, comm, torch.from_numpy(x0).cuda(), out, ws)
    comm.destroy()
    full = _oracle_full(L, h1, h2, bits)
    ref = O.pipeline_attn(full, x0.astype(np.float64), n_dec, heads) if heads else \
        O.pipeline(full, x0.astype(np.float64), n_dec)
    got = out.cpu().numpy()
    for t in range(1 + n_dec):
        assert nw(got[:, t], ref[:, t]) <= TOL, (t, nw(got[:, t], ref[:, t]))
    if heads == 0:
        assert st["graph_replays"] > 0   # the virtual TP decode step replays from the graph cache
