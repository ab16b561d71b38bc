"""GPU parity of the attention + KV cache row against the oracle O8.

sq_attention (kv_append + prefill / decode kernels) vs O.attention on the same fp16 q, k, v; the cache
bytes bit-exact; the stage with attention vs O.stage_attn; the pipeline (micro-batched, chunked prefill
kappa, 2 virtual stages) vs O.pipeline_attn on configs[0] shapes; an OPT-66B-shaped decode step on
sampled heads.  Tolerance normwise 2e-3 (R10).
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


def _qkv(seed, T, h1, scale=1.0):
    return (synth.act_f16(seed, T, 3 * h1).astype(np.float32) * np.float32(scale)).astype(np.float16)


@pytest.mark.parametrize("dh", [64, 128])
@pytest.mark.parametrize("B,nseq,seq0", [(3, 2, 1), (1, 1, 0)])
def test_attention_prefill_chunks_then_decode(dh, B, nseq, seq0):
    sq, R = sqm()
    H = 3 if dh == 128 else 4
    h1 = H * dh
    L1, L2, n_dec = 70, 33, 3
    max_len = L1 + L2 + n_dec + 5
    kc = torch.zeros((B, max_len, h1), dtype=torch.float16, device="cuda")
    vc = torch.zeros_like(kc)
    okc, ovc = np.zeros((B, max_len, h1)), np.zeros((B, max_len, h1))
    steps = [(L1, 0), (L2, L1)] + [(1, L1 + L2 + t) for t in range(n_dec)]
    for si, (length, pos0) in enumerate(steps):
        qkv = _qkv(100 + si, nseq * length, h1, 0.5)
        out = torch.empty((nseq * length, h1), dtype=torch.float16, device="cuda")
        sq.sq_attention(torch.from_numpy(qkv).cuda(), nseq, length, pos0, seq0, H, kc, vc, out)
        torch.cuda.synchronize()
        ref = O.attention(qkv.astype(np.float64), nseq, length, pos0, seq0, H, okc, ovc)
        assert nw(out.float().cpu().numpy(), ref) <= TOL, (si, nw(out.float().cpu().numpy(), ref))
    # the cache holds exactly the fp16 k / v rows written so far (bit-exact), zeros elsewhere
    np.testing.assert_array_equal(kc.float().cpu().numpy(), okc.astype(np.float16).astype(np.float32))
    np.testing.assert_array_equal(vc.float().cpu().numpy(), ovc.astype(np.float16).astype(np.float32))


def test_attention_decode_full_size_sampled():
    # OPT-66B attention shape (72 heads x 128), decode micro-batch of 32 sequences at position 600,
    # cache prefilled with synthetic fp16 rows; oracle on 4 sampled sequences (all heads)
    sq, R = sqm()
    H, dh, B, pos = 72, 128, 32, 600
    h1 = H * dh
    max_len = 640
    kc = torch.empty((B, max_len, h1), dtype=torch.float16, device="cuda")
    vc = torch.empty_like(kc)
    synth.device_fill_f16(kc.data_ptr(), 31, 0, kc.numel(), 0.5, False)
    synth.device_fill_f16(vc.data_ptr(), 32, 0, vc.numel(), 1.0, False)
    qkv = _qkv(33, B, h1, 0.5)
    out = torch.empty((B, h1), dtype=torch.float16, device="cuda")
    sq.sq_attention(torch.from_numpy(qkv).cuda(), B, 1, pos, 0, H, kc, vc, out)
    torch.cuda.synchronize()
    o = out.float().cpu().numpy()
    for b in (0, 7, 19, 31):
        okc = kc[b:b + 1, :pos + 1].float().cpu().numpy().astype(np.float64)
        ovc = vc[b:b + 1, :pos + 1].float().cpu().numpy().astype(np.float64)
        okc[0, pos] = qkv[b, h1:2 * h1]
        ovc[0, pos] = qkv[b, 2 * h1:]
        okc = np.ascontiguousarray(okc)
        ovc = np.ascontiguousarray(ovc)
        # positions 0..pos-1 are already in the cache: attend with a 1-token call at pos
        ref = O.attention(qkv[b:b + 1].astype(np.float64), 1, 1, pos, 0, H, okc, ovc)
        assert nw(o[b:b + 1], ref) <= TOL


def _layers(L, h1, h2, bits, act=0):
    sq, R = sqm()
    g = R.build_layers(L, h1, h2, bits, act=act)
    o = []
    for l in range(L):
        q = {}
        for name, (n, k) in {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}.items():
            seed = synth.weight_seed(l, name)
            q[name] = O.QWeight(synth.weight_f16(seed, n, k), int(bits[l]), bias=synth.bias_f16(seed, n))
        o.append(O.Layer(int(bits[l]), act, q["qkv"], q["o"], q["fc1"], q["fc2"]))
    return g, o


@pytest.mark.parametrize("h1,H", [(768, 12), (256, 2)])
def test_stage_attn_prefill_then_decode(h1, H):
    sq, R = sqm()
    L, B, s = 3, 2, 40
    bits = [4, 16, 3]
    g, o = _layers(L, h1, 4 * h1, bits)
    cache = R.KVCache(L, B, s + 2, h1)
    ocache = O.KVCache(L, B, s + 2, h1)
    x = synth.hidden_f32(7, B * s, h1)
    ws = R.StageWorkspace(g, B * s)
    xo = torch.empty((B * s, h1), dtype=torch.float32, device="cuda")
    R.sq_stage_forward_attn(g, 0, torch.from_numpy(x).cuda(), xo, ws, cache, H, 0, B, s, 0)
    torch.cuda.synchronize()
    ref = O.stage_attn(o, x.astype(np.float64), B, s, 0, 0, H, ocache)
    assert nw(xo.cpu().numpy(), ref) <= TOL
    for t in range(2):
        e = synth.hidden_f32(20 + t, B, h1)
        xd = torch.empty((B, h1), dtype=torch.float32, device="cuda")
        R.sq_stage_forward_attn(g, 1, torch.from_numpy(e).cuda(), xd, ws, cache, H, 0, B, 1, s + t)
        torch.cuda.synchronize()
        refd = O.stage_attn(o, e.astype(np.float64), B, 1, s + t, 0, H, ocache)
        assert nw(xd.cpu().numpy(), refd) <= TOL


@pytest.mark.parametrize("kappa,stages", [(1, [0] * 12), (2, [0] * 5 + [1] * 7), (4, [0] * 12)])
def test_pipeline_attn_configs0(kappa, stages):
    # configs[0] shapes (OPT-125m: 12 heads x 64) with real attention: B = 3 sequences, eta = 2, xi = 2,
    # prompt 32 (kappa chunks), 8 decode steps, 1 or 2 virtual stages; end to end vs O.pipeline_attn
    sq, R = sqm()
    h1, h2, L, H = 768, 3072, 12, 12
    B, eta, xi, s, n_dec = 3, 2, 2, 32, 8
    bits = [int(b) for b in synth.bits_plan(2, L)]
    g, o = _layers(L, h1, h2, bits)
    plan = R.Plan(bits, stages, h1, h2, B, eta, xi, s, n_dec, n_heads=H, kappa=kappa)
    R.sq_plan_check(plan)
    comm = R.Comm.local(plan.n_stages)
    ws = R.PipelineWorkspace(plan, g, -1)
    x0 = synth.hidden_f32(1, B * s, h1).reshape(B, s, h1)
    out = torch.zeros((B, 1 + n_dec, h1), dtype=torch.float32, device="cuda")
    R.sq_pipeline_run(plan, -1, g, comm, torch.from_numpy(x0).cuda(), out, ws)
    comm.destroy()
    ref = O.pipeline_attn(o, x0.astype(np.float64), n_dec, H)
    got = out.cpu().numpy()
    for t in range(1 + n_dec):
        assert nw(got[:, t], ref[:, t]) <= TOL, (t, nw(got[:, t], ref[:, t]))
