"""Pins for the tensor-parallel stage (P:63 intra-node TP, P:236 2-D meshes,
P:318 TP4 / TP2+PP2; R27) and a gloo world-size-2 run of the in-place all-reduce scheme the
C-ABI uses (sq.h sq_stage_forward_tp).

Pins (none of them re-types stage_tp's loop):
  * shard codes / scales / zeros equal the matching slices of the unsharded weight's (bit-exact: the
    groups run along k and h1/T, h2/T are multiples of 128);
  * O10 (shard by shard, partial products summed) equals O6 on the unsharded layers to fp64 rounding,
    for T = 1, 2, 3, mixed bit-widths, ReLU and GeLU, with and without attention;
  * with attention, the T per-rank KV caches side by side are the unsharded cache (bit-identical in
    the first layer);
  * a bias added on every rank (the classic row-parallel mistake) is caught.
"""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

from oracle import oracle as O
import synth

DIMS = lambda h1, h2: {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}


def _fp16_model(L, h1, h2):
    out = []
    for l in range(L):
        d = {}
        for name, (n, k) in DIMS(h1, h2).items():
            seed = synth.weight_seed(l, name)
            d[name] = (synth.weight_f16(seed, n, k), synth.bias_f16(seed, n))
        out.append(d)
    return out


def _full_layers(model, bits, act):
    return [O.Layer(bits[l], act, *[O.QWeight(model[l][nm][0], bits[l], bias=model[l][nm][1])
                                    for nm in ("qkv", "o", "fc1", "fc2")]) for l in range(len(model))]


def _shard_layers(model, bits, act, T, ranks=None, bias_everywhere=False):
    ranks = range(T) if ranks is None else ranks
    sets = []
    for r in ranks:
        layers = []
        for l in range(len(model)):
            q = {}
            for nm in ("qkv", "o", "fc1", "fc2"):
                w, b = model[l][nm]
                ws, bs = O.tp_shard(nm, w, b, r, T)
                if bias_everywhere and nm in ("o", "fc2"):
                    bs = b
                q[nm] = O.QWeight(ws, bits[l], bias=bs)
            layers.append(O.Layer(bits[l], act, q["qkv"], q["o"], q["fc1"], q["fc2"]))
        sets.append(layers)
    return sets


def nw(a, b):
    return float(np.abs(a - b).max() / np.abs(b).max())


@pytest.mark.parametrize("bits", [3, 4, 8])
@pytest.mark.parametrize("T", [2, 3])
def test_shard_codes_are_slices_of_full_codes(bits, T):
    h1, h2 = 768, 1536
    model = _fp16_model(1, h1, h2)[0]
    for nm, (w, b) in model.items():
        c, s, z = O.quantize_groups(w, bits)
        for r in range(T):
            ws, _ = O.tp_shard(nm, w, b, r, T)
            cs, ss, zs = O.quantize_groups(ws, bits)
            n, k = w.shape
            if nm == "qkv":
                h, sl = n // 3, n // 3 // T
                rows = np.concatenate([np.arange(j * h + r * sl, j * h + (r + 1) * sl) for j in range(3)])
                ref = (c[rows], s[rows], z[rows])
            elif nm == "fc1":
                sl = n // T
                ref = (c[r * sl:(r + 1) * sl], s[r * sl:(r + 1) * sl], z[r * sl:(r + 1) * sl])
            else:
                sl, g = k // T, k // T // 128
                ref = (c[:, r * sl:(r + 1) * sl], s[:, r * g:(r + 1) * g], z[:, r * g:(r + 1) * g])
            assert np.array_equal(cs, ref[0])
            assert np.array_equal(ss.view(np.uint16), ref[1].view(np.uint16))
            assert np.array_equal(zs.view(np.uint16), ref[2].view(np.uint16))


@pytest.mark.parametrize("T", [1, 2, 3])
@pytest.mark.parametrize("act", [0, 1])
def test_tp_stage_equals_unsharded_stage(T, act):
    h1, h2, L = 768, 1536, 3
    bits = [4, 16, 3]
    model = _fp16_model(L, h1, h2)
    full = _full_layers(model, bits, act)
    sets = _shard_layers(model, bits, act, T)
    x = synth.hidden_f32(5, 7, h1).astype(np.float64)
    ref, _ = O.stage(full, x)
    got = O.stage_tp(sets, x)
    assert nw(got, ref) <= 1e-12


def test_bias_on_every_rank_is_caught():
    h1, h2 = 256, 512
    model = _fp16_model(1, h1, h2)
    full = _full_layers(model, [8], 0)
    x = synth.hidden_f32(6, 4, h1).astype(np.float64)
    ref, _ = O.stage(full, x)
    bad = O.stage_tp(_shard_layers(model, [8], 0, 2, bias_everywhere=True), x)
    assert nw(bad, ref) > 1e-3


@pytest.mark.parametrize("T", [2, 3])
def test_tp_attention_head_parallel_equals_full(T):
    # 12 heads x 64 (head-parallel: 12 / T heads per rank); prefill 2 sequences x 5 tokens, then a decode
    h1, h2, L, H, B = 768, 1536, 2, 12, 2
    bits = [4, 8]
    model = _fp16_model(L, h1, h2)
    full = _full_layers(model, bits, 0)
    sets = _shard_layers(model, bits, 0, T)
    cache = O.KVCache(L, B, 8, h1)
    caches = [O.KVCache(L, B, 8, h1 // T) for _ in range(T)]
    x = synth.hidden_f32(8, B * 5, h1).astype(np.float64)
    ref = O.stage_attn(full, x, B, 5, 0, 0, H, cache)
    got = O.stage_tp(sets, x, H, B, 5, 0, 0, caches)
    assert nw(got, ref) <= 1e-12
    e = synth.hidden_f32(9, B, h1).astype(np.float64)
    ref = O.stage_attn(full, e, B, 1, 5, 0, H, cache)
    got = O.stage_tp(sets, e, H, B, 1, 5, 0, caches)
    assert nw(got, ref) <= 1e-12
    # per-rank caches side by side == the unsharded cache: bit for bit in layer 0 (same input, same dot
    # products in the same order), to fp64 rounding after it (the residual sums differ in order)
    for name in ("k", "v"):
        cat = np.concatenate([getattr(c, name) for c in caches], axis=3)
        assert np.array_equal(cat[0], getattr(cache, name)[0])
        assert nw(cat, getattr(cache, name)) <= 1e-12


# ---------------------------------------------------------------- gloo world 2: the C-ABI's reduce scheme
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _tp_worker(rank, world, port, q):
    """Rank `rank` of a TP group, executing sq_stage_forward_tp's order of operations on the oracle's
    arithmetic: rank 0 accumulates x + p_0 in place, ranks r > 0 hold p_r in a zeroed buffer, one
    in-place all-reduce (sum) per sub-layer returns x + sum_r p_r on every rank."""
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    h1, h2, L = 256, 1024, 2
    bits = [3, 16]
    model = _fp16_model(L, h1, h2)
    mine = _shard_layers(model, bits, 0, world, ranks=[rank])[0]
    x = synth.hidden_f32(11, 5, h1).astype(np.float64)
    for Ly in mine:
        a = O.layernorm(x)
        hs = Ly.o.k
        p = O.linear(O.linear(a, Ly.qkv)[:, 2 * hs:3 * hs], Ly.o)
        buf = torch.from_numpy(x + p if rank == 0 else p)
        dist.all_reduce(buf)
        x = buf.numpy().copy()
        a = O.layernorm(x)
        p = O.linear(np.maximum(O.linear(a, Ly.fc1), 0.0), Ly.fc2)
        buf = torch.from_numpy(x + p if rank == 0 else p)
        dist.all_reduce(buf)
        x = buf.numpy().copy()
    q.put((rank, x))
    dist.barrier()
    dist.destroy_process_group()


def test_gloo_tp_world2_matches_unsharded_stage():
    import multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_tp_worker, args=(r, 2, port, q)) for r in range(2)]
    for p_ in procs:
        p_.start()
    outs = dict(q.get(timeout=600) for _ in range(2))
    for p_ in procs:
        p_.join(timeout=120)
        assert p_.exitcode == 0
    model = _fp16_model(2, 256, 1024)
    ref, _ = O.stage(_full_layers(model, [3, 16], 0), synth.hidden_f32(11, 5, 256).astype(np.float64))
    assert np.array_equal(outs[0], outs[1])       # replicated residual after every all-reduce
    assert nw(outs[0], ref) <= 1e-12
