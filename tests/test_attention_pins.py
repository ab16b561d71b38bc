"""Pins for the oracle's attention + KV cache (O8; R23-R25).

Every pin is a closed form or an invariant, not the oracle's formula retyped: a single visible key
returns its value (the R12 stub is the first position's exact case), equal keys / a zero query give the
running mean of the values, a hand-built score gap of sqrt(dh) ln 3 gives weights 1/4 and 3/4 (pins the
1/sqrt(dh) scale and the softmax), heads use only their own columns, the cache makes a decode step equal
the last row of a longer prefill, and chunked prefill equals one chunk.
"""
from __future__ import annotations

import math

import numpy as np
import pytest

from oracle import oracle as O
import synth


def _qkv(rng, T, h1):
    return rng.standard_normal((T, 3 * h1))


def _cache(B, L, h1):
    return np.zeros((B, L, h1)), np.zeros((B, L, h1))


def test_first_position_returns_its_value_and_cache_is_written():
    rng = np.random.default_rng(1)
    h1, H, s = 64, 4, 5
    qkv = _qkv(rng, 2 * s, h1)
    kc, vc = _cache(3, 8, h1)
    out = O.attention(qkv, 2, s, 0, 1, H, kc, vc)
    for i in range(2):
        np.testing.assert_array_equal(out[i * s], qkv[i * s, 2 * h1:])  # softmax over one key = 1
        np.testing.assert_array_equal(kc[1 + i, :s], qkv[i * s:(i + 1) * s, h1:2 * h1])
        np.testing.assert_array_equal(vc[1 + i, :s], qkv[i * s:(i + 1) * s, 2 * h1:])
    assert not kc[0].any() and not kc[1:, s:].any()


@pytest.mark.parametrize("how", ["zero_query", "equal_keys"])
def test_uniform_weights_give_running_mean(how):
    rng = np.random.default_rng(2)
    h1, H, s = 128, 2, 7
    qkv = _qkv(rng, s, h1)
    if how == "zero_query":
        qkv[:, :h1] = 0.0
    else:
        qkv[:, h1:2 * h1] = qkv[0, h1:2 * h1]
    kc, vc = _cache(1, s, h1)
    out = O.attention(qkv, 1, s, 0, 0, H, kc, vc)
    v = qkv[:, 2 * h1:]
    ref = np.cumsum(v, 0) / np.arange(1, s + 1)[:, None]
    np.testing.assert_allclose(out, ref, rtol=1e-13, atol=1e-13)


@pytest.mark.parametrize("dh", [64, 128])
def test_scale_and_softmax_hand_example(dh):
    # one head; key 0 and key 1 with q.k1 - q.k0 = sqrt(dh) ln 3 -> weights 1/4, 3/4 for the query at p = 1
    h1 = dh
    qkv = np.zeros((2, 3 * h1))
    qkv[1, 0] = 1.0                                   # q of position 1 = e_0
    qkv[0, h1] = 0.5                                  # k0 . q = 0.5
    qkv[1, h1] = 0.5 + math.sqrt(dh) * math.log(3.0)  # k1 . q
    qkv[0, 2 * h1:] = 2.0                             # v0
    qkv[1, 2 * h1:] = -6.0                            # v1
    kc, vc = _cache(1, 2, h1)
    out = O.attention(qkv, 1, 2, 0, 0, 1, kc, vc)
    np.testing.assert_allclose(out[1], 0.25 * 2.0 + 0.75 * -6.0, rtol=1e-13)


def test_heads_use_their_own_columns():
    # head 0 query zero (uniform), head 1 query one-hot on a huge score for key 0
    h1, H, s = 128, 2, 4
    dh = h1 // H
    rng = np.random.default_rng(3)
    qkv = _qkv(rng, s, h1) * 0.01
    qkv[:, :dh] = 0.0
    qkv[:, dh:h1] = 0.0
    qkv[:, dh] = 1.0
    qkv[:, h1 + dh] = 0.0
    qkv[0, h1 + dh] = 1e4                                # key 0 of head 1 dominates
    kc, vc = _cache(1, s, h1)
    out = O.attention(qkv, 1, s, 0, 0, H, kc, vc)
    v = qkv[:, 2 * h1:]
    np.testing.assert_allclose(out[:, dh:], np.broadcast_to(v[0, dh:], (s, dh)), rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(out[:, :dh], np.cumsum(v[:, :dh], 0) / np.arange(1, s + 1)[:, None], rtol=1e-12)


def test_decode_step_equals_last_row_of_longer_prefill_and_chunking_is_invariant():
    rng = np.random.default_rng(4)
    h1, H, s = 128, 4, 9
    qkv = _qkv(rng, s + 1, h1)
    kc, vc = _cache(1, s + 1, h1)
    full = O.attention(qkv, 1, s + 1, 0, 0, H, kc, vc)
    kc2, vc2 = _cache(1, s + 1, h1)
    a = O.attention(qkv[:4], 1, 4, 0, 0, H, kc2, vc2)      # chunk 1
    b = O.attention(qkv[4:s], 1, s - 4, 4, 0, H, kc2, vc2)  # chunk 2 (reads chunk 1 from the cache)
    d = O.attention(qkv[s:], 1, 1, s, 0, H, kc2, vc2)       # decode step at position s
    np.testing.assert_allclose(np.concatenate([a, b, d]), full, rtol=1e-13, atol=1e-13)


def _layers(h1=128, L=2, bits=(4, 16)):
    out = []
    for l in range(L):
        b = bits[l % len(bits)]
        mk = lambda name, n, k: O.QWeight(synth.weight_f16(synth.weight_seed(l, name), n, k), b,
                                          bias=synth.bias_f16(synth.weight_seed(l, name), n))
        out.append(O.Layer(b, 0, mk("qkv", 3 * h1, h1), mk("o", h1, h1), mk("fc1", 4 * h1, h1), mk("fc2", h1, 4 * h1)))
    return out


def test_stage_attn_first_position_equals_stub_stage():
    # at position 0 the attention output is v exactly, i.e. the R12 stub: the first row of every
    # sequence must match O.stage (which implements the stub) bitwise
    layers = _layers()
    x = synth.hidden_f32(5, 2 * 6, 128).astype(np.float64)
    cache = O.KVCache(2, 2, 6, 128)
    y = O.stage_attn(layers, x, 2, 6, 0, 0, 2, cache)
    stub, _ = O.stage(layers, x[[0, 6]])
    np.testing.assert_array_equal(y[[0, 6]], stub)


def test_pipeline_attn_is_per_sequence():
    # sequences are independent: the 2-sequence run equals each sequence run alone
    layers = _layers()
    x0 = synth.hidden_f32(6, 2 * 5, 128).reshape(2, 5, 128).astype(np.float64)
    both = O.pipeline_attn(layers, x0, 3, 2)
    for b in range(2):
        one = O.pipeline_attn(layers, x0[b:b + 1], 3, 2)
        np.testing.assert_allclose(both[b], one[0], rtol=1e-13, atol=1e-13)
