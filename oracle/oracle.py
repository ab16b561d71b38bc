"""ORACLE — TEST INFRASTRUCTURE ONLY (see oracle/sq_oracle.c header).

Thin numpy/ctypes wrapper over liboracle.so plus the sequential pipeline
simulation O7.  Only tests/, __graft_entry__.smoke()
and bench.py's cpu_baseline / --impl reference legs may import this module.
It never imports the CUDA package, and the CUDA package never imports it.

Functions whose pin is missing are marked "parity unpinned" (none at present;
throughput has no paper number to pin).

f2 (variance indicator, eq. 3): scale_sq_sum / act_moments / variance_indicator, pinned by
closed-form scales (grid-spanning groups), constant groups (omega = 0) and Theorem 1's
bound on the realised rounding error (tests/test_indicator.py).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "sq_oracle.c")
CFLAGS = ["-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-std=gnu11"]


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", _SO, "-lm"])
    return _SO


_L = None
P = ctypes.c_void_p
I64 = ctypes.c_int64


def _lib() -> ctypes.CDLL:
    global _L
    if _L is None:
        L = ctypes.CDLL(build())
        L.oq_quantize_groups.argtypes = [P, I64, I64, ctypes.c_int, ctypes.c_int, P, P, P]
        L.oq_quantize_groups_ex.argtypes = [P, I64, I64, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_uint64,
                                            P, P, P]
        L.oq_splitmix64.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        L.oq_splitmix64.restype = ctypes.c_uint64
        L.oq_uniform24.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        L.oq_uniform24.restype = ctypes.c_float
        L.oq_pack.argtypes = [P, P, P, I64, I64, ctypes.c_int, ctypes.c_int, P, P]
        L.oq_unpack.argtypes = [P, I64, I64, ctypes.c_int, P]
        L.oq_dequant.argtypes = [P, P, I64, I64, ctypes.c_int, ctypes.c_int, P]
        L.oq_linear.argtypes = [P, I64, I64, P, P, I64, ctypes.c_int, ctypes.c_int, P, P]
        L.oq_layernorm.argtypes = [P, I64, I64, ctypes.c_double, P]
        L.oq_layernorm.restype = None
        L.oq_stage.argtypes = [P, ctypes.c_int, P, I64, I64, P]
        L.oq_packed_bytes.argtypes = [I64, I64, ctypes.c_int]
        L.oq_packed_bytes.restype = ctypes.c_size_t
        L.oq_attention.argtypes = [P, I64, I64, I64, I64, I64, ctypes.c_int, P, P, I64, P]
        L.oq_stage_attn.argtypes = [P, ctypes.c_int, P, I64, I64, I64, I64, I64, ctypes.c_int, I64, I64, P, P]
        L.oq_quantize_w8_channel.argtypes = [P, I64, I64, P, P]
        L.oq_quantize_act8.argtypes = [P, I64, I64, P, P]
        L.oq_linear_w8a8.argtypes = [P, P, I64, I64, P, P, I64, P, P, P]
        L.oq_set_threads.argtypes = [ctypes.c_int]
        L.oq_set_threads.restype = None
        L.oq_max_threads.restype = ctypes.c_int
        _L = L
    return _L


def set_threads(n: int) -> int:
    """OpenMP threads of the oracle's parallel loops (timing only); returns the new maximum."""
    _lib().oq_set_threads(int(n))
    return int(_lib().oq_max_threads())


def _p(a: np.ndarray | None):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _check(rc: int, what: str) -> None:
    if rc != 0:
        raise RuntimeError(f"oracle {what} failed rc={rc}")


def quantize_groups(w: np.ndarray, bits: int, group: int = 128):
    """O1.  w fp16 [n, k] -> (codes u8 [n,k], scales fp16 [n,k/g], zeros fp16 [n,k/g])."""
    w = np.ascontiguousarray(w, dtype=np.float16)
    n, k = w.shape
    codes = np.empty((n, k), np.uint8)
    s = np.empty((n, k // group), np.float16)
    z = np.empty((n, k // group), np.float16)
    _check(_lib().oq_quantize_groups(_p(w), n, k, bits, group, _p(codes), _p(s), _p(z)), "quantize")
    return codes, s, z


SYMMETRIC, STOCHASTIC = 1, 2


def quantize_groups_ex(w: np.ndarray, bits: int, group: int = 128, mode: int = 0, seed: int = 0):
    """O1 with the variants (P:184 symmetric S_W, R21; Theorem 1 stochastic rounding, R22).
    mode = SYMMETRIC | STOCHASTIC bits; seed of the counter-based uniform generator."""
    w = np.ascontiguousarray(w, dtype=np.float16)
    n, k = w.shape
    codes = np.empty((n, k), np.uint8)
    s = np.empty((n, k // group), np.float16)
    z = np.empty((n, k // group), np.float16)
    _check(_lib().oq_quantize_groups_ex(_p(w), n, k, bits, group, mode, seed, _p(codes), _p(s), _p(z)), "quantize_ex")
    return codes, s, z


def splitmix64(seed: int, i: int) -> int:
    return int(_lib().oq_splitmix64(seed, i))


def uniform24(seed: int, i: int) -> float:
    return float(_lib().oq_uniform24(seed, i))


def scale_sq_sum(w: np.ndarray, bits: int, group: int = 128, mode: int = 0) -> float:
    """f2, eq. (3) weight term: D_W * S_W(b)^2 with the per-group scale of reading R4
    (R17) = sum over groups of group * s_g(b)^2, s_g(b) the scale O1 stores (asymmetric or,
    mode & SYMMETRIC, P:184's symmetric S_W).  fp64."""
    _, s, _ = quantize_groups_ex(w, bits, group, mode & SYMMETRIC, 0)
    sd = s.astype(np.float64)
    return float(np.sum(group * sd * sd))


def act_moments(x: np.ndarray) -> tuple[float, float]:
    """E[X], Var[X] (population) over all elements, fp64 (G(X) of eq. 3 is Var[X]/4)."""
    xd = np.asarray(x, np.float64).ravel()
    mu = float(np.sum(xd) / xd.size)
    return mu, float(np.sum((xd - mu) ** 2) / xd.size)


def variance_indicator(weights: list[np.ndarray], acts: list[np.ndarray], bits: int, group: int = 128,
                       stochastic: bool = False) -> float:
    """Proposition 1, eq. (3): omega_{i,b} = sum_o D_{W_o} S_{W_o}(b)^2 G(X_o) over the
    linear operators o of a layer; G(X) = Var[X]/4 (deterministic rounding) or (E[X]^2 + Var[X])/6
    (stochastic).  bits == 16 (not quantized, R7) -> 0."""
    if bits == 16:
        return 0.0
    om = 0.0
    for w, x in zip(weights, acts):
        mu, var = act_moments(x)
        g = (mu * mu + var) / 6.0 if stochastic else var / 4.0
        om += scale_sq_sum(w, bits, group) * g
    return om


def pack(codes: np.ndarray, scales: np.ndarray, zeros: np.ndarray, bits: int, group: int = 128):
    """O2 (DESIGN.md layouts L8/L4/L3 + tiling T16).

    -> (packed u8 [n/16, k/128, 16, 128*bits/8] flattened to [n, k*bits/8] bytes,
        meta u32 [n/16, k/128, 16] flattened)."""
    codes = np.ascontiguousarray(codes, np.uint8)
    n, k = codes.shape
    packed = np.empty((n, k * bits // 8), np.uint8)
    meta = np.empty((n // 16, k // 128, 16), np.uint32)
    _check(_lib().oq_pack(_p(codes), _p(np.ascontiguousarray(scales, np.float16)),
                          _p(np.ascontiguousarray(zeros, np.float16)), n, k, bits, group,
                          _p(packed), _p(meta)), "pack")
    return packed, meta


def unpack(packed: np.ndarray, n: int, k: int, bits: int) -> np.ndarray:
    """O3: inverse of the code packing."""
    packed = np.ascontiguousarray(packed, np.uint8)
    codes = np.empty((n, k), np.uint8)
    _check(_lib().oq_unpack(_p(packed), n, k, bits, _p(codes)), "unpack")
    return codes


def packed_bytes(n: int, k: int, bits: int) -> int:
    return int(_lib().oq_packed_bytes(n, k, bits))


class QWeight:
    """Oracle-side quantized linear: packed codes + meta (or fp16 W at bits 16)."""

    def __init__(self, w16: np.ndarray, bits: int, group: int = 128, bias: np.ndarray | None = None,
                 mode: int = 0, seed: int = 0):
        self.n, self.k = w16.shape
        self.bits, self.group = bits, group
        self.bias = None if bias is None else np.ascontiguousarray(bias, np.float16)
        if bits == 16:
            self.packed = np.ascontiguousarray(w16, np.float16).view(np.uint8)
            self.meta = None
            self.codes = self.scales = self.zeros = None
        else:
            self.codes, self.scales, self.zeros = quantize_groups_ex(w16, bits, group, mode, seed)
            self.packed, self.meta = pack(self.codes, self.scales, self.zeros, bits, group)

    def dequant(self) -> np.ndarray:
        """O4: W~ in fp64 [n, k]."""
        out = np.empty((self.n, self.k), np.float64)
        _check(_lib().oq_dequant(_p(self.packed), _p(self.meta), self.n, self.k, self.bits,
                                 self.group, _p(out)), "dequant")
        return out

    def c_struct(self):
        return _OqWeight(self.bits, self.group, self.n, self.k, _p(self.packed), _p(self.meta), _p(self.bias))


def linear(x: np.ndarray, qw: QWeight) -> np.ndarray:
    """O5: y = x W~^T (+bias) in fp64.  x: [m, k] (any float dtype, taken exactly)."""
    x = np.ascontiguousarray(x, np.float64)
    m, k = x.shape
    assert k == qw.k
    y = np.empty((m, qw.n), np.float64)
    _check(_lib().oq_linear(_p(x), m, k, _p(qw.packed), _p(qw.meta), qw.n, qw.bits, qw.group,
                            _p(qw.bias), _p(y)), "linear")
    return y


def layernorm(x: np.ndarray, eps: float = 1e-5) -> np.ndarray:
    x = np.ascontiguousarray(x, np.float64)
    out = np.empty_like(x)
    _lib().oq_layernorm(_p(x), x.shape[0], x.shape[1], eps, _p(out))
    return out


class _OqWeight(ctypes.Structure):
    _fields_ = [("bits", ctypes.c_int32), ("group", ctypes.c_int32), ("n", ctypes.c_int64),
                ("k", ctypes.c_int64), ("packed", ctypes.c_void_p), ("meta", ctypes.c_void_p),
                ("bias", ctypes.c_void_p)]


class _OqLayer(ctypes.Structure):
    _fields_ = [("bits", ctypes.c_int32), ("act", ctypes.c_int32), ("qkv", _OqWeight),
                ("o", _OqWeight), ("fc1", _OqWeight), ("fc2", _OqWeight)]


class Layer:
    """Oracle decoder layer (P:160 linear set; R11/R12)."""

    def __init__(self, bits: int, act: int, qkv: QWeight, o: QWeight, fc1: QWeight, fc2: QWeight):
        self.bits, self.act = bits, act
        self.qkv, self.o, self.fc1, self.fc2 = qkv, o, fc1, fc2

    def c_struct(self):
        return _OqLayer(self.bits, self.act, self.qkv.c_struct(), self.o.c_struct(),
                        self.fc1.c_struct(), self.fc2.c_struct())


def stage(layers: list[Layer], x: np.ndarray, want_qkv: bool = False):
    """O6: run consecutive layers on x fp64 [t, h1]; returns (x_out, qkv of last layer | None)."""
    x = np.array(x, dtype=np.float64, order="C", copy=True)
    t, h1 = x.shape
    arr = (_OqLayer * len(layers))(*[L.c_struct() for L in layers])
    qkv = np.empty((t, 3 * h1), np.float64) if want_qkv else None
    _check(_lib().oq_stage(arr, len(layers), _p(x), t, h1, _p(qkv)), "stage")
    return x, qkv


def pipeline(layers: list[Layer], x0: np.ndarray, n_decode: int) -> np.ndarray:
    """O7: sequential simulation of the pipelined generation (R13/R14).

    x0: fp32/fp64 embeddings [B, s, h1].  Prefill runs every prompt row through all
    layers (rows are independent under the attention stub, so micro-batching and the
    stage partition cannot change the result).  out[b, 0] = hidden at the last prompt
    position; decode input e_1 = LN(out[b, 0]); out[b, t] = F(e_t), e_{t+1} = LN(out[b, t]).
    Returns out [B, 1 + n_decode, h1] in fp64."""
    B, s, h1 = x0.shape
    # prefill only needs the last prompt position of each sequence (rows independent)
    last = np.ascontiguousarray(x0[:, s - 1, :], np.float64)
    out = np.empty((B, 1 + n_decode, h1), np.float64)
    h, _ = stage(layers, last)
    out[:, 0] = h
    for t in range(1, n_decode + 1):
        e = layernorm(out[:, t - 1])
        h, _ = stage(layers, e)
        out[:, t] = h
    return out


# ---------------------------------------------------------------- O8: attention + KV cache (f3)
class KVCache:
    """Oracle-side KV cache of a stage: k, v fp64 [n_layers][B][max_len][h1] (P:162 sizing)."""

    def __init__(self, n_layers: int, B: int, max_len: int, h1: int):
        self.k = np.zeros((n_layers, B, max_len, h1), np.float64)
        self.v = np.zeros_like(self.k)
        self.B, self.max_len, self.h1 = B, max_len, h1


def attention(qkv: np.ndarray, nseq: int, length: int, pos0: int, seq0: int, n_heads: int,
              kc: np.ndarray, vc: np.ndarray) -> np.ndarray:
    """O8 for one layer: qkv fp64 [nseq*length, 3*h1] (rows = (sequence, position)); kc/vc one layer's
    cache [B][max_len][h1], updated in place.  Returns the attention output [nseq*length, h1]."""
    qkv = np.ascontiguousarray(qkv, np.float64)
    h1 = qkv.shape[1] // 3
    assert kc.flags.c_contiguous and vc.flags.c_contiguous and kc.dtype == np.float64
    out = np.empty((nseq * length, h1), np.float64)
    _check(_lib().oq_attention(_p(qkv), nseq, length, pos0, seq0, h1, n_heads, _p(kc), _p(vc), kc.shape[1], _p(out)),
           "attention")
    return out


def stage_attn(layers: list[Layer], x: np.ndarray, nseq: int, length: int, pos0: int, seq0: int, n_heads: int,
               cache: KVCache) -> np.ndarray:
    """O6 with O8: run the stage's layers on x [nseq*length, h1] (rows = (sequence, position))."""
    x = np.array(x, dtype=np.float64, order="C", copy=True)
    h1 = x.shape[1]
    arr = (_OqLayer * len(layers))(*[L.c_struct() for L in layers])
    _check(_lib().oq_stage_attn(arr, len(layers), _p(x), nseq, length, pos0, seq0, h1, n_heads, cache.B,
                                cache.max_len, _p(cache.k), _p(cache.v)), "stage_attn")
    return x


def pipeline_attn(layers: list[Layer], x0: np.ndarray, n_decode: int, n_heads: int) -> np.ndarray:
    """O7 with attention: every sequence's whole prompt through all layers (positions 0..s-1 fill the
    cache), out[b, 0] = hidden at the last prompt position, then n_decode steps at positions s + t - 1
    with e_1 = LN(out[b, 0]), e_{t+1} = LN(out[b, t]) (R14).  Sequences are independent, so micro-batch
    sizes, chunking and the stage partition cannot change the exact result.  -> [B, 1 + n_decode, h1]."""
    B, s, h1 = x0.shape
    cache = KVCache(len(layers), B, s + n_decode, h1)
    out = np.empty((B, 1 + n_decode, h1), np.float64)
    h = stage_attn(layers, np.asarray(x0, np.float64).reshape(B * s, h1), B, s, 0, 0, n_heads, cache)
    out[:, 0] = h.reshape(B, s, h1)[:, -1]
    for t in range(1, n_decode + 1):
        e = layernorm(out[:, t - 1])
        out[:, t] = stage_attn(layers, e, B, 1, s + t - 1, 0, n_heads, cache)
    return out


# ---------------------------------------------------------------- O9: W8A8 (f4)
def quantize_w8_channel(w: np.ndarray):
    """R26: symmetric per-output-channel INT8 weights -> (codes int8 [n,k], scales fp16 [n])."""
    w = np.ascontiguousarray(w, np.float16)
    n, k = w.shape
    q = np.empty((n, k), np.int8)
    s = np.empty(n, np.float16)
    _check(_lib().oq_quantize_w8_channel(_p(w), n, k, _p(q), _p(s)), "quantize_w8")
    return q, s


def quantize_act8(x: np.ndarray):
    """R26: symmetric per-token INT8 activations -> (codes int8 [m,k], scales fp32 [m])."""
    x = np.ascontiguousarray(x, np.float16)
    m, k = x.shape
    q = np.empty((m, k), np.int8)
    s = np.empty(m, np.float32)
    _check(_lib().oq_quantize_act8(_p(x), m, k, _p(q), _p(s)), "quantize_act8")
    return q, s


def linear_w8a8(xq, sx, wq, sw, bias=None):
    """O9: exact integer accumulation, y = acc * s_x * s_w (+ bias) in fp64 -> (y [m,n] fp64, acc int64)."""
    xq = np.ascontiguousarray(xq, np.int8)
    wq = np.ascontiguousarray(wq, np.int8)
    m, k = xq.shape
    n = wq.shape[0]
    acc = np.empty((m, n), np.int64)
    y = np.empty((m, n), np.float64)
    b = None if bias is None else np.ascontiguousarray(bias, np.float16)
    _check(_lib().oq_linear_w8a8(_p(xq), _p(np.ascontiguousarray(sx, np.float32)), m, k, _p(wq),
                                 _p(np.ascontiguousarray(sw, np.float16)), n, _p(b), _p(acc), _p(y)), "linear_w8a8")
    return y, acc


# ---------------------------------------------------------------- O10: tensor-parallel stage (f4)
def tp_shard(name: str, w16: np.ndarray, bias: np.ndarray | None, r: int, T: int):
    """R27 (P:63 intra-node TP, Megatron split): shard r of T of one fp16 linear -> (w16, bias).
    qkv: rows [r h/T, (r+1) h/T) of each of the q, k, v blocks (h = n / 3); fc1: output rows
    [r n/T, (r+1) n/T); o, fc2: input columns [r k/T, (r+1) k/T), bias kept by rank 0 only."""
    n, k = w16.shape
    if name == "qkv":
        h = n // 3
        s = h // T
        rows = [np.arange(j * h + r * s, j * h + (r + 1) * s) for j in range(3)]
        idx = np.concatenate(rows)
        return np.ascontiguousarray(w16[idx]), None if bias is None else np.ascontiguousarray(bias[idx])
    if name == "fc1":
        s = n // T
        return np.ascontiguousarray(w16[r * s:(r + 1) * s]), None if bias is None else bias[r * s:(r + 1) * s].copy()
    s = k // T
    return np.ascontiguousarray(w16[:, r * s:(r + 1) * s]), (None if bias is None or r != 0 else bias.copy())


def _act(u: np.ndarray, act: int) -> np.ndarray:
    if act == 0:
        return np.maximum(u, 0.0)
    return 0.5 * u * (1.0 + np.tanh(0.7978845608028654 * (u + 0.044715 * u * u * u)))


def stage_tp(shards: list[list[Layer]], x: np.ndarray, n_heads: int = 0, nseq: int = 0, length: int = 0,
             pos0: int = 0, seq0: int = 0, caches: list[KVCache] | None = None) -> np.ndarray:
    """O10: one stage (the O6 layer, R11/R12) computed shard by shard under T-way TP, fp64.
    shards[r][l] = rank r's layer l (tp_shard of every linear).  Per layer: a = LN(x); every rank
    computes its q/k/v columns (and, with caches, attention over its n_heads / T heads and its cache of
    width h1 / T), then its partial o-projection p_r = v_r W_o,r^T (+ bias on rank 0); x <- x + sum_r p_r;
    a = LN(x); u_r = act(a W_1,r^T + b_1,r); x <- x + sum_r u_r W_2,r^T (+ bias on rank 0).
    In exact arithmetic this equals O6 on the unsharded layer (the sum over r of the column blocks is the
    full product), which is what pins it (tests/test_tp_pins.py)."""
    T = len(shards)
    x = np.array(x, dtype=np.float64, order="C", copy=True)
    for l in range(len(shards[0])):
        a = layernorm(x)
        p = np.zeros_like(x)
        for r in range(T):
            L = shards[r][l]
            qkv = linear(a, L.qkv)
            hs = L.o.k
            if caches is not None:
                v = attention(qkv, nseq, length, pos0, seq0, n_heads // T, caches[r].k[l], caches[r].v[l])
            else:
                v = qkv[:, 2 * hs:3 * hs]
            p += linear(v, L.o)
        x = x + p
        a = layernorm(x)
        p = np.zeros_like(x)
        for r in range(T):
            L = shards[r][l]
            p += linear(_act(linear(a, L.fc1), L.act), L.fc2)
        x = x + p
    return x
