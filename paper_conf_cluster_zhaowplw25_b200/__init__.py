"""Python binding of libsq (include/sq.h) — argument marshalling only.

Every step of the hot path runs in libsq's CUDA kernels; PyTorch provides
device memory, streams and process groups.  There is no CPU fallback: if
libsq.so is missing or cannot be loaded this module raises ImportError.

Names mirror the C-ABI: ``sq_quantize_groups``, ``sq_pack``,
``sq_linear_decode``, ``sq_linear_prefill``, ``sq_stage_forward``,
``sq_pipeline_run`` (+ helpers).  Tensor arguments are torch CUDA tensors.
"""
from __future__ import annotations

import ctypes
import os

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SQ_LIB_PATH") or os.path.join(_HERE, "libsq.so")  # SQ_LIB_PATH: experiment builds
if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} not built: run `python __graft_entry__.py build` (no CPU fallback exists)")
_L = ctypes.CDLL(LIB_PATH)

SQ_OK, SQ_EINVAL, SQ_ENOTSUP, SQ_ENOMEM, SQ_ECUDA, SQ_ENCCL, SQ_EINTERNAL = range(7)
SQ_EPI_F16, SQ_EPI_F16_RELU, SQ_EPI_F16_GELU, SQ_EPI_F32_ACCUM = range(4)
SQ_PREFILL, SQ_DECODE = 0, 1

P = ctypes.c_void_p
I64 = ctypes.c_int64
I32 = ctypes.c_int32


class SQError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"libsq status {status}: {msg}")
        self.status = status


class sq_qweight(ctypes.Structure):
    _fields_ = [("bits", I32), ("group", I32), ("n", I64), ("k", I64), ("packed", P), ("meta", P), ("bias", P)]


class sq_layer(ctypes.Structure):
    _fields_ = [("bits", I32), ("act", I32), ("qkv", sq_qweight), ("o", sq_qweight), ("fc1", sq_qweight),
                ("fc2", sq_qweight)]


class sq_plan(ctypes.Structure):
    _fields_ = [("n_layers", I32), ("n_stages", I32), ("hidden", I32), ("ffn", I32), ("group", I32),
                ("bits", ctypes.POINTER(I32)), ("stage_of_layer", ctypes.POINTER(I32)), ("B", I32), ("eta", I32),
                ("xi", I32), ("prompt_len", I32), ("n_decode", I32), ("n_heads", I32), ("kappa", I32), ("tp", I32)]


class sq_attn(ctypes.Structure):
    _fields_ = [("n_heads", I32), ("max_len", I32), ("n_seq_cache", I64), ("k_cache", ctypes.POINTER(P)),
                ("v_cache", ctypes.POINTER(P)), ("seq0", I64), ("nseq", I32), ("seq_len", I32), ("pos0", I32)]


class sq_run_stats(ctypes.Structure):
    _fields_ = [("t_total_ms", ctypes.c_double), ("t_prefill_ms", ctypes.c_double), ("t_decode_ms", ctypes.c_double),
                ("tokens_per_s", ctypes.c_double), ("bytes_sent", I64), ("gpu_launches", I64),
                ("host_enqueue_ms", ctypes.c_double), ("graph_replays", I64)]


class sq_sched_op(ctypes.Structure):
    _fields_ = [("kind", I32), ("item", I32), ("phase", I32), ("t", I32), ("slot", I32), ("peer", I32),
                ("seq0", I64), ("nseq", I64), ("rows", I64)]


SQ_OP_NAMES = ["RECV_LB", "RECV_ACT", "COMPUTE", "SEND_ACT", "OUT", "SEND_LB", "LOOPBACK_LOCAL"]


class sq_profile(ctypes.Structure):
    _fields_ = [("launches", I64 * 6), ("ms", ctypes.c_double * 6), ("bytes", ctypes.c_double * 6),
                ("flops", ctypes.c_double * 6)]


def _sig(name, restype, *argtypes):
    fn = getattr(_L, name)
    fn.restype = restype
    fn.argtypes = list(argtypes)
    return fn


_sig("sq_last_error", ctypes.c_char_p)
_sig("sq_version", ctypes.c_char_p)
_sig("sq_abi_version", ctypes.c_int)
_sig("sq_packed_bytes", ctypes.c_size_t, I64, I64, ctypes.c_int)
_sig("sq_meta_bytes", ctypes.c_size_t, I64, I64, ctypes.c_int)
_sig("sq_quantize_groups", ctypes.c_int, P, I64, I64, ctypes.c_int, ctypes.c_int, P, P, P, P)
_sig("sq_quantize_groups_ex", ctypes.c_int, P, I64, I64, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_uint64,
     P, P, P, P, P)
_sig("sq_pack", ctypes.c_int, P, P, P, I64, I64, ctypes.c_int, ctypes.c_int, P, P, P)
_sig("sq_linear_workspace_bytes", ctypes.c_size_t, ctypes.POINTER(sq_qweight), I64)
_sig("sq_linear_decode", ctypes.c_int, ctypes.POINTER(sq_qweight), P, I64, I64, P, I64, ctypes.c_int, P, P,
     ctypes.c_size_t, P)
_sig("sq_xsum", ctypes.c_int, P, I64, I64, I64, P, P)
_sig("sq_linear_prefill", ctypes.c_int, ctypes.POINTER(sq_qweight), P, I64, I64, P, I64, ctypes.c_int, P)
_sig("sq_profile_enable", ctypes.c_int, ctypes.c_int)
_sig("sq_profile_read", ctypes.c_int, ctypes.POINTER(sq_profile))
_sig("sq_launch_count", I64)

EXPORTED = [
    "sq_last_error", "sq_version", "sq_abi_version", "sq_packed_bytes", "sq_meta_bytes", "sq_quantize_groups",
    "sq_pack", "sq_linear_workspace_bytes", "sq_linear_decode", "sq_xsum", "sq_linear_prefill",
    "sq_stage_workspace_bytes", "sq_stage_forward", "sq_layernorm_f32", "sq_comm_unique_id_bytes",
    "sq_comm_get_unique_id", "sq_comm_init", "sq_comm_init_local", "sq_comm_destroy",
    "sq_pipeline_workspace_bytes", "sq_pipeline_run", "sq_plan_check", "sq_profile_enable", "sq_profile_read",
    "sq_launch_count", "sq_pipeline_schedule", "sq_scale_sq_sums_workspace_bytes", "sq_scale_sq_sums",
    "sq_act_moments_workspace_bytes", "sq_act_moments", "sq_quantize_groups_ex", "sq_attention",
    "sq_stage_forward_attn", "sq_quantize_w8", "sq_quantize_act8", "sq_linear_w8a8_workspace_bytes",
    "sq_linear_w8a8", "sq_stage_tp_workspace_bytes", "sq_stage_forward_tp", "sq_comm_init_mesh",
]


def _opt(name, restype, *argtypes):
    if hasattr(_L, name):
        _sig(name, restype, *argtypes)


_opt("sq_stage_workspace_bytes", ctypes.c_size_t, ctypes.POINTER(sq_layer), ctypes.c_int, I64)
_opt("sq_stage_forward", ctypes.c_int, ctypes.POINTER(sq_layer), ctypes.c_int, ctypes.c_int, P, I64, P, P, P,
     ctypes.c_size_t, P)
_opt("sq_layernorm_f32", ctypes.c_int, P, I64, I64, P, P)
_opt("sq_quantize_w8", ctypes.c_int, P, I64, I64, P, P, P)
_opt("sq_quantize_act8", ctypes.c_int, P, I64, I64, I64, P, P, P)
_opt("sq_linear_w8a8_workspace_bytes", ctypes.c_size_t, I64, I64, I64)
_opt("sq_linear_w8a8", ctypes.c_int, P, P, P, I64, I64, P, P, I64, P, I64, ctypes.c_int, P, ctypes.c_size_t, P)
_opt("sq_attention", ctypes.c_int, P, I64, I64, I64, I64, I64, I64, ctypes.c_int, P, P, I64, I64, P, I64, P)
_opt("sq_stage_forward_attn", ctypes.c_int, ctypes.POINTER(sq_layer), ctypes.c_int, ctypes.c_int,
     ctypes.POINTER(sq_attn), P, I64, P, P, ctypes.c_size_t, P)
_opt("sq_stage_tp_workspace_bytes", ctypes.c_size_t, ctypes.POINTER(sq_layer), ctypes.c_int, I64)
_opt("sq_stage_forward_tp", ctypes.c_int, ctypes.POINTER(sq_layer), ctypes.c_int, ctypes.c_int, ctypes.c_int, P,
     ctypes.c_int, ctypes.POINTER(sq_attn), P, I64, P, P, ctypes.c_size_t, P)
_opt("sq_comm_unique_id_bytes", ctypes.c_size_t)
_opt("sq_comm_get_unique_id", ctypes.c_int, P)
_opt("sq_comm_init", ctypes.c_int, ctypes.POINTER(P), P, ctypes.c_int, ctypes.c_int)
_opt("sq_comm_init_local", ctypes.c_int, ctypes.POINTER(P), ctypes.c_int)
_opt("sq_comm_init_mesh", ctypes.c_int, ctypes.POINTER(P), P, ctypes.c_int, ctypes.c_int, ctypes.c_int)
_opt("sq_comm_destroy", ctypes.c_int, P)
_opt("sq_pipeline_workspace_bytes", ctypes.c_size_t, ctypes.POINTER(sq_plan), ctypes.POINTER(sq_layer), ctypes.c_int)
_opt("sq_pipeline_run", ctypes.c_int, ctypes.POINTER(sq_plan), ctypes.c_int, ctypes.POINTER(sq_layer), ctypes.c_int,
     P, P, P, P, ctypes.c_size_t, ctypes.POINTER(sq_run_stats), P)
_opt("sq_plan_check", ctypes.c_int, ctypes.POINTER(sq_plan))
_opt("sq_pipeline_schedule", I64, ctypes.POINTER(sq_plan), ctypes.c_int, ctypes.POINTER(sq_sched_op), I64)
_opt("sq_scale_sq_sums_workspace_bytes", ctypes.c_size_t, I64, I64)
_opt("sq_scale_sq_sums", ctypes.c_int, P, I64, I64, ctypes.c_int, ctypes.POINTER(I32), ctypes.c_int, P, P,
     ctypes.c_size_t, P)
_opt("sq_act_moments_workspace_bytes", ctypes.c_size_t, I64)
_opt("sq_act_moments", ctypes.c_int, P, I64, P, P, ctypes.c_size_t, P)


def _check(st: int) -> None:
    if st != SQ_OK:
        raise SQError(st, _L.sq_last_error().decode(errors="replace"))


def _ptr(t: torch.Tensor | None):
    return None if t is None else ctypes.c_void_p(t.data_ptr())


def _stream(stream=None):
    s = torch.cuda.current_stream() if stream is None else stream
    return ctypes.c_void_p(s.cuda_stream)


def lib() -> ctypes.CDLL:
    return _L


# ---------------------------------------------------------------- a1 / a2
def sq_quantize_groups(w: torch.Tensor, bits: int, group: int = 128, stream=None):
    """a1: fp16 W [n,k] -> (codes u8 [n,k], scales fp16 [n,k/g], zeros fp16 [n,k/g])."""
    assert w.is_cuda and w.dtype == torch.float16 and w.is_contiguous()
    n, k = w.shape
    codes = torch.empty((n, k), dtype=torch.uint8, device=w.device)
    s = torch.empty((n, k // group), dtype=torch.float16, device=w.device)
    z = torch.empty_like(s)
    _check(_L.sq_quantize_groups(_ptr(w), n, k, bits, group, _ptr(codes), _ptr(s), _ptr(z), _stream(stream)))
    return codes, s, z


SQ_QUANT_SYMMETRIC, SQ_QUANT_STOCHASTIC = 1, 2


def sq_quantize_groups_ex(w: torch.Tensor, bits: int, group: int = 128, mode: int = 0, seed: int = 0, stream=None):
    """a1 variants (include/sq.h): mode = SQ_QUANT_SYMMETRIC | SQ_QUANT_STOCHASTIC (Theorem 1).
    Raises if a symmetric group's zero point overflows fp16 (checked after a stream sync)."""
    assert w.is_cuda and w.dtype == torch.float16 and w.is_contiguous()
    n, k = w.shape
    codes = torch.empty((n, k), dtype=torch.uint8, device=w.device)
    s = torch.empty((n, k // group), dtype=torch.float16, device=w.device)
    z = torch.empty_like(s)
    status = torch.zeros(1, dtype=torch.int32, device=w.device) if mode & SQ_QUANT_SYMMETRIC else None
    _check(_L.sq_quantize_groups_ex(_ptr(w), n, k, bits, group, mode, seed, _ptr(codes), _ptr(s), _ptr(z),
                                    _ptr(status), _stream(stream)))
    if status is not None and int(status.item()) != 0:
        raise SQError(1, "sq_quantize_groups_ex: a symmetric zero point overflows fp16 (max|w| too close to 65504)")
    return codes, s, z


def sq_pack(codes: torch.Tensor, scales: torch.Tensor, zeros: torch.Tensor, bits: int, group: int = 128, stream=None):
    """a2: codes -> (packed u8 [n, k*bits/8] bytes in placement T16, meta int32 [n/16, k/128, 16] (u32 bits))."""
    n, k = codes.shape
    packed = torch.empty((n, k * bits // 8), dtype=torch.uint8, device=codes.device)
    meta = torch.empty((n // 16, k // 128, 16), dtype=torch.int32, device=codes.device)
    _check(_L.sq_pack(_ptr(codes), _ptr(scales), _ptr(zeros), n, k, bits, group, _ptr(packed), _ptr(meta),
                      _stream(stream)))
    return packed, meta


class QLinear:
    """Device-resident quantized linear (owning torch tensors + the sq_qweight view)."""

    def __init__(self, bits: int, n: int, k: int, packed: torch.Tensor, meta: torch.Tensor | None,
                 bias: torch.Tensor | None = None, group: int = 128):
        self.bits, self.n, self.k, self.group = bits, n, k, group
        self.packed, self.meta, self.bias = packed, meta, bias
        self.c = sq_qweight(bits, group, n, k, packed.data_ptr(), meta.data_ptr() if meta is not None else None,
                            bias.data_ptr() if bias is not None else None)

    @classmethod
    def from_fp16(cls, w: torch.Tensor, bits: int, bias: torch.Tensor | None = None, group: int = 128, stream=None,
                  mode: int = 0, seed: int = 0):
        n, k = w.shape
        if bits == 16:
            return cls(16, n, k, w.contiguous(), None, bias, group)
        if mode:
            codes, s, z = sq_quantize_groups_ex(w, bits, group, mode, seed, stream)
        else:
            codes, s, z = sq_quantize_groups(w, bits, group, stream)
        packed, meta = sq_pack(codes, s, z, bits, group, stream)
        return cls(bits, n, k, packed, meta, bias, group)

    def nbytes(self) -> int:
        return self.packed.numel() * self.packed.element_size() + (0 if self.meta is None else self.meta.numel() * 4)


def sq_linear_workspace_bytes(w: QLinear, m: int) -> int:
    return int(_L.sq_linear_workspace_bytes(ctypes.byref(w.c), m))


def sq_xsum(x: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    m, k = x.shape
    if out is None:
        out = torch.empty((k // 128, 32, 2), dtype=torch.float32, device=x.device)
    _check(_L.sq_xsum(_ptr(x), x.stride(0), m, k, _ptr(out), _stream(stream)))
    return out


def sq_linear_decode(w: QLinear, x: torch.Tensor, y: torch.Tensor, epi: int = SQ_EPI_F16, xsum=None,
                     ws: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """a4: y = epi(x W~^T), m = x.shape[0] in [1, 32].  ws: zero-initialised uint8 workspace."""
    m = x.shape[0]
    if ws is None:
        ws = torch.zeros(sq_linear_workspace_bytes(w, m), dtype=torch.uint8, device=x.device)
    _check(_L.sq_linear_decode(ctypes.byref(w.c), _ptr(x), x.stride(0), m, _ptr(y), y.stride(0), epi, _ptr(xsum),
                               _ptr(ws), ws.numel(), _stream(stream)))
    return y


def sq_linear_prefill(w: QLinear, x: torch.Tensor, y: torch.Tensor, epi: int = SQ_EPI_F16, stream=None) -> torch.Tensor:
    """a3: y = epi(x W~^T) on tcgen05 tensor cores, any m >= 1."""
    m = x.shape[0]
    _check(_L.sq_linear_prefill(ctypes.byref(w.c), _ptr(x), x.stride(0), m, _ptr(y), y.stride(0), epi,
                                _stream(stream)))
    return y


# ---------------------------------------------------------------- f2: variance indicator inputs
def sq_scale_sq_sums(w: torch.Tensor, bits=(3, 4, 8), group: int = 128, stream=None) -> list[float]:
    """sum_g group * s_g(b)^2 for each b (fp64, on the GPU), W fp16 [n, k] contiguous."""
    assert w.is_cuda and w.dtype == torch.float16 and w.dim() == 2 and w.is_contiguous()
    n, k = w.shape
    bl = (I32 * len(bits))(*bits)
    out = torch.empty(len(bits), dtype=torch.float64, device=w.device)
    nb = _L.sq_scale_sq_sums_workspace_bytes(n, k)
    ws = torch.empty(max(nb, 8), dtype=torch.uint8, device=w.device)
    _check(_L.sq_scale_sq_sums(_ptr(w), n, k, group, bl, len(bits), _ptr(out), _ptr(ws), ws.numel(), _stream(stream)))
    return [float(v) for v in out.cpu()]


def sq_act_moments(x: torch.Tensor, stream=None) -> tuple[float, float]:
    """(E[X], Var[X]) of fp16 activations (all elements), fp64 on the GPU."""
    assert x.is_cuda and x.dtype == torch.float16 and x.is_contiguous()
    out = torch.empty(2, dtype=torch.float64, device=x.device)
    nb = _L.sq_act_moments_workspace_bytes(x.numel())
    ws = torch.empty(max(nb, 8), dtype=torch.uint8, device=x.device)
    _check(_L.sq_act_moments(_ptr(x), x.numel(), _ptr(out), _ptr(ws), ws.numel(), _stream(stream)))
    o = out.cpu()
    return float(o[0]), float(o[1])


def sq_profile_enable(on: bool = True) -> None:
    _check(_L.sq_profile_enable(1 if on else 0))


def sq_profile_read() -> dict:
    p = sq_profile()
    _check(_L.sq_profile_read(ctypes.byref(p)))
    names = ["gemv", "gemm", "glue", "quant", "attn_decode", "attn_prefill"]
    return {names[i]: {"launches": p.launches[i], "ms": p.ms[i], "bytes": p.bytes[i], "flops": p.flops[i]}
            for i in range(6)}


def sq_launch_count() -> int:
    return int(_L.sq_launch_count())


from . import runtime  # noqa: E402,F401  (stage / pipeline wrappers)


# ---------------------------------------------------------------- f3: attention + KV cache
def sq_attention(qkv: torch.Tensor, nseq: int, length: int, pos0: int, seq0: int, n_heads: int,
                 k_cache: torch.Tensor, v_cache: torch.Tensor, out: torch.Tensor, stream=None) -> torch.Tensor:
    """One layer's causal attention over its KV cache (include/sq.h sq_attention).  qkv fp16
    [nseq*length, 3*h1] rows (sequence, position); caches fp16 [n_seq_cache, max_len, h1]; out fp16
    [nseq*length, h1].  Appends the new k, v to the caches."""
    h1 = qkv.shape[1] // 3
    assert k_cache.shape == v_cache.shape and k_cache.shape[2] == h1
    _check(_L.sq_attention(_ptr(qkv), qkv.stride(0), nseq, length, pos0, seq0, h1, n_heads, _ptr(k_cache),
                           _ptr(v_cache), k_cache.shape[1], k_cache.shape[0], _ptr(out), out.stride(0), _stream(stream)))
    return out


# ---------------------------------------------------------------- f4: W8A8
SQ_W8A8_I32 = 4


class W8Linear:
    """W8A8 linear (include/sq.h): int8 codes [n, k] + fp16 per-channel scales (+ fp16 bias)."""

    def __init__(self, codes: torch.Tensor, scales: torch.Tensor, bias: torch.Tensor | None = None):
        self.codes, self.scales, self.bias = codes, scales, bias
        self.n, self.k = codes.shape

    @classmethod
    def from_fp16(cls, w: torch.Tensor, bias: torch.Tensor | None = None, stream=None) -> "W8Linear":
        assert w.is_cuda and w.dtype == torch.float16 and w.is_contiguous()
        n, k = w.shape
        q = torch.empty((n, k), dtype=torch.int8, device=w.device)
        s = torch.empty(n, dtype=torch.float16, device=w.device)
        _check(_L.sq_quantize_w8(_ptr(w), n, k, _ptr(q), _ptr(s), _stream(stream)))
        return cls(q, s, bias)


def sq_quantize_act8(x: torch.Tensor, stream=None):
    m, k = x.shape
    q = torch.empty((m, k), dtype=torch.int8, device=x.device)
    s = torch.empty(m, dtype=torch.float32, device=x.device)
    _check(_L.sq_quantize_act8(_ptr(x), m, k, x.stride(0), _ptr(q), _ptr(s), _stream(stream)))
    return q, s


def sq_linear_w8a8(w: W8Linear, xq: torch.Tensor, sx: torch.Tensor, y: torch.Tensor, mode: int = SQ_EPI_F16,
                   ws: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    m = xq.shape[0]
    need = int(_L.sq_linear_w8a8_workspace_bytes(w.n, w.k, m))
    if need and (ws is None or ws.numel() < need):
        ws = torch.empty(need, dtype=torch.uint8, device=xq.device)
    _check(_L.sq_linear_w8a8(_ptr(w.codes), _ptr(w.scales), _ptr(w.bias), w.n, w.k, _ptr(xq), _ptr(sx), m, _ptr(y),
                             y.stride(0) if mode != SQ_W8A8_I32 else w.n, mode, _ptr(ws) if need else None,
                             need, _stream(stream)))
    return y
