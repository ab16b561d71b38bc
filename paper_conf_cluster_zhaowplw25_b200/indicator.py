"""f2 — SplitQuant's variance indicator (Proposition 1, eq. 3), a host-side planner
input computed with the library's kernels.

    omega_{i,b} = sum_{o in layer i} D_{W_o} S_{W_o}(b)^2 G(X_o),   G(X) = Var[X] / 4

(deterministic round-to-nearest, Theorem 1).  D_W S_W(b)^2 uses the per-group scale
the quantizer stores (reading R17: sum over groups of group * s_g(b)^2, ``sq_scale_sq_sums``);
G(X_o) comes from calibration activations (``sq_act_moments``).  Calibration data (C4)
and trained weights are out of scope: the calibration tokens are synthetic
and flow through the layer's own linears (K3 prefill kernels) to give the inputs of o and fc2.
"""
from __future__ import annotations

import torch

from . import (QLinear, SQ_EPI_F16, SQ_EPI_F16_GELU, SQ_EPI_F16_RELU, SQ_EPI_F32_ACCUM, sq_act_moments,
               sq_linear_prefill, sq_scale_sq_sums)

LINEARS = ("qkv", "o", "fc1", "fc2")


def _ln16(x: torch.Tensor) -> torch.Tensor:
    from .runtime import sq_layernorm_f32
    y = torch.empty_like(x)
    sq_layernorm_f32(x, y)
    return y.half()


def layer_terms(layer_idx: int, h1: int, h2: int, bits_set=(3, 4, 8), act: int = 0, calib_tokens: int = 256,
                seed: int = 77) -> dict:
    """For one synthetic decoder layer: {"S2": {linear: {b: D_W S_W(b)^2}}, "G": {linear: Var/4}}."""
    import synth
    dims = {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}
    ws = {}
    for name, (n, k) in dims.items():
        w = torch.empty((n, k), dtype=torch.float16, device="cuda")
        synth.device_weight_f16(w.data_ptr(), synth.weight_seed(layer_idx, name), n, k)
        ws[name] = w
    s2 = {name: dict(zip(bits_set, sq_scale_sq_sums(ws[name], tuple(bits_set)))) for name in LINEARS}
    # calibration pass (fp16 weights, the library's prefill kernels): inputs of the four linears
    x = torch.empty((calib_tokens, h1), dtype=torch.float32, device="cuda")
    synth.device_fill_f32(x.data_ptr(), seed, 0, x.numel(), 1.0, False)
    a = _ln16(x)
    qkv = torch.empty((calib_tokens, 3 * h1), dtype=torch.float16, device="cuda")
    sq_linear_prefill(QLinear.from_fp16(ws["qkv"], 16), a, qkv, SQ_EPI_F16)
    v = qkv[:, 2 * h1:].contiguous()
    r = x.clone()  # residual stream: the o-proj epilogue adds its product in fp32 (r += v W_o^T), as in the stage
    sq_linear_prefill(QLinear.from_fp16(ws["o"], 16), v, r, SQ_EPI_F32_ACCUM)
    h2in = _ln16(r)
    u = torch.empty((calib_tokens, h2), dtype=torch.float16, device="cuda")
    sq_linear_prefill(QLinear.from_fp16(ws["fc1"], 16), h2in, u, SQ_EPI_F16_RELU if act == 0 else SQ_EPI_F16_GELU)
    g = {}
    for name, xin in (("qkv", a), ("o", v), ("fc1", h2in), ("fc2", u)):
        _, var = sq_act_moments(xin)
        g[name] = var / 4.0
    return {"S2": s2, "G": g}


def omega(terms: dict, bits: int) -> float:
    """omega_{i,b} from ``layer_terms`` (0 for fp16, R7)."""
    if bits == 16:
        return 0.0
    return sum(terms["S2"][o][bits] * terms["G"][o] for o in LINEARS)
