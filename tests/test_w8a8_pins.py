"""Pins for the oracle's W8A8 linear (O9: the weight-activation INT8 scheme of P:93;
DESIGN.md R26): per-output-channel symmetric INT8 weights, per-token symmetric INT8 activations,
exact integer accumulation, y = acc * s_x * s_w.

Pins: brute-force nearest codes with exact rationals (ties to even), the closed-form scales (the amax
element maps to +-127), the half-step bound, exact recovery of grid-aligned inputs, the integer
accumulator against a plain int64 matrix product, and the a-priori error bound of the scheme against
the unquantized product.
"""
from __future__ import annotations

from fractions import Fraction

import numpy as np
import pytest

from oracle import oracle as O
import synth


def _nearest(v: Fraction, s: Fraction) -> int:
    best, bd = None, None
    for c in range(-127, 128):
        d = abs(v - s * c)
        if bd is None or d < bd or (d == bd and c % 2 == 0):
            best, bd = c, d
    return best


def test_weight_codes_bruteforce_and_scale():
    w = synth.weight_f16(3, 4, 96)
    q, s = O.quantize_w8_channel(w)
    amax = np.abs(w.astype(np.float64)).max(1)
    assert (np.abs(s.astype(np.float64) - amax / 127) <= amax / 127 * 2.0 ** -11 * 1.0001).all()
    for r in range(4):
        S = Fraction(float(s[r]))
        for j in range(96):
            b = _nearest(Fraction(float(w[r, j])), S)
            if b != int(q[r, j]):  # only fp32-rounding near-ties may differ
                W = Fraction(float(w[r, j]))
                assert abs(abs(W - S * int(q[r, j])) - abs(W - S * b)) <= S * Fraction(1, 1 << 20)
        assert abs(int(q[r, np.argmax(np.abs(w[r].astype(np.float64)))])) >= 126


def test_activation_codes_hand_example():
    # one token: max |x| = 2.54 -> s = 0.02 (fp32); 1.27 -> 63.5 -> tie -> 64 (even); -2.54 -> -127; 0.01 -> 0.5 -> 0
    x = np.array([[2.54, 1.27, -2.54, 0.01]], np.float16)
    q, s = O.quantize_act8(x)
    sf = np.float32(np.float32(np.float16(2.54)) / np.float32(127))
    assert s[0] == sf
    ref = [int(np.rint(np.float32(np.float16(v)) / sf)) for v in (2.54, 1.27, -2.54, 0.01)]
    assert list(q[0]) == ref and q[0, 0] == 127 and q[0, 2] == -127


@pytest.mark.parametrize("seed", [1, 2])
def test_half_step_bounds_and_zero_rows(seed):
    w = synth.weight_f16(seed, 16, 256)
    w[5] = np.float16(0.0)
    x = synth.act_f16(seed + 10, 9, 256)
    x[3] = np.float16(0.0)
    qw, sw = O.quantize_w8_channel(w)
    qx, sx = O.quantize_act8(x)
    assert (qw[5] == 0).all() and sw[5] == 0 and (qx[3] == 0).all() and sx[3] == 0
    ew = np.abs(qw.astype(np.float64) * sw.astype(np.float64)[:, None] - w.astype(np.float64))
    ex = np.abs(qx.astype(np.float64) * sx.astype(np.float64)[:, None] - x.astype(np.float64))
    # (fp32 division before rint: a tie may land 127 * 2^-24 relative past the exact half step)
    assert (ew <= sw.astype(np.float64)[:, None] / 2 * (1 + 1e-4) + 1e-300).all()
    assert (ex <= sx.astype(np.float64)[:, None] / 2 * (1 + 1e-4) + 1e-300).all()


def test_integer_accumulator_and_scaled_output():
    rng = np.random.default_rng(4)
    xq = rng.integers(-127, 128, size=(7, 320)).astype(np.int8)
    wq = rng.integers(-127, 128, size=(24, 320)).astype(np.int8)
    sx = rng.uniform(0.01, 0.1, 7).astype(np.float32)
    sw = rng.uniform(0.01, 0.1, 24).astype(np.float16)
    b = rng.standard_normal(24).astype(np.float16)
    y, acc = O.linear_w8a8(xq, sx, wq, sw, b)
    ref = xq.astype(np.int64) @ wq.astype(np.int64).T
    assert np.array_equal(acc, ref)
    np.testing.assert_allclose(y, ref * sx.astype(np.float64)[:, None] * sw.astype(np.float64)[None, :]
                               + b.astype(np.float64), rtol=1e-15, atol=1e-12)


def test_grid_aligned_is_exact_and_error_bound():
    # x = s_x * integers, W = s_w * integers (amax = 127 steps) -> the scheme is exact
    rng = np.random.default_rng(5)
    iw = rng.integers(-127, 128, size=(8, 128))
    iw[:, 0] = 127
    ix = rng.integers(-127, 128, size=(3, 128))
    ix[:, 0] = -127
    w = (iw * 2.0 ** -8).astype(np.float16)
    x = (ix * 2.0 ** -6).astype(np.float16)
    qw, sw = O.quantize_w8_channel(w)
    qx, sx = O.quantize_act8(x)
    assert np.array_equal(qw, iw.astype(np.int8)) and np.array_equal(qx, ix.astype(np.int8))
    y, _ = O.linear_w8a8(qx, sx, qw, sw)
    np.testing.assert_allclose(y, x.astype(np.float64) @ w.astype(np.float64).T, rtol=1e-12, atol=1e-12)
    # general inputs: |y - x W^T| <= sum_k (|x_k| s_w/2 + |w_k| s_x/2 + s_x s_w/4) per output
    w = synth.weight_f16(6, 8, 384)
    x = synth.act_f16(7, 5, 384)
    qw, sw = O.quantize_w8_channel(w)
    qx, sx = O.quantize_act8(x)
    y, _ = O.linear_w8a8(qx, sx, qw, sw)
    X, W = x.astype(np.float64), w.astype(np.float64)
    SW, SX = sw.astype(np.float64), sx.astype(np.float64)
    bound = (np.abs(X).sum(1)[:, None] * SW[None, :] / 2 + SX[:, None] * np.abs(W).sum(1)[None, :] / 2
             + 384 * SX[:, None] * SW[None, :] / 4)
    assert (np.abs(y - X @ W.T) <= bound * (1 + 1e-9)).all()


# ---------------------------------------------------------------- GPU parity (kind::i8 tensor cores)
def _sq():
    import paper_conf_cluster_zhaowplw25_b200 as sq
    return sq


@pytest.mark.gpu
def test_gpu_w8a8_codes_bit_exact():
    import torch
    sq = _sq()
    w = synth.adversarial_weight_f16(9, 256, 640)
    x = synth.act_f16(10, 37, 640)
    x[5] = np.float16(0.0)
    qw, sw = O.quantize_w8_channel(w)
    qx, sx = O.quantize_act8(x)
    g = sq.W8Linear.from_fp16(torch.from_numpy(w).cuda())
    gx, gs = sq.sq_quantize_act8(torch.from_numpy(x).cuda())
    assert np.array_equal(g.codes.cpu().numpy(), qw) and np.array_equal(g.scales.cpu().numpy().view(np.uint16), sw.view(np.uint16))
    assert np.array_equal(gx.cpu().numpy(), qx) and np.array_equal(gs.cpu().numpy().view(np.uint32), sx.view(np.uint32))


@pytest.mark.gpu
@pytest.mark.parametrize("m", [1, 5, 32, 33, 100, 300])
@pytest.mark.parametrize("n,k", [(256, 640), (1024, 4096), (128, 128)])
def test_gpu_w8a8_accumulator_exact(m, n, k):
    """the int32 accumulator of tcgen05 kind::i8 equals the oracle's integer sum exactly (every tile
    size BT = 32..256, split-k for narrow grids, ragged token tiles)"""
    import torch
    sq = _sq()
    rng = np.random.default_rng(m * 7 + n)
    qx = rng.integers(-127, 128, size=(m, k)).astype(np.int8)
    qw = rng.integers(-127, 128, size=(n, k)).astype(np.int8)
    sx = np.ones(m, np.float32)
    sw = np.ones(n, np.float16)
    _, acc = O.linear_w8a8(qx, sx, qw, sw)
    g = sq.W8Linear(torch.from_numpy(qw).cuda(), torch.from_numpy(sw).cuda())
    y = torch.empty((m, n), dtype=torch.int32, device="cuda")
    sq.sq_linear_w8a8(g, torch.from_numpy(qx).cuda(), torch.from_numpy(sx).cuda(), y, sq.SQ_W8A8_I32)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy().astype(np.int64), acc)


@pytest.mark.gpu
@pytest.mark.parametrize("mode", [0, 1, 2, 3])
@pytest.mark.parametrize("m", [3, 32, 300])
def test_gpu_w8a8_linear_epilogues(mode, m):
    import torch
    sq = _sq()
    n, k = 384, 1280
    w = synth.weight_f16(20, n, k)
    b = synth.bias_f16(21, n)
    x = synth.act_f16(22 + m, m, k)
    qw, sw = O.quantize_w8_channel(w)
    qx, sx = O.quantize_act8(x)
    ref, _ = O.linear_w8a8(qx, sx, qw, sw, b)
    if mode == 1:
        ref = np.maximum(ref, 0)
    elif mode == 2:
        ref = 0.5 * ref * (1 + np.tanh(np.sqrt(2 / np.pi) * (ref + 0.044715 * ref ** 3)))
    g = sq.W8Linear.from_fp16(torch.from_numpy(w).cuda(), torch.from_numpy(b).cuda())
    gx, gs = sq.sq_quantize_act8(torch.from_numpy(x).cuda())
    if mode == 3:
        y0 = synth.hidden_f32(23, m, n)
        y = torch.from_numpy(y0.copy()).cuda()
        sq.sq_linear_w8a8(g, gx, gs, y, mode)
        got = y.cpu().numpy().astype(np.float64) - y0
    else:
        y = torch.empty((m, n), dtype=torch.float16, device="cuda")
        sq.sq_linear_w8a8(g, gx, gs, y, mode)
        got = y.float().cpu().numpy()
    torch.cuda.synchronize()
    assert np.abs(got - ref).max() / np.abs(ref).max() <= 2e-3
