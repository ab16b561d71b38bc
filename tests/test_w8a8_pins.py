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
