"""f2 — variance indicator (Proposition 1, eq. 3; Theorem 1).

CPU: the oracle's D_W S_W(b)^2 term is pinned by closed-form scales (groups that span exactly
(2^b - 1) * 2^e), constant groups (R6: s = 0), and Theorem 1's bound |w - w~| <= s/2 on the
realised rounding error; the moments by a hand example.  GPU: sq_scale_sq_sums / sq_act_moments
against the oracle, and the layer-level indicator's bit-width ratios against the closed form
s(3)/s(4) = 15/7.
"""
from __future__ import annotations

import numpy as np
import pytest

import synth
from oracle import oracle as O


def test_scale_sq_closed_form_int4():
    # every group of 128 spans 0 .. 15 * 2^-6 -> s(4) = 2^-6 exactly
    n, k = 32, 512
    w = np.tile((np.arange(128) % 16).astype(np.float16) * np.float16(2.0 ** -6), (n, k // 128))
    assert O.scale_sq_sum(w, 4) == pytest.approx(128 * (2.0 ** -6) ** 2 * n * (k // 128), rel=0, abs=0)


def test_scale_sq_closed_form_int8_group64():
    # groups of 64 spanning 0 .. 255 * 2^-10 (fp16 exact) -> s(8) = 2^-10
    n, k = 16, 256
    row = np.linspace(0, 255, 64).round().astype(np.float16) * np.float16(2.0 ** -10)
    w = np.tile(row, (n, k // 64))
    assert w.max() == np.float16(255 * 2.0 ** -10) and w.min() == 0
    assert O.scale_sq_sum(w, 8, group=64) == 64 * (2.0 ** -10) ** 2 * n * (k // 64)


def test_constant_groups_have_zero_term():
    w = np.full((8, 256), np.float16(0.375))
    for b in (3, 4, 8):
        assert O.scale_sq_sum(w, b) == 0.0
    x = np.full((4, 256), np.float16(2.0))
    assert O.variance_indicator([w], [x], 4) == 0.0
    assert O.variance_indicator([synth.weight_f16(1, 64, 256)], [x], 16) == 0.0  # fp16: not quantized (R7)


def test_act_moments_hand_example():
    mu, var = O.act_moments(np.array([[1, 2], [3, 4]], np.float16))
    assert mu == 2.5 and var == 1.25
    # stochastic G = (E^2 + Var) / 6
    w = np.tile((np.arange(128) % 16).astype(np.float16) * np.float16(2.0 ** -6), (1, 1))
    om = O.variance_indicator([w], [np.array([1, 2, 3, 4], np.float16)], 4, stochastic=True)
    assert om == pytest.approx(128 * 2.0 ** -12 * (2.5 ** 2 + 1.25) / 6.0, rel=1e-15)


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_theorem1_bound_on_realised_error(bits):
    # |w - w~| <= s/2 per weight  =>  sum (w - w~)^2 <= sum_g group s_g^2 / 4 (= omega / Var[X]);
    # for RTN the realised energy is ~ 1/3 of the bound (uniform rounding error: s^2/12)
    w = synth.weight_f16(40 + bits, 64, 1024)
    qw = O.QWeight(w, bits)
    e = qw.dequant() - w.astype(np.float64)
    bound = O.scale_sq_sum(w, bits) / 4.0
    energy = float(np.sum(e * e))
    assert energy <= bound
    assert 0.2 * bound <= energy <= 0.5 * bound


@pytest.mark.gpu
@pytest.mark.parametrize("group", [128, 64, 32])
def test_scale_sq_sums_gpu_parity(group):
    import torch
    import paper_conf_cluster_zhaowplw25_b200 as sq
    for (n, k, seed) in ((48, 640, 1), (1024, 4096, 2), (5, 128, 3)):
        w = synth.weight_f16(seed, n, k)
        got = sq.sq_scale_sq_sums(torch.from_numpy(w).cuda(), (3, 4, 8), group)
        for b, g in zip((3, 4, 8), got):
            ref = O.scale_sq_sum(w, b, group)
            assert g == pytest.approx(ref, rel=1e-12), (n, k, b, g, ref)


@pytest.mark.gpu
def test_act_moments_gpu_parity():
    import torch
    import paper_conf_cluster_zhaowplw25_b200 as sq
    for shape, seed in (((37, 384), 5), ((4096, 9216), 6), ((1,), 7)):
        x = synth.act_f16(seed, int(np.prod(shape)), 1).reshape(shape) if len(shape) == 1 else synth.act_f16(seed, *shape)
        mu, var = sq.sq_act_moments(torch.from_numpy(np.ascontiguousarray(x)).cuda())
        rmu, rvar = O.act_moments(x)
        assert mu == pytest.approx(rmu, rel=1e-12, abs=1e-15) and var == pytest.approx(rvar, rel=1e-12, abs=1e-15)


@pytest.mark.gpu
def test_layer_indicator_bit_ratio():
    # omega(3) / omega(4) = sum s(3)^2 / sum s(4)^2 ~ (15/7)^2 (fp16 rounding of s only); fp16 -> 0
    from paper_conf_cluster_zhaowplw25_b200 import indicator
    t = indicator.layer_terms(0, 256, 1024, calib_tokens=64)
    w3, w4, w8 = (indicator.omega(t, b) for b in (3, 4, 8))
    assert w3 > w4 > w8 > 0 and indicator.omega(t, 16) == 0.0
    assert w3 / w4 == pytest.approx((15 / 7) ** 2, rel=2e-3)
    assert w4 / w8 == pytest.approx((255 / 15) ** 2, rel=5e-3)
    # LayerNorm outputs (qkv, fc1 inputs) have Var = 1 up to fp16 rounding -> G = 1/4
    assert t["G"]["qkv"] == pytest.approx(0.25, rel=2e-3) and t["G"]["fc1"] == pytest.approx(0.25, rel=2e-3)
