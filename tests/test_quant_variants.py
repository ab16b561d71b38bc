"""Pins for the quantizer variants of the oracle (R21/R22):
P:184's symmetric scale S_W = max(|W_max|, |W_min|) / (2^(b-1) - 1) and Theorem 1's stochastic
rounding, driven by the counter-based splitmix64 stream.

Each pin is something other than the oracle's own formula: published generator vectors, brute force
over exact rationals, sign symmetry, hand-computed codes, the rounding frequencies, unbiasedness and
Theorem 1's stochastic variance D S^2 (E[X]^2 + Var[X]) / 6 (which rounding to nearest does not meet).
"""
from __future__ import annotations

from fractions import Fraction

import numpy as np
import pytest

from oracle import oracle as O
import synth

SYM, STO = O.SYMMETRIC, O.STOCHASTIC


def test_splitmix64_published_vectors():
    # splitmix64 seeded 0 (Vigna's reference splitmix64.c): first three outputs
    assert O.splitmix64(0, 0) == 0xE220A8397B1DCDAF
    assert O.splitmix64(0, 1) == 0x6E789E6AA1B965F4
    assert O.splitmix64(0, 2) == 0x06C45D188009454F


def test_uniform24_is_uniform():
    u = np.array([O.uniform24(7, i) for i in range(64000)])
    assert (u >= 0).all() and (u < 1).all()
    assert (np.round(u * 2 ** 24) == u * 2 ** 24).all()  # 24-bit grid, exact in fp32
    hist, _ = np.histogram(u, bins=16, range=(0, 1))
    chi2 = ((hist - 4000.0) ** 2 / 4000.0).sum()
    assert chi2 < 37.7  # chi-square, 15 dof, p = 0.001


# ---------------------------------------------------------------- symmetric S_W (R21)
def _brute_sym(w, S, bits):
    half = 1 << (bits - 1)
    Sf = Fraction(float(S))
    out = []
    for wj in w:
        W = Fraction(float(wj))
        best, bd = None, None
        for c in range(1, 2 * half):
            d = abs(W - Sf * (c - half))
            if bd is None or d < bd or (d == bd and (c - half) % 2 == 0):
                best, bd = c, d
        out.append(best)
    return np.array(out)


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_symmetric_matches_bruteforce_and_closed_form(bits):
    w = synth.weight_f16(17 + bits, 3, 256)
    codes, s, z = O.quantize_groups_ex(w, bits, 128, SYM)
    half = 1 << (bits - 1)
    g = w.astype(np.float64).reshape(3, 2, 128)
    amax = np.abs(g).max(-1)
    rel = np.abs(s.astype(np.float64) - amax / (half - 1)) / (amax / (half - 1))
    assert rel.max() <= 2.0 ** -11 * 1.0001
    assert np.array_equal(z.astype(np.float64), -half * s.astype(np.float64))
    for r in range(3):
        for gi in range(2):
            sl = slice(128 * gi, 128 * gi + 128)
            bc = _brute_sym(w[r, sl], s[r, gi], bits)
            oc = codes[r, sl].astype(np.int64)
            for j in np.nonzero(bc != oc)[0]:  # only fp32-rounding near-ties may differ
                W, S = Fraction(float(w[r, sl][j])), Fraction(float(s[r, gi]))
                assert abs(abs(W - S * (int(oc[j]) - half)) - abs(W - S * (int(bc[j]) - half))) <= S * Fraction(1, 1 << 20)
    assert codes.min() >= 1 and codes.max() <= 2 ** bits - 1


def test_symmetric_hand_example():
    # INT4: max|w| = 7/16 -> S = 1/16 exactly, q = -8/16 = -0.5; w = 0.125 -> c^ = 2 -> c = 10;
    # w = -7/16 -> c^ = -7 -> c = 1; w = 0.09375 = 1.5 S -> tie -> even c^ = 2 -> c = 10; w = 0 -> c = 8
    w = np.zeros((1, 128), np.float16)
    w[0, :4] = [0.4375, 0.125, -0.4375, 0.09375]
    codes, s, z = O.quantize_groups_ex(w, 4, 128, SYM)
    assert float(s[0, 0]) == 0.0625 and float(z[0, 0]) == -0.5
    assert list(codes[0, :5]) == [15, 10, 1, 10, 8]


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_symmetric_sign_symmetry_and_half_step(bits):
    # round-half-even is odd-symmetric: c(-w) = 2^b - c(w); and |w - w~| <= S/2
    w = synth.weight_f16(23, 16, 512)
    c1, s1, z1 = O.quantize_groups_ex(w, bits, 128, SYM)
    c2, s2, z2 = O.quantize_groups_ex(-w, bits, 128, SYM)
    assert np.array_equal(s1, s2) and np.array_equal(z1, z2)
    assert np.array_equal(c2.astype(np.int64), (1 << bits) - c1.astype(np.int64))
    q = O.QWeight(w, bits, mode=SYM)
    err = np.abs(q.dequant() - w.astype(np.float64))
    assert (err <= q.scales.astype(np.float64).repeat(128, 1) / 2 * (1 + 1e-6)).all()


def test_symmetric_zero_group_and_overflow_rejected():
    w = np.zeros((1, 128), np.float16)
    c, s, z = O.quantize_groups_ex(w, 4, 128, SYM)
    assert (c == 8).all() and s[0, 0] == 0 and z[0, 0].view(np.uint16) == 0
    w[0, 0] = np.float16(60000.0)  # S = fp16(60000/7) = 8568 -> q = -8 * 8568 = -68544 overflows fp16
    with pytest.raises(RuntimeError):
        O.quantize_groups_ex(w, 4, 128, SYM)


# ---------------------------------------------------------------- stochastic rounding (Thm. 1, R22)
@pytest.mark.parametrize("mode", [STO, STO | SYM])
@pytest.mark.parametrize("bits", [3, 4, 8])
def test_stochastic_codes_are_floor_or_ceil(mode, bits):
    w = synth.weight_f16(31, 8, 256)
    codes, s, z = O.quantize_groups_ex(w, bits, 128, mode, seed=5)
    half = (1 << (bits - 1)) if mode & SYM else 0
    for r in range(8):
        for g in range(2):
            S, Z = Fraction(float(s[r, g])), Fraction(float(z[r, g]))
            for j in range(128 * g, 128 * g + 128):
                d = (Fraction(float(w[r, j])) - Z) / S          # exact scaled value
                c = int(codes[r, j])
                lo, hi = int(np.floor(float(d))), int(np.ceil(float(d)))
                assert c in (lo, hi) or abs(d - c) < Fraction(1, 1 << 18), (r, j, float(d), c)
                assert 0 <= c <= (1 << bits) - 1 and (not half or c >= 1)


def test_stochastic_round_up_frequency_equals_fraction():
    # grid s0 = 2^-6 spanning [0, 15 s0]; weights at c + 1/4 and c + 3/4 of a step: P(up) = 1/4 and 3/4
    s0 = 2.0 ** -6
    w = np.zeros((64, 128), np.float64)
    w[:, 1] = 15 * s0
    w[:, 2:58] = (np.arange(56) % 14 + 0.25) * s0
    w[:, 58:114] = (np.arange(56) % 14 + 0.75) * s0
    w = w.astype(np.float16)
    codes, s, z = O.quantize_groups_ex(w, 4, 128, STO, seed=11)
    assert (s.astype(np.float64) == s0).all()
    base = np.arange(56) % 14
    up_q = (codes[:, 2:58].astype(np.int64) - base).astype(np.float64)
    up_3q = (codes[:, 58:114].astype(np.int64) - base).astype(np.float64)
    assert set(np.unique(up_q)) <= {0.0, 1.0} and set(np.unique(up_3q)) <= {0.0, 1.0}
    n = up_q.size
    sd = np.sqrt(0.25 * 0.75 / n)
    assert abs(up_q.mean() - 0.25) < 5 * sd and abs(up_3q.mean() - 0.75) < 5 * sd


def test_stochastic_is_unbiased():
    # E[w~] = w: the mean over 400 seeds of w~ - w, in units of its theoretical standard deviation
    # s sqrt(f (1 - f) / N) (f = fractional part of the exact scaled value), is ~N(0, 1); weights whose
    # ceiling would be clamped (above 2^b - 1) are excluded
    w = synth.weight_f16(41, 16, 128)
    N = 400
    acc = np.zeros(w.shape)
    for seed in range(N):
        acc += O.QWeight(w, 3, mode=STO, seed=seed).dequant() - w.astype(np.float64)
    mean = acc / N
    _, s, z = O.quantize_groups_ex(w, 3, 128, STO)
    S, Z = s.astype(np.float64).repeat(128, 1), z.astype(np.float64).repeat(128, 1)
    d = (w.astype(np.float64) - Z) / S
    f = d - np.floor(d)
    ok = (np.floor(d) + 1 <= 7) & (f > 1e-6) & (f < 1 - 1e-6)
    zsc = np.abs(mean[ok]) / (S[ok] * np.sqrt(f[ok] * (1 - f[ok]) / N))
    assert ok.sum() > 1800
    assert zsc.mean() < 0.9 and np.mean(zsc < 4) > 0.999   # E|N(0,1)| = 0.80
    agg = abs(mean[ok].sum()) / np.sqrt((S[ok] ** 2 * f[ok] * (1 - f[ok])).sum() / N)  # ~|N(0, 1)|
    assert agg < 4


@pytest.mark.parametrize("bits", [3, 4])
def test_theorem1_stochastic_variance(bits):
    # P:176-180 Thm. 1, stochastic case: the rounding adds D S^2 (E[X]^2 + Var[X]) / 6 to the output
    # variance (over the rounding randomness; uniform fractional parts give E[f(1-f)] = 1/6 exactly).
    # Rounding to nearest would give ~1/12 of Var-only terms: the E[X]^2 term and the 1/6 are pinned.
    n, k, m, N = 16, 1024, 24, 120
    w = synth.weight_f16(51, n, k)
    x = (synth.act_f16(52, m, k).astype(np.float64) + 0.75).astype(np.float16)
    y_exact = x.astype(np.float64) @ w.astype(np.float64).T
    dy2 = np.zeros((m, n))
    for seed in range(N):
        dy = O.linear(x, O.QWeight(w, bits, mode=STO, seed=seed)) - y_exact
        dy2 += dy * dy
    added = (dy2 / N).mean(0)                                  # per output row
    s2 = (O.quantize_groups_ex(w, bits, 128, STO)[1].astype(np.float64) ** 2)
    xd = x.astype(np.float64)
    bound = (128 * s2).sum(1) * (xd.mean() ** 2 + xd.var()) / 6.0
    ratio = added / bound
    assert 0.85 <= ratio.mean() <= 1.15, ratio.mean()
    assert ratio.mean() > 1.15 * (xd.var() / (xd.mean() ** 2 + xd.var()))  # the E[X]^2 term matters


def test_indicator_symmetric_scale():
    # eq. (3) weight term with P:184's symmetric S_W: sum over groups of 128 * S_g^2
    w = synth.weight_f16(61, 4, 256)
    _, s, _ = O.quantize_groups_ex(w, 4, 128, SYM)
    assert O.scale_sq_sum(w, 4, 128, SYM) == pytest.approx(float((128 * s.astype(np.float64) ** 2).sum()), rel=1e-15)
    assert O.scale_sq_sum(w, 4, 128, SYM) > O.scale_sq_sum(w, 4, 128)  # symmetric grids are coarser


# ---------------------------------------------------------------- GPU: bit-exact with the oracle
def _sq():
    import paper_conf_cluster_zhaowplw25_b200 as sq
    return sq


@pytest.mark.gpu
@pytest.mark.parametrize("mode", [SYM, STO, SYM | STO])
@pytest.mark.parametrize("bits", [3, 4, 8])
@pytest.mark.parametrize("group", [128, 64, 32])
def test_gpu_variants_bit_exact(mode, bits, group):
    import torch
    sq = _sq()
    w = synth.adversarial_weight_f16(70 + bits, 64, 512)
    if mode & SYM:  # keep every symmetric zero point inside fp16 (the overflow case is tested below)
        w = (w.astype(np.float32) * np.float32(0.5)).astype(np.float16)
    codes, s, z = O.quantize_groups_ex(w, bits, group, mode, seed=1234 + bits)
    gc, gs, gz = sq.sq_quantize_groups_ex(torch.from_numpy(w).cuda(), bits, group, mode, 1234 + bits)
    assert np.array_equal(gc.cpu().numpy(), codes)
    assert np.array_equal(gs.cpu().numpy().view(np.uint16), s.view(np.uint16))
    assert np.array_equal(gz.cpu().numpy().view(np.uint16), z.view(np.uint16))


@pytest.mark.gpu
@pytest.mark.parametrize("mode", [SYM, STO])
def test_gpu_variants_bit_exact_opt13b_and_linear(mode):
    # full OPT-13B 5120 x 5120 (device-generated, same generator); then a decode and a prefill linear
    # on the variant-quantized weight vs the oracle's (the stored form is the same (code, s, z))
    import torch
    sq = _sq()
    n = k = 5120
    seed = synth.weight_seed(0, "o")
    wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
    synth.device_weight_f16(wd.data_ptr(), seed, n, k)
    w = synth.weight_f16(seed, n, k)
    codes, s, z = O.quantize_groups_ex(w, 4, 128, mode, seed=99)
    gc, gs, gz = sq.sq_quantize_groups_ex(wd, 4, 128, mode, 99)
    assert np.array_equal(gc.cpu().numpy(), codes)
    assert np.array_equal(gs.cpu().numpy().view(np.uint16), s.view(np.uint16))
    rows = np.arange(0, n, 40)
    qg = sq.QLinear.from_fp16(wd, 4, mode=mode, seed=99)
    packed, meta = O.pack(codes, s, z, 4)
    assert np.array_equal(qg.packed.cpu().numpy(), packed)
    x = synth.act_f16(5, 8, k)
    y = torch.empty((8, n), dtype=torch.float16, device="cuda")
    sq.sq_linear_decode(qg, torch.from_numpy(x).cuda(), y, 0)
    torch.cuda.synchronize()
    # y = x (s c + z)^T on sampled rows from the oracle's codes (O4/O5 written out in fp64)
    ref = x.astype(np.float64) @ (codes[rows].astype(np.float64) * s[rows].astype(np.float64).repeat(128, 1)
                                  + z[rows].astype(np.float64).repeat(128, 1)).T
    yy = y.float().cpu().numpy()[:, rows]
    assert np.abs(yy - ref).max() / np.abs(ref).max() <= 2e-3


@pytest.mark.gpu
def test_gpu_symmetric_overflow_flag():
    import torch
    sq = _sq()
    w = np.zeros((16, 128), np.float16)
    w[3, 9] = np.float16(60000.0)
    with pytest.raises(RuntimeError):
        O.quantize_groups_ex(w, 4, 128, SYM)
    with pytest.raises(sq.SQError):
        sq.sq_quantize_groups_ex(torch.from_numpy(w).cuda(), 4, 128, SYM)
