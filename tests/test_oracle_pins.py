"""Pins for the CPU oracle (oracle/) against what the paper and mathematics fix.

Each test pins one oracle function to something other than itself (brute force,
closed forms, invariants, textbook routines, hand-derived golden words), chosen
so that a dropped term, a wrong sign/index or a transposed operand fails one.
Citations: PAPER.md line numbers (P:<line>); readings R1..R16.
"""
from __future__ import annotations

import os
from fractions import Fraction

import numpy as np
import pytest

from oracle import oracle as O
import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "pack_words.txt")


def _f16(a):
    return np.asarray(a, dtype=np.float16)


# ---------------------------------------------------------------- O1 quantize
def _brute_codes(w: np.ndarray, s: float, z: float, bits: int) -> np.ndarray:
    """argmin_c |w - (s c + z)| over all 2^b grid points, exact rationals, ties -> even c."""
    qmax = (1 << bits) - 1
    S, Z = Fraction(float(s)), Fraction(float(z))
    out = np.empty(len(w), np.int64)
    for j, wj in enumerate(w):
        W = Fraction(float(wj))
        best, bestd = None, None
        for c in range(qmax + 1):
            d = abs(W - (S * c + Z))
            if bestd is None or d < bestd or (d == bestd and c % 2 == 0):
                best, bestd = c, d
        out[j] = best
    return out


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_quantize_matches_bruteforce_argmin(bits):
    # P:91 round((x - q_x)/s_x) == nearest grid point; R1 half-even at exact ties.
    w = synth.weight_f16(7 + bits, 3, 256)
    codes, s, z = O.quantize_groups(w, bits, 128)
    for r in range(w.shape[0]):
        for g in range(2):
            sl = slice(128 * g, 128 * (g + 1))
            bc = _brute_codes(w[r, sl], s[r, g], z[r, g], bits)
            oc = codes[r, sl].astype(np.int64)
            bad = np.nonzero(bc != oc)[0]
            for j in bad:  # only fp32-rounding near-ties may differ; both then within s/2
                W = Fraction(float(w[r, sl][j]))
                S, Z = Fraction(float(s[r, g])), Fraction(float(z[r, g]))
                assert abs(abs(W - (S * int(oc[j]) + Z)) - abs(W - (S * int(bc[j]) + Z))) <= S * Fraction(1, 1 << 20)


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_exact_ties_round_half_even(bits):
    # R1: P:91's rounding function at EXACT ties.  s0 = 2^-6 and the group spans [0, qmax*s0], so the
    # stored scale is exactly s0 and (w - z)/s = c + 1/2 exactly in fp32: half-to-even must give the
    # even neighbour (roundf / floor(x + 0.5) give c + 1 at every even c and fail).
    qmax = (1 << bits) - 1
    s0 = 2.0 ** -6
    w = np.zeros((1, 128), np.float64)
    w[0, 0], w[0, 1] = 0.0, qmax * s0
    nt = min(qmax, 126)
    w[0, 2:2 + nt] = (np.arange(nt) + 0.5) * s0
    codes, s, z = O.quantize_groups(w.astype(np.float16), bits)
    assert float(s[0, 0]) == s0 and float(z[0, 0]) == 0.0
    want = np.arange(nt) + (np.arange(nt) % 2)  # c + 1/2 -> c if c even, c + 1 if c odd
    assert np.array_equal(codes[0, 2:2 + nt].astype(np.int64), want)
    if bits == 3:  # written out by hand: 0.5, 1.5, ..., 6.5 -> 0, 2, 2, 4, 4, 6, 6
        assert list(codes[0, 2:9]) == [0, 2, 2, 4, 4, 6, 6]


# R20 hand computation for a group holding +-65504 (the rest 0):
#   INT3: s = fp16(131008/7 = 18715.43) = 18720 (spacing 16); c(65504) = rint(6.998) = 7 -> 65536 -> 65504;
#         c(0) = rint(65504/18720 = 3.499) = 3 -> 3*18720 - 65504 = -9344
#   INT4: s = fp16(131008/15 = 8733.87) = 8736 (spacing 8);  c(65504) = 15 -> 65536 -> 65504;
#         c(0) = rint(7.498) = 7 -> 61152 - 65504 = -4352
#   INT8: s = fp16(131008/255 = 513.76) = 514 (spacing 0.5); c(65504) = rint(254.88) = 255 -> 65566 -> 65504;
#         c(0) = rint(127.44) = 127 -> 65278 - 65504 = -226
@pytest.mark.parametrize("bits,scale,w_zero", [(3, 18720.0, -9344.0), (4, 8736.0, -4352.0), (8, 514.0, -226.0)])
def test_dequant_saturates_at_fp16_max(bits, scale, w_zero):
    w = np.zeros((16, 128), np.float16)
    w[0, 0], w[0, 1] = np.float16(65504.0), np.float16(-65504.0)
    q = O.QWeight(w, bits)
    assert float(q.scales[0, 0]) == scale and float(q.zeros[0, 0]) == -65504.0
    wt = q.dequant()
    assert wt[0, 0] == 65504.0 and wt[0, 1] == -65504.0 and wt[0, 2] == w_zero
    assert np.isfinite(wt).all()


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_scale_zero_closed_form(bits):
    # P:91 s = (x_max - x_min)/(2^b - 1), q = x_min (R3), scale stored fp16 (R5).
    w = synth.weight_f16(11, 16, 512)
    codes, s, z = O.quantize_groups(w, bits, 128)
    qmax = (1 << bits) - 1
    g = w.astype(np.float64).reshape(16, 4, 128)
    mn, mx = g.min(-1), g.max(-1)
    assert np.array_equal(z.astype(np.float64), mn + 0.0)
    exact = (mx - mn) / qmax
    rel = np.abs(s.astype(np.float64) - exact) / exact
    assert rel.max() <= 2.0 ** -11 * 1.0001
    c = codes.reshape(16, 4, 128)
    assert (c.min(-1) == 0).all() and (c.max(-1) == qmax).all()  # group min -> 0, max -> 2^b-1


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_half_step_bound_with_outliers(bits):
    # |w - w~| <= s/2 for every weight incl. the clamped top (R5).
    w = synth.weight_f16(21, 64, 1024).copy()
    w[3, 5] = np.float16(60000.0)
    w[9, 700] = np.float16(-65504.0)
    w[10, 128:256] = np.float16(6.1e-5)  # subnormal-scale neighbourhood
    q = O.QWeight(w, bits)
    wt = q.dequant()
    s = q.scales.astype(np.float64).repeat(128, axis=1)
    err = np.abs(wt - w.astype(np.float64))
    assert (err <= s / 2 * (1 + 1e-6) + 1e-300).all()


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_grid_aligned_weights_recovered_exactly(bits):
    # Special case: W on a quantization grid with codes spanning 0..2^b-1 -> lossless.
    w, c, s, z = synth.grid_aligned_weight_f16(5, 16, 256, bits)
    codes, s2, z2 = O.quantize_groups(w, bits, 128)
    assert np.array_equal(codes, c)
    assert np.array_equal(s2, s) and np.array_equal(z2, z)
    q = O.QWeight(w, bits)
    assert np.array_equal(q.dequant(), w.astype(np.float64))


def test_constant_and_negative_zero_groups():
    # R6: mx == mn -> s = 0, all codes 0, w~ = z = w exactly; -0.0 min canonicalised to +0.
    w = np.zeros((2, 256), np.float16)
    w[0, :128] = np.float16(-1.5)
    w[1, 128:] = np.float16(-0.0)
    codes, s, z = O.quantize_groups(w, 4, 128)
    assert (codes == 0).all() and (s.view(np.uint16) == 0).all()
    assert z[0, 0] == np.float16(-1.5) and z[1, 1].view(np.uint16) == 0


# ---------------------------------------------------------------- O2/O3 packing
def _golden():
    rows = []
    for line in open(GOLDEN):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        parts = line.split()
        words = {int(a): int(b, 16) for a, b in (p.split(":") for p in parts[2:])}
        rows.append((int(parts[0]), parts[1], words))
    return rows


def _example_codes(bits, name):
    c = np.zeros((16, 128), np.uint8)  # one 16-row tile (T16); the example lives in row 0
    if name == "ramp":
        c[0] = np.arange(128) % (1 << bits)
    elif name == "single13":
        c[0, 13] = 0xA
    elif name == "single3":
        c[0, 13], c[0, 22], c[0, 30], c[0, 63], c[0, 100] = 5, 6, 5, 3, 7
    elif name == "single5":
        c[0, 5] = 200
    return c


@pytest.mark.parametrize("row", _golden(), ids=lambda r: f"b{r[0]}-{r[1]}")
def test_pack_hand_derived_words(row):
    bits, name, words = row
    c = _example_codes(bits, name)
    s = np.zeros((16, 1), np.float16)
    packed, meta = O.pack(c, s, s, bits)
    gb = 128 * bits // 8
    got = packed.reshape(-1)[:gb].view("<u4")  # row 0's chunk of unit (tile 0, group 0)
    assert not packed.reshape(-1)[gb:].any()
    for i, wv in words.items():
        assert got[i] == wv, (i, hex(got[i]), hex(wv))
    if name.startswith("single"):
        rest = [i for i in range(len(got)) if i not in words]
        assert (got[rest] == 0).all()


@pytest.mark.parametrize("bits", [3, 4, 8])
@pytest.mark.parametrize("shape", [(16, 128), (32, 384), (48, 1024)])
def test_pack_unpack_round_trip(bits, shape):
    rng = np.random.default_rng(bits * 100 + shape[1])
    c = rng.integers(0, 1 << bits, size=shape).astype(np.uint8)
    s = np.zeros((shape[0], shape[1] // 128), np.float16)
    packed, _ = O.pack(c, s, s, bits)
    assert packed.shape == (shape[0], shape[1] * bits // 8)
    assert np.array_equal(O.unpack(packed, *shape, bits), c)


def test_tile_placement_t16():
    # T16: the packed bytes are [n/16 tiles][k/128 groups][16 rows][GB] --
    # written here as a numpy reshape/transpose of the row-major codes (not the oracle's index
    # arithmetic), plus byte offsets derived by hand from the layout definition:
    #   n = 32, k = 384, bits 8 (GB = 128, kg = 3): row 17, k 130 -> tile 1, group 1, row-in-tile 1
    #   -> unit 1*3 + 1 = 4 -> byte (4*16 + 1)*128 + 2 = 8322;  row 0, k 383 -> unit 2 -> 2*16*128 + 127 = 4223;
    #   meta of (row 31, group 0) -> unit 3, entry 3*16 + 15 = 63.
    rng = np.random.default_rng(3)
    n, k, bits = 32, 384, 8
    c = rng.integers(0, 256, size=(n, k)).astype(np.uint8)
    s = rng.standard_normal((n, 3)).astype(np.float16)
    z = rng.standard_normal((n, 3)).astype(np.float16)
    packed, meta = O.pack(c, s, z, bits)
    flat = packed.reshape(-1)
    assert np.array_equal(flat, c.reshape(2, 16, 3, 128).transpose(0, 2, 1, 3).reshape(-1))
    assert flat[8322] == c[17, 130] and flat[4223] == c[0, 383]
    word = s.view(np.uint16).astype(np.uint32) | (z.view(np.uint16).astype(np.uint32) << 16)
    assert np.array_equal(meta.reshape(-1), word.reshape(2, 16, 3).transpose(0, 2, 1).reshape(-1))
    assert meta.reshape(-1)[63] == word[31, 0]
    # L4 under T16: the same transpose on the nibble-packed rows (2 rows x 1 group = 2 x 64 bytes)
    c4 = rng.integers(0, 16, size=(16, 256)).astype(np.uint8)
    p4, _ = O.pack(c4, s[:16, :2], z[:16, :2], 4)
    one = np.stack([O.pack(c4[:, 128 * g:128 * (g + 1)], s[:16, :1], z[:16, :1], 4)[0] for g in range(2)])
    assert np.array_equal(p4.reshape(-1), one.reshape(-1))  # group-minor units of 16 rows x 64 B


@pytest.mark.parametrize("h1", [768, 5120, 7168, 9216, 14336])
@pytest.mark.parametrize("bits", [3, 4, 8])
def test_packed_bytes_equal_paper_memory_model(h1, bits):
    # decoder-layer weight bytes = (4 h1^2 + 2 h1 h2) * 4*bit/32, h2 = 4 h1 (R11).
    h2 = 4 * h1
    paper = (4 * h1 * h1 + 2 * h1 * h2) * 4 * bits // 32
    ours = (O.packed_bytes(3 * h1, h1, bits) + O.packed_bytes(h1, h1, bits)
            + O.packed_bytes(h2, h1, bits) + O.packed_bytes(h1, h2, bits))
    assert ours == paper


# ---------------------------------------------------------------- O4/O5 linear
def test_linear_fp16_equals_numpy_matmul():
    # R7: bits = 16 is the unquantized W.A16 linear; textbook fp64 GEMM.
    w = synth.weight_f16(31, 96, 384)
    x = synth.act_f16(32, 7, 384)
    b = synth.bias_f16(33, 96)
    y = O.linear(x, O.QWeight(w, 16, bias=b))
    ref = x.astype(np.float64) @ w.astype(np.float64).T + b.astype(np.float64)
    np.testing.assert_allclose(y, ref, rtol=1e-13, atol=1e-13)


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_linear_grid_aligned_equals_unquantized(bits):
    w, *_ = synth.grid_aligned_weight_f16(9, 48, 256, bits)
    x = synth.act_f16(10, 5, 256)
    yq = O.linear(x, O.QWeight(w, bits))
    y16 = x.astype(np.float64) @ w.astype(np.float64).T
    np.testing.assert_allclose(yq, y16, rtol=1e-13, atol=1e-13)


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_linear_is_x_times_dequantized_transpose(bits):
    # y[i, j] = sum_k x[i,k] (s c + z)[j,k]: numpy from the unpacked codes (catches a
    # transposed operand or a wrong scale/zero index in the C loops).
    w = synth.weight_f16(41, 48, 512)
    x = synth.act_f16(42, 3, 512)
    q = O.QWeight(w, bits)
    c = O.unpack(q.packed, 48, 512, bits).astype(np.float64)
    wt = c * q.scales.astype(np.float64).repeat(128, 1) + q.zeros.astype(np.float64).repeat(128, 1)
    np.testing.assert_allclose(O.linear(x, q), x.astype(np.float64) @ wt.T, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_theorem1_output_variance_bound(bits):
    # P:176-182 Thm. 1 (deterministic rounding): added variance <= D_W S_W^2 Var[X] / 4.
    # Uniform rounding error has variance S^2/12, so added/bound ~ 1/3.
    n, k, m = 64, 2048, 1024
    w = synth.weight_f16(51, n, k)
    x = synth.act_f16(52, m, k)
    q = O.QWeight(w, bits)
    dy = O.linear(x, q) - x.astype(np.float64) @ w.astype(np.float64).T
    added = dy.var(axis=0)
    s2 = (q.scales.astype(np.float64) ** 2)
    bound = (128 * s2).sum(axis=1) / 4.0 * x.astype(np.float64).var()
    ratio = added / bound
    assert 0.25 <= ratio.mean() <= 0.40
    assert ratio.max() <= 1.0


# ---------------------------------------------------------------- O6/O7 stage and pipeline
def test_layernorm_moments():
    x = synth.hidden_f32(61, 9, 768).astype(np.float64) * 3 + 1
    a = O.layernorm(x)
    np.testing.assert_allclose(a.mean(1), 0, atol=1e-12)
    v = x.var(1)
    np.testing.assert_allclose(a.var(1), v / (v + 1e-5), rtol=1e-12)


def _tiny_layers(h1=128, n_layers=3, bits=(4, 16, 3), act=0, bias=True):
    layers = []
    for l in range(n_layers):
        b = bits[l % len(bits)]
        mk = lambda name, n, k: O.QWeight(synth.weight_f16(synth.weight_seed(l, name), n, k), b,
                                          bias=synth.bias_f16(synth.weight_seed(l, name), n) if bias else None)
        layers.append(O.Layer(b, act, mk("qkv", 3 * h1, h1), mk("o", h1, h1), mk("fc1", 4 * h1, h1), mk("fc2", h1, 4 * h1)))
    return layers


@pytest.mark.parametrize("act", [0, 1])
def test_stage_equals_numpy_composition(act):
    # P:160 linear set per layer; R11 pre-LN glue; R12 attention stub out = V.
    layers = _tiny_layers(act=act)
    x = synth.hidden_f32(71, 6, 128).astype(np.float64)
    got, qkv = O.stage(layers, x, want_qkv=True)
    ref = x.copy()
    for L in layers:
        def lin(a, q):
            return a @ q.dequant().T + q.bias.astype(np.float64)
        def ln(t):
            mu = t.mean(1, keepdims=True)
            return (t - mu) / np.sqrt(((t - mu) ** 2).mean(1, keepdims=True) + 1e-5)
        qkv_ref = lin(ln(ref), L.qkv)
        hres = ref + lin(qkv_ref[:, 256:384], L.o)
        u = lin(ln(hres), L.fc1)
        u = np.maximum(u, 0) if act == 0 else 0.5 * u * (1 + np.tanh(np.sqrt(2 / np.pi) * (u + 0.044715 * u ** 3)))
        ref = hres + lin(u, L.fc2)
    np.testing.assert_allclose(got, ref, rtol=1e-10, atol=1e-10)
    np.testing.assert_allclose(qkv, qkv_ref, rtol=1e-10, atol=1e-10)


def test_stage_partition_invariance_and_row_independence():
    # Contiguous partition (eqs. 15-16) must not change results: stage(A+B) = stage(B)(stage(A)).
    layers = _tiny_layers(n_layers=4, bits=(3, 8, 16, 4))
    x = synth.hidden_f32(81, 5, 128).astype(np.float64)
    full, _ = O.stage(layers, x)
    a, _ = O.stage(layers[:1], x)
    b, _ = O.stage(layers[1:], a)
    assert np.array_equal(full, b)
    # a 1-token prefill equals the decode of that token (rows independent under the stub)
    one, _ = O.stage(layers, x[2:3])
    assert np.array_equal(one[0], full[2])


def test_pipeline_loopback_definition():
    # R13/R14 with layers whose stage function is known in closed form: every weight 0 (bits 16) and
    # only fc2 carrying a bias b, so a stage of L layers maps x -> x + L*b (the stub's v = 0, o = 0,
    # fc1 = 0 -> ReLU(0) = 0).  Then out[:, 0] = x0[:, s-1] + L b (LAST prompt position) and
    # out[:, t] = LN(out[:, t-1]) + L b, with LN the textbook numpy formula (eps 1e-5).
    h1, L = 128, 3
    rng = np.random.default_rng(5)
    bvec = rng.standard_normal(h1).astype(np.float16)
    zero = lambda n, k, bias=None: O.QWeight(np.zeros((n, k), np.float16), 16, bias=bias)
    layers = [O.Layer(16, 0, zero(3 * h1, h1), zero(h1, h1), zero(4 * h1, h1), zero(h1, 4 * h1, bvec))
              for _ in range(L)]
    x0 = synth.hidden_f32(91, 2 * 3 * h1, 1).reshape(2, 3, h1)
    out = O.pipeline(layers, x0, 2)
    lb = L * bvec.astype(np.float64)

    def ln(t):
        mu = t.mean(-1, keepdims=True)
        return (t - mu) / np.sqrt(((t - mu) ** 2).mean(-1, keepdims=True) + 1e-5)

    ref0 = x0[:, 2].astype(np.float64) + lb
    np.testing.assert_allclose(out[:, 0], ref0, rtol=1e-13, atol=1e-13)
    ref1 = ln(ref0) + lb
    np.testing.assert_allclose(out[:, 1], ref1, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(out[:, 2], ln(ref1) + lb, rtol=1e-12, atol=1e-12)
