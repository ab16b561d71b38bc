"""GPU parity: quantize/pack bit-exact and decode/prefill linears vs the CPU oracle.

Tolerance for floating point (R10, BASELINE.json north_star):
normwise max|y - y_ref| / max|y_ref| <= 2e-3 against the fp64 oracle.
Codes, scales, zeros, packed words and meta must match bit-exactly.
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import synth
from oracle import oracle as O

pytestmark = pytest.mark.gpu
TOL = 2e-3


def sqm():
    import paper_conf_cluster_zhaowplw25_b200 as sq
    return sq


def normwise(y, ref):
    y = np.asarray(y, np.float64)
    ref = np.asarray(ref, np.float64)
    return float(np.abs(y - ref).max() / max(np.abs(ref).max(), 1e-30))


def adversarial_weight(n=64, k=512, seed=3):
    return synth.adversarial_weight_f16(seed, n, k)


ADV_ROWS = [3, 8, 9, 10, 11, 12]  # rows holding +-65504 (their outputs dwarf the others)


def check_adversarial(y, ref):
    """Finite outputs; normwise over the tensor (R10), and separately over the ordinary rows, whose
    magnitudes the +-65504 rows would otherwise hide."""
    assert np.isfinite(y).all()
    assert normwise(y, ref) <= TOL, normwise(y, ref)
    keep = np.setdiff1d(np.arange(ref.shape[1]), ADV_ROWS)
    assert normwise(y[:, keep], ref[:, keep]) <= TOL, normwise(y[:, keep], ref[:, keep])


@pytest.mark.parametrize("bits", [3, 4, 8])
@pytest.mark.parametrize("group", [128, 64, 32])
def test_quantize_bit_exact_adversarial(bits, group):
    sq = sqm()
    w = adversarial_weight()
    codes, s, z = O.quantize_groups(w, bits, group)
    gc, gs, gz = sq.sq_quantize_groups(torch.from_numpy(w).cuda(), bits, group)
    assert np.array_equal(gc.cpu().numpy(), codes)
    assert np.array_equal(gs.cpu().numpy().view(np.uint16), s.view(np.uint16))
    assert np.array_equal(gz.cpu().numpy().view(np.uint16), z.view(np.uint16))


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_pack_bit_exact(bits):
    sq = sqm()
    w = adversarial_weight(n=48, k=640, seed=bits)
    codes, s, z = O.quantize_groups(w, bits)
    packed, meta = O.pack(codes, s, z, bits)
    gp, gm = sq.sq_pack(torch.from_numpy(codes).cuda(), torch.from_numpy(s).cuda(), torch.from_numpy(z).cuda(), bits)
    assert np.array_equal(gp.cpu().numpy(), packed)
    assert np.array_equal(gm.cpu().numpy().view(np.uint32).reshape(-1), meta.reshape(-1))


@pytest.mark.parametrize("bits", [3, 4, 8])
def test_quantize_pack_bit_exact_opt13b_linear(bits):
    # full OPT-13B q/k/v/o shape (5120 x 5120), device-generated weights (same generator)
    sq = sqm()
    n = k = 5120
    seed = synth.weight_seed(0, "o")
    wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
    synth.device_weight_f16(wd.data_ptr(), seed, n, k)
    w = synth.weight_f16(seed, n, k)
    assert np.array_equal(wd.cpu().numpy().view(np.uint16), w.view(np.uint16))
    codes, s, z = O.quantize_groups(w, bits)
    packed, meta = O.pack(codes, s, z, bits)
    q = sq.QLinear.from_fp16(wd, bits)
    assert np.array_equal(q.packed.cpu().numpy(), packed)
    assert np.array_equal(q.meta.cpu().numpy().view(np.uint32).reshape(-1), meta.reshape(-1))


def _make(bits, n, k, seed, bias=True):
    sq = sqm()
    w = synth.weight_f16(seed, n, k)
    b = synth.bias_f16(seed, n) if bias else None
    qo = O.QWeight(w, bits, bias=b)
    qg = sq.QLinear.from_fp16(torch.from_numpy(w).cuda(), bits, torch.from_numpy(b).cuda() if bias else None)
    return qo, qg


def _ref_epi(y, epi):
    if epi == 1:
        return np.maximum(y, 0)
    if epi == 2:
        return 0.5 * y * (1 + np.tanh(np.sqrt(2 / np.pi) * (y + 0.044715 * y ** 3)))
    return y


def _run_linear(kind, qg, x, epi, y0=None):
    sq = sqm()
    m = x.shape[0]
    xt = torch.from_numpy(x).cuda()
    if epi == sq.SQ_EPI_F32_ACCUM:
        y = torch.from_numpy(y0.copy()).cuda()
    else:
        y = torch.empty((m, qg.n), dtype=torch.float16, device="cuda")
    if kind == "decode":
        sq.sq_linear_decode(qg, xt, y, epi)
    else:
        sq.sq_linear_prefill(qg, xt, y, epi)
    torch.cuda.synchronize()
    return y.float().cpu().numpy().astype(np.float64)


SHAPES = [(256, 512), (144, 384), (768, 768), (1024, 128), (528, 1280)]


@pytest.mark.parametrize("bits", [3, 4, 8, 16])
@pytest.mark.parametrize("m", [1, 2, 5, 8, 9, 16, 17, 32])
def test_decode_parity(bits, m):
    for si, (n, k) in enumerate(SHAPES):
        qo, qg = _make(bits, n, k, seed=100 + si)
        x = synth.act_f16(200 + m, m, k)
        ref = O.linear(x, qo)
        y = _run_linear("decode", qg, x, 0)
        assert normwise(y, ref) <= TOL, (n, k, normwise(y, ref))


@pytest.mark.parametrize("bits", [3, 4, 8, 16])
@pytest.mark.parametrize("epi", [1, 2, 3])
@pytest.mark.parametrize("n,m", [(272, 3), (640, 32)])
def test_decode_epilogues(bits, epi, n, m):
    k = 640
    qo, qg = _make(bits, n, k, seed=300)
    x = synth.act_f16(301, m, k)
    lin = O.linear(x, qo)
    if epi == 3:
        y0 = synth.hidden_f32(302, m, n)
        y = _run_linear("decode", qg, x, epi, y0)
        assert normwise(y - y0, lin) <= TOL
    else:
        y = _run_linear("decode", qg, x, epi)
        assert normwise(y, _ref_epi(lin, epi)) <= TOL


@pytest.mark.parametrize("bits", [3, 4, 8, 16])
@pytest.mark.parametrize("m", [7, 32])
def test_decode_deterministic(bits, m):
    n, k = 2048, 1536
    qo, qg = _make(bits, n, k, seed=400)
    x = synth.act_f16(401, m, k)
    a = _run_linear("decode", qg, x, 0)
    b = _run_linear("decode", qg, x, 0)
    assert np.array_equal(a, b)


@pytest.mark.parametrize("bits", [3, 4, 8])
@pytest.mark.parametrize("m", [12, 32])
@pytest.mark.parametrize("n,k", [(640, 9216), (128, 4992), (1920, 384)])
def test_decode_tc_split_panels(bits, m, n, k):
    """tcgen05 path (m > 8): panels split over many CTAs (fix-up order), a ragged last panel,
    one-tile panels and odd k/128 (one group per unit)."""
    qo, qg = _make(bits, n, k, seed=500 + n)
    x = synth.act_f16(501 + m, m, k)
    ref = O.linear(x, qo)
    y = _run_linear("decode", qg, x, 0)
    assert normwise(y, ref) <= TOL, (n, k, normwise(y, ref))
    assert np.array_equal(y, _run_linear("decode", qg, x, 0))


@pytest.mark.parametrize("bits", [3, 4, 8])
@pytest.mark.parametrize("shape", [(20480, 5120), (5120, 20480)])
def test_decode_full_size_sampled(bits, shape):
    # OPT-13B fc1 / fc2 at micro-batch 32 (configs[1]); oracle on 48 sampled output rows
    sq = sqm()
    n, k = shape
    seed = synth.weight_seed(1, "fc1" if n > k else "fc2")
    wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
    synth.device_weight_f16(wd.data_ptr(), seed, n, k)
    qg = sq.QLinear.from_fp16(wd, bits)
    del wd
    m = 32
    x = synth.act_f16(7, m, k)
    y = _run_linear("decode", qg, x, 0)
    rows = np.random.default_rng(bits).choice(n, 48, replace=False)
    rows[0], rows[1] = 0, n - 1
    wr = synth.weight_f16(seed, n, k, rows=rows)
    ref = O.linear(x, O.QWeight(wr, bits))
    assert normwise(y[:, rows], ref) <= TOL


@pytest.mark.parametrize("bits", [3, 4, 8, 16])
@pytest.mark.parametrize("m", [1, 37, 128, 300, 513])
def test_prefill_parity(bits, m):
    for si, (n, k) in enumerate([(256, 512), (384, 1280), (128, 128)]):
        qo, qg = _make(bits, n, k, seed=500 + si)
        x = synth.act_f16(600 + m, m, k)
        ref = O.linear(x, qo)
        y = _run_linear("prefill", qg, x, 0)
        assert normwise(y, ref) <= TOL, (n, k, m, normwise(y, ref))


@pytest.mark.parametrize("bits", [4, 16])
@pytest.mark.parametrize("epi", [1, 2, 3])
def test_prefill_epilogues(bits, epi):
    n, k, m = 384, 512, 77
    qo, qg = _make(bits, n, k, seed=700)
    x = synth.act_f16(701, m, k)
    lin = O.linear(x, qo)
    if epi == 3:
        y0 = synth.hidden_f32(702, m, n)
        y = _run_linear("prefill", qg, x, epi, y0)
        assert normwise(y - y0, lin) <= TOL
    else:
        y = _run_linear("prefill", qg, x, epi)
        assert normwise(y, _ref_epi(lin, epi)) <= TOL


def test_one_token_prefill_equals_decode_function():
    # S8c: a 1-token prefill computes the same function as a decode step
    qo, qg = _make(4, 512, 1024, seed=800)
    x = synth.act_f16(801, 1, 1024)
    a = _run_linear("prefill", qg, x, 0)
    b = _run_linear("decode", qg, x, 0)
    ref = O.linear(x, qo)
    assert normwise(a, ref) <= TOL and normwise(b, ref) <= TOL


@pytest.mark.parametrize("path", ["mma", "mma-k2", "mma-k2s", "mma-k2s16", "tc", "tc-nocluster"])
def test_decode_forced_path(path):
    """Every decode kernel (mma.sync K2 and its strip form K2s, tcgen05 K2c) for every bit width and m
    in 1..32, whatever the automatic choice (gemv_path, use_k2s) would pick: SQ_GEMV_PATH forces the
    family, SQ_K2S=0 / 1 K2 / K2s for m <= 8 (read once per process).  "tc-nocluster" forces K2c's
    global-memory split-k fix-up instead of the cluster/DSMEM reduction (SQ_TC_CLUSTER=0), the
    fallback taken when the clusters cannot all be resident."""
    import os
    import subprocess
    import sys
    env = dict(os.environ, SQ_GEMV_PATH=path.split("-")[0])
    if path == "tc-nocluster":
        env["SQ_TC_CLUSTER"] = "0"
    if path.startswith("mma-k2"):
        env["SQ_K2S"] = "1" if path.startswith("mma-k2s") else "0"
    if path == "mma-k2s16":
        env["SQ_K2S16"] = "1"  # m in 9..16 on K2s too (two token tiles)
    script = os.path.join(os.path.dirname(os.path.abspath(__file__)), "_decode_path_check.py")
    r = subprocess.run([sys.executable, script], env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]


def _adv_case(bits, m, seed):
    sq = sqm()
    n, k = 256, 512
    w = adversarial_weight(n, k, seed=seed)
    b = synth.bias_f16(seed, n)
    qo = O.QWeight(w, bits, bias=b)
    qg = sq.QLinear.from_fp16(torch.from_numpy(w).cuda(), bits, torch.from_numpy(b).cuda())
    # fp16 outputs: activations scaled by 1/16 (exact) so the +-65504 rows stay inside fp16's range
    x = (synth.act_f16(seed + 1, m, k) * np.float16(0.0625)).astype(np.float16)
    x32 = synth.act_f16(seed + 2, m, k)
    return qo, qg, x, x32


@pytest.mark.parametrize("bits", [3, 4, 8])
@pytest.mark.parametrize("m", [1, 8, 32])
def test_decode_adversarial(bits, m):
    """R20: groups spanning +-65504 dequantize to a finite top code on every decode kernel; constant,
    -0, subnormal and tie groups in the same tile (both the fp16 and the fp32-residual epilogues)."""
    qo, qg, x, x32 = _adv_case(bits, m, 40 + bits)
    check_adversarial(_run_linear("decode", qg, x, 0), O.linear(x, qo))
    y0 = synth.hidden_f32(43, m, qg.n)
    y = _run_linear("decode", qg, x32, 3, y0)
    check_adversarial(y - y0, O.linear(x32, qo))


@pytest.mark.parametrize("bits", [3, 4, 8])
@pytest.mark.parametrize("m", [1, 300])
def test_prefill_adversarial(bits, m):
    qo, qg, x, x32 = _adv_case(bits, m, 50 + bits)
    check_adversarial(_run_linear("prefill", qg, x, 0), O.linear(x, qo))
    y0 = synth.hidden_f32(53, m, qg.n)
    y = _run_linear("prefill", qg, x32, 3, y0)
    check_adversarial(y - y0, O.linear(x32, qo))


@pytest.mark.parametrize("bits", [3, 4])
def test_decode_bloom_full_size_sampled(bits):
    """Maximum sizes of the workloads: BLOOM-176B fc1 / fc2 (configs[4], INT3 / INT4) on the automatic
    decode path at m = 1, 8, 32 -- 32 sampled rows vs the oracle and a bitwise repeat."""
    import os
    import subprocess
    import sys
    script = os.path.join(os.path.dirname(os.path.abspath(__file__)), "_decode_path_check.py")
    r = subprocess.run([sys.executable, script, "bloom", str(bits)], capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]


@pytest.mark.parametrize("kern", ["k2", "k2s"])
def test_decode_mma_writes_in_bounds(kern):
    """K2 / K2s write nothing outside y's window and the workspace, and reset every split-k counter
    (sentinel-filled buffers; the substitute for compute-sanitizer, which this pool has closed)."""
    import os
    import subprocess
    import sys
    env = dict(os.environ, SQ_GEMV_PATH="mma", SQ_K2S="1" if kern == "k2s" else "0")
    script = os.path.join(os.path.dirname(os.path.abspath(__file__)), "_decode_path_check.py")
    r = subprocess.run([sys.executable, script, "canary"], env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]


@pytest.mark.parametrize("kern", ["k2", "k2s"])
@pytest.mark.parametrize("bits", [3, 4, 8])
def test_decode_mma_full_grid_sampled(bits, kern):
    """The mma.sync decode kernels at the configs[1] launch shape: OPT-13B fc1 (20480 x 5120) at m = 1
    (K2: one 16-warp CTA per SM, units split evenly; K2s: two 8-warp CTAs per SM, strip items split
    evenly; tiles / strips straddling CTAs -> cross-CTA fix-up), forced with SQ_GEMV_PATH=mma and
    SQ_K2S in a subprocess; 64 sampled output rows vs the oracle, and a bitwise repeat."""
    import os
    import subprocess
    import sys
    env = dict(os.environ, SQ_GEMV_PATH="mma", SQ_K2S="1" if kern == "k2s" else "0")
    script = os.path.join(os.path.dirname(os.path.abspath(__file__)), "_decode_path_check.py")
    r = subprocess.run([sys.executable, script, "full", str(bits)], env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]


def test_prefill_cta_pair_bitwise(tmp_path):
    """K3's CTA-pair tile (cta_group::2, the default for even n/128) and the one-CTA tile
    (SQ_GEMM_CG=1) accumulate every output in the same k order: their outputs are bit-identical
    (fp16 and fp32-residual epilogues, ragged token tiles whose second half is out of range)."""
    import os
    import subprocess
    import sys
    script = os.path.join(os.path.dirname(os.path.abspath(__file__)), "_prefill_cg_dump.py")
    res = {}
    for cg in ("1", "2"):
        env = dict(os.environ, SQ_GEMM_CG=cg)
        path = str(tmp_path / f"cg{cg}.npz")
        r = subprocess.run([sys.executable, script, path], env=env, capture_output=True, text=True, timeout=600)
        assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
        res[cg] = np.load(path)
    for key in res["1"].files:
        a, b = res["1"][key], res["2"][key]
        assert np.array_equal(a.view(np.uint8), b.view(np.uint8)), key
