"""GPU parity for stage forward (a5) and the pipeline run (a6) against the oracle.

configs[0] (OPT-125m shapes, 12 layers, bits {3,4,8,16}, prefill 1x32 + 8 decode
steps) end to end; larger shapes teacher-forced on sampled rows; partition
invariance of the virtual pipeline bitwise.
Tolerance: normwise 2e-3 (R10).
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import synth
from oracle import oracle as O

pytestmark = pytest.mark.gpu
TOL = 2e-3


def normwise(y, ref):
    y = np.asarray(y, np.float64)
    ref = np.asarray(ref, np.float64)
    return float(np.abs(y - ref).max() / max(np.abs(ref).max(), 1e-30))


def oracle_layers(n_layers, h1, h2, bits, act=0, bias=True, layer_offset=0, rows=None):
    """Same weights as runtime.build_layers (same seeds), quantized by the oracle."""
    layers = []
    dims = {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}
    for i in range(n_layers):
        l = layer_offset + i
        q = {}
        for name, (n, k) in dims.items():
            seed = synth.weight_seed(l, name)
            w = synth.weight_f16(seed, n, k)
            q[name] = O.QWeight(w, int(bits[i]), bias=synth.bias_f16(seed, n) if bias else None)
        layers.append(O.Layer(int(bits[i]), act, q["qkv"], q["o"], q["fc1"], q["fc2"]))
    return layers


def rt():
    import paper_conf_cluster_zhaowplw25_b200 as sq
    from paper_conf_cluster_zhaowplw25_b200 import runtime as R
    return sq, R


H1, H2, L = 768, 3072, 12   # OPT-125m (configs[0])


@pytest.fixture(scope="module")
def opt125m():
    sq, R = rt()
    bits = synth.bits_plan(2, L)
    g = R.build_layers(L, H1, H2, bits)
    o = oracle_layers(L, H1, H2, bits)
    return bits, g, o


@pytest.mark.parametrize("phase,T", [(0, 32), (0, 300), (1, 1), (1, 5), (1, 32)])
def test_stage_parity_opt125m(opt125m, phase, T):
    sq, R = rt()
    bits, g, o = opt125m
    x = synth.hidden_f32(11 + T, T, H1)
    ws = R.StageWorkspace(g, T)
    xi = torch.from_numpy(x).cuda()
    xo = torch.empty_like(xi)
    qkv = torch.empty((T, 3 * H1), dtype=torch.float16, device="cuda")
    R.sq_stage_forward(g, phase, xi, xo, ws, qkv_dbg=qkv)
    torch.cuda.synchronize()
    ref, ref_qkv = O.stage(o, x.astype(np.float64), want_qkv=True)
    assert normwise(xo.cpu().numpy(), ref) <= TOL
    assert normwise(qkv.float().cpu().numpy(), ref_qkv) <= TOL


@pytest.mark.parametrize("T", [1, 8, 32])
def test_decode_stage_cuda_graph(opt125m, T):
    """configs[0] decode step captured in ONE CUDA graph (SURVEY D-1): the stage forward is
    asynchronous on the caller's stream and allocation-free, so it captures as-is (PDL edges
    included); replays equal the eager run bitwise and the oracle within 2e-3."""
    sq, R = rt()
    bits, g, o = opt125m
    x = synth.hidden_f32(700 + T, T, H1)
    ws = R.StageWorkspace(g, T)
    xi = torch.from_numpy(x).cuda()
    xo_eager = torch.empty_like(xi)
    R.sq_stage_forward(g, 1, xi, xo_eager, ws)
    torch.cuda.synchronize()
    xo = torch.empty_like(xi)
    arr = R.layer_array(g)
    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(side):  # warm-up on the capture stream
        R.sq_stage_forward(g, 1, xi, xo, ws, arr=arr)
    torch.cuda.current_stream().wait_stream(side)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph):
        R.sq_stage_forward(g, 1, xi, xo, ws, arr=arr)
    for _ in range(3):
        xo.zero_()
        graph.replay()
    torch.cuda.synchronize()
    assert torch.equal(xo, xo_eager)
    ref, _ = O.stage(o, x.astype(np.float64))
    assert normwise(xo.cpu().numpy(), ref) <= TOL
    # graph replay vs eager launches: per-step latency of the 12-layer decode step
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(20):
        graph.replay()
    e1.record()
    torch.cuda.synchronize()
    print(f"configs[0] decode step T={T}: {e0.elapsed_time(e1) / 20 * 1e3:.1f} us per step (CUDA graph)")


def test_stage_in_place_and_gelu():
    sq, R = rt()
    bits = [4, 16]
    g = R.build_layers(2, 256, 1024, bits, act=1, layer_offset=40)
    o = oracle_layers(2, 256, 1024, bits, act=1, layer_offset=40)
    x = synth.hidden_f32(5, 7, 256)
    for phase in (0, 1):
        ws = R.StageWorkspace(g, 7)
        xt = torch.from_numpy(x).cuda()
        R.sq_stage_forward(g, phase, xt, xt, ws)  # x_in aliases x_out
        torch.cuda.synchronize()
        ref, _ = O.stage(o, x.astype(np.float64))
        assert normwise(xt.cpu().numpy(), ref) <= TOL


def _run_pipeline(R, g, bits, sol, B, eta, xi, s, n_dec, h1, h2, x0):
    plan = R.Plan(bits, sol, h1, h2, B, eta, xi, s, n_dec)
    R.sq_plan_check(plan)
    comm = R.Comm.local(plan.n_stages)
    ws = R.PipelineWorkspace(plan, g, -1)
    out = torch.zeros((B, 1 + n_dec, h1), dtype=torch.float32, device="cuda")
    st = R.sq_pipeline_run(plan, -1, g, comm, x0, out, ws)
    comm.destroy()
    return out.cpu().numpy(), st


def test_pipeline_configs0_end_to_end(opt125m):
    # BASELINE.json configs[0]: 12 layers, bits {3,4,8,16}, prefill 1x32 tokens + 8 decode steps
    sq, R = rt()
    bits, g, o = opt125m
    B, s, n_dec = 1, 32, 8
    x0 = synth.hidden_f32(1, B * s, H1).reshape(B, s, H1)
    out, st = _run_pipeline(R, g, bits, [0] * L, B, 1, 1, s, n_dec, H1, H2, torch.from_numpy(x0).cuda())
    ref = O.pipeline(o, x0, n_dec)
    for t in range(1 + n_dec):
        assert normwise(out[:, t], ref[:, t]) <= TOL, (t, normwise(out[:, t], ref[:, t]))
    assert st["gpu_launches"] > 0 and st["t_total_ms"] > 0


def test_decode_graph_replay_bitwise_equals_eager(opt125m, tmp_path):
    """sq_pipeline_run replays cached CUDA graphs of the decode micro-batches (stub path): a second run
    replays them (graph_replays > 0), and the output equals a run with SQ_GRAPH=0 (eager launches,
    subprocess) bit for bit."""
    import os
    import subprocess
    import sys
    sq, R = rt()
    bits, g, o = opt125m
    B, eta, xi, s, n_dec = 3, 2, 2, 16, 4
    x0 = torch.from_numpy(synth.hidden_f32(9, B * s, H1).reshape(B, s, H1)).cuda()
    plan = R.Plan(bits, [0] * 6 + [1] * 6, H1, H2, B, eta, xi, s, n_dec)
    comm = R.Comm.local(2)
    ws = R.PipelineWorkspace(plan, g, -1)
    out = torch.zeros((B, 1 + n_dec, H1), dtype=torch.float32, device="cuda")
    R.sq_pipeline_run(plan, -1, g, comm, x0, out, ws)      # captures
    a = out.cpu().numpy()
    out.zero_()
    st = R.sq_pipeline_run(plan, -1, g, comm, x0, out, ws)  # replays
    comm.destroy()
    b = out.cpu().numpy()
    assert np.array_equal(a, b) and st["graph_replays"] > 0
    assert st["host_enqueue_ms"] > 0
    np.save(tmp_path / "graph.npy", b)
    code = f"""
import sys; sys.path.insert(0, {os.path.dirname(os.path.dirname(os.path.abspath(__file__)))!r})
import numpy as np, torch, synth
from paper_conf_cluster_zhaowplw25_b200 import runtime as R
H1, H2, L = {H1}, {H2}, {L}
bits = synth.bits_plan(2, L)
g = R.build_layers(L, H1, H2, bits)
plan = R.Plan(bits, [0] * 6 + [1] * 6, H1, H2, {B}, {eta}, {xi}, {s}, {n_dec})
comm = R.Comm.local(2)
ws = R.PipelineWorkspace(plan, g, -1)
x0 = torch.from_numpy(synth.hidden_f32(9, {B} * {s}, H1).reshape({B}, {s}, H1)).cuda()
out = torch.zeros(({B}, 1 + {n_dec}, H1), dtype=torch.float32, device="cuda")
st = R.sq_pipeline_run(plan, -1, g, comm, x0, out, ws)
assert st["graph_replays"] == 0
np.save({str(tmp_path / "eager.npy")!r}, out.cpu().numpy())
"""
    r = subprocess.run([sys.executable, "-c", code], env=dict(os.environ, SQ_GRAPH="0"), capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    assert np.array_equal(np.load(tmp_path / "eager.npy"), b)


def test_virtual_pipeline_partition_invariance(opt125m):
    # eqs. (15)-(16) contiguous uneven partitions must not change a single bit
    sq, R = rt()
    bits, g, o = opt125m
    B, eta, xi, s, n_dec = 4, 2, 2, 16, 3
    x0 = torch.from_numpy(synth.hidden_f32(3, B * s, H1).reshape(B, s, H1)).cuda()
    base, _ = _run_pipeline(R, g, bits, [0] * L, B, eta, xi, s, n_dec, H1, H2, x0)
    for sol in ([0] * 5 + [1] * 7, [0, 0, 0, 1, 1, 2, 2, 2, 2, 3, 3, 3], [0] * 11 + [1]):
        out, _ = _run_pipeline(R, g, bits, sol, B, eta, xi, s, n_dec, H1, H2, x0)
        assert np.array_equal(out, base), sol
    # micro-batch sizes change kernel shapes but not the function
    out, _ = _run_pipeline(R, g, bits, [0] * L, B, 4, 1, s, n_dec, H1, H2, x0)
    assert normwise(out, base) <= TOL
    ref = O.pipeline(o, x0.cpu().numpy(), n_dec)
    assert normwise(base, ref) <= TOL


def test_plan_check_rejects_non_contiguous():
    sq, R = rt()
    bad = R.Plan([4] * 4, [0, 1, 0, 1], 768, 3072, 1, 1, 1, 4, 1)
    with pytest.raises(sq.SQError):
        R.sq_plan_check(bad)
    with pytest.raises(sq.SQError):
        R.sq_plan_check(R.Plan([4, 5], [0, 0], 768, 3072, 1, 1, 1, 4, 1))
    with pytest.raises(sq.SQError):
        R.sq_plan_check(R.Plan([4, 4], [0, 0], 768, 3072, 1, 1, 33, 4, 1))


@pytest.mark.parametrize("bits", [3, 4, 8, 16])
def test_stage_opt13b_layer_teacher_forced(bits):
    # one OPT-13B-shaped layer (d = 5120), decode 32 tokens and prefill 512 tokens; oracle on 3 rows
    sq, R = rt()
    h1, h2 = 5120, 20480
    g = R.build_layers(1, h1, h2, [bits], layer_offset=7)
    o = oracle_layers(1, h1, h2, [bits], layer_offset=7)
    for phase, T in ((1, 32), (0, 512)):
        x = synth.hidden_f32(17 + T, T, h1)
        ws = R.StageWorkspace(g, T)
        xi = torch.from_numpy(x).cuda()
        xo = torch.empty_like(xi)
        R.sq_stage_forward(g, phase, xi, xo, ws)
        torch.cuda.synchronize()
        rows = [0, T // 2, T - 1]
        ref, _ = O.stage(o, x[rows].astype(np.float64))
        assert normwise(xo.cpu().numpy()[rows], ref) <= TOL


@pytest.mark.parametrize("bits", [3, 4])  # (8 and 16 at full OPT-13B size above; ~70 s of oracle each)
def test_stage_opt66b_layer_bench_config(bits):
    """One OPT-66B-shaped layer (d = 9216, configs[3]) in the launch configuration bench.py times:
    decode micro-batch xi = 32 tokens and prefill micro-batch eta x s = 8 x 512 = 4096 tokens;
    oracle teacher-forced on sampled rows (first, middle, last)."""
    sq, R = rt()
    h1, h2 = 9216, 36864
    g = R.build_layers(1, h1, h2, [bits], layer_offset=21)
    o = oracle_layers(1, h1, h2, [bits], layer_offset=21)
    for phase, T in ((1, 32), (0, 4096)):
        x = synth.hidden_f32(31 + T, T, h1)
        ws = R.StageWorkspace(g, T)
        xi = torch.from_numpy(x).cuda()
        xo = torch.empty_like(xi)
        R.sq_stage_forward(g, phase, xi, xo, ws)
        torch.cuda.synchronize()
        rows = [0, T // 2 + 1, T - 1]
        ref, _ = O.stage(o, x[rows].astype(np.float64))
        assert normwise(xo.cpu().numpy()[rows], ref) <= TOL, (phase, T)


def test_stage_bloom_width_layer():
    """configs[4] width: d = 14336 (BLOOM-176B LayerNorm, fused QKV 43008 x 14336, GeLU), with a
    reduced FFN (h2 = 4096) to bound the oracle's cost; decode 32 tokens and prefill 512 tokens,
    oracle teacher-forced on sampled rows."""
    sq, R = rt()
    h1, h2 = 14336, 4096
    g = R.build_layers(1, h1, h2, [4], act=1, layer_offset=69)
    o = oracle_layers(1, h1, h2, [4], act=1, layer_offset=69)
    for phase, T in ((1, 32), (0, 512)):
        x = synth.hidden_f32(41 + T, T, h1)
        ws = R.StageWorkspace(g, T)
        xi = torch.from_numpy(x).cuda()
        xo = torch.empty_like(xi)
        R.sq_stage_forward(g, phase, xi, xo, ws)
        torch.cuda.synchronize()
        rows = [0, T - 1]
        ref, _ = O.stage(o, x[rows].astype(np.float64))
        assert normwise(xo.cpu().numpy()[rows], ref) <= TOL, (phase, T)
