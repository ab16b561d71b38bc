"""smoke(): one small invocation of the whole hot path on cuda:0, checked against the oracle.

a1/a2: quantize + pack bit-exact; a3/a4: prefill + decode linears; a5/a6: a 2-stage
virtual pipeline (prefill 2 x 32 tokens + 3 decode steps) end to end.  Raises on mismatch.
"""
from __future__ import annotations

import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def _nw(y, r):
    y = np.asarray(y, np.float64)
    return float(np.abs(y - r).max() / np.abs(r).max())


def run() -> None:
    import torch
    import synth
    from oracle import oracle as O
    import paper_conf_cluster_zhaowplw25_b200 as sq
    from paper_conf_cluster_zhaowplw25_b200 import runtime as R

    assert torch.cuda.is_available(), "smoke() needs cuda:0"
    torch.cuda.set_device(0)
    # a1 + a2 bit-exact
    w = synth.weight_f16(3, 128, 512)
    for bits in (3, 4, 8):
        codes, s, z = O.quantize_groups(w, bits)
        packed, meta = O.pack(codes, s, z, bits)
        q = sq.QLinear.from_fp16(torch.from_numpy(w).cuda(), bits)
        assert np.array_equal(q.packed.cpu().numpy(), packed), f"pack mismatch bits={bits}"
        assert np.array_equal(q.meta.cpu().numpy().view(np.uint32).reshape(-1), meta.reshape(-1))
        # a3 / a4
        for m, kind in ((3, "decode"), (40, "prefill")):
            x = synth.act_f16(9 + m, m, 512)
            y = torch.empty((m, 128), dtype=torch.float16, device="cuda")
            xt = torch.from_numpy(x).cuda()
            if kind == "decode":
                sq.sq_linear_decode(q, xt, y)
            else:
                sq.sq_linear_prefill(q, xt, y)
            torch.cuda.synchronize()
            err = _nw(y.float().cpu().numpy(), O.linear(x, O.QWeight(w, bits)))
            assert err <= 2e-3, f"{kind} bits={bits} err={err}"
    # a5 + a6: 4 layers, 2 uneven stages, virtual pipeline
    h1, h2, L = 256, 1024, 4
    bits = [3, 16, 4, 8]
    g = R.build_layers(L, h1, h2, bits)
    o = []
    for l in range(L):
        qs = {}
        for name, (n, k) in {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}.items():
            seed = synth.weight_seed(l, name)
            qs[name] = O.QWeight(synth.weight_f16(seed, n, k), bits[l], bias=synth.bias_f16(seed, n))
        o.append(O.Layer(bits[l], 0, qs["qkv"], qs["o"], qs["fc1"], qs["fc2"]))
    B, s, n_dec = 2, 32, 3
    plan = R.Plan(bits, [0, 1, 1, 1], h1, h2, B, 1, 2, s, n_dec)
    x0 = synth.hidden_f32(1, B * s, h1).reshape(B, s, h1)
    comm = R.Comm.local(2)
    ws = R.PipelineWorkspace(plan, g, -1)
    out = torch.zeros((B, 1 + n_dec, h1), dtype=torch.float32, device="cuda")
    st = R.sq_pipeline_run(plan, -1, g, comm, torch.from_numpy(x0).cuda(), out, ws)
    comm.destroy()
    ref = O.pipeline(o, x0, n_dec)
    err = _nw(out.cpu().numpy(), ref)
    assert err <= 2e-3, f"pipeline err={err}"
    print(f"smoke ok: pipeline normwise err {err:.2e}, {st['gpu_launches']} kernel launches")


if __name__ == "__main__":
    run()
