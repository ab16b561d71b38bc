"""Error budget of the GPU linears vs the fp64 oracle (normwise), per bits / phase / m."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))  # repo root (tests/diag/..)
import numpy as np, torch, synth
from oracle import oracle as O
import paper_conf_cluster_zhaowplw25_b200 as sq

def nw(y, r):
    return float(np.abs(y - r).max() / np.abs(r).max())

for (n, k) in ((512, 5120), (512, 20480)):
    for bits in (3, 4, 8, 16):
        w = synth.weight_f16(77, n, k)
        qo = O.QWeight(w, bits)
        qg = sq.QLinear.from_fp16(torch.from_numpy(w).cuda(), bits)
        res = {}
        for m in (1, 8, 32, 256):
            x = synth.act_f16(5 + m, m, k)
            ref = O.linear(x, qo)
            xt = torch.from_numpy(x).cuda()
            if m <= 32:
                y = torch.empty((m, n), dtype=torch.float32, device="cuda").zero_()
                sq.sq_linear_decode(qg, xt, y, sq.SQ_EPI_F32_ACCUM)
                res[f"dec{m}"] = nw(y.cpu().numpy(), ref)
            y = torch.zeros((m, n), dtype=torch.float32, device="cuda")
            sq.sq_linear_prefill(qg, xt, y, sq.SQ_EPI_F32_ACCUM)
            res[f"pre{m}"] = nw(y.cpu().numpy(), ref)
        print(n, k, bits, {a: f"{b:.2e}" for a, b in res.items()}, flush=True)
