import sys, os
sys.path.insert(0, "/root/repo")
import numpy as np, torch, synth
import paper_conf_cluster_zhaowplw25_b200 as sq
from oracle import oracle as O
bits, n, k, m = (int(a) for a in sys.argv[1:5])
w = synth.weight_f16(5, n, k)
q = sq.QLinear.from_fp16(torch.from_numpy(w).cuda(), bits)
for src in ("synth", "randn"):
    x = synth.act_f16(7, m, k) if src == "synth" else torch.randn(m, k).half().numpy()
    xt = torch.from_numpy(x).cuda()
    y = torch.empty(m, n, device="cuda", dtype=torch.float16)
    sq.sq_linear_decode(q, xt, y)
    torch.cuda.synchronize()
    ref = O.linear(x, O.QWeight(w, bits))
    yy = y.float().cpu().numpy()
    print(src, bits, n, k, m, "err", np.abs(yy - ref).max() / np.abs(ref).max(), "nan", np.isnan(yy).sum(), "xmax", np.abs(x).max())
