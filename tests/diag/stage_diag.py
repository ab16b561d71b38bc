"""Where does the stage error come from?  One OPT-13B layer, GPU stage vs oracle, plus
teacher-forced per-step errors (each GPU step fed the GPU's own previous output)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))  # repo root (tests/diag/..)
import numpy as np, torch, synth
from oracle import oracle as O
import paper_conf_cluster_zhaowplw25_b200 as sq
from paper_conf_cluster_zhaowplw25_b200 import runtime as R
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))  # tests/
from test_gpu_stage import oracle_layers

def nw(y, r):
    return float(np.abs(np.asarray(y, np.float64) - r).max() / np.abs(r).max())

h1, h2 = 5120, 20480
bits = int(sys.argv[1]) if len(sys.argv) > 1 else 3
g = R.build_layers(1, h1, h2, [bits], layer_offset=7)
o = oracle_layers(1, h1, h2, [bits], layer_offset=7)
L = o[0]
for phase, T in ((1, 32), (0, 512)):
    x = synth.hidden_f32(17 + T, T, h1)
    rows = [0, T // 2, T - 1]
    ws = R.StageWorkspace(g, T)
    xi = torch.from_numpy(x).cuda(); xo = torch.empty_like(xi)
    qkv = torch.empty((T, 3 * h1), dtype=torch.float16, device="cuda")
    R.sq_stage_forward(g, phase, xi, xo, ws, qkv_dbg=qkv)
    torch.cuda.synchronize()
    ref, ref_qkv = O.stage(o, x[rows].astype(np.float64), want_qkv=True)
    print("phase", phase, "stage out", nw(xo.cpu().numpy()[rows], ref), "qkv", nw(qkv.float().cpu().numpy()[rows], ref_qkv))
    # oracle with fp16-rounded activations (what W.A16 computes)
    xr = x[rows].astype(np.float64)
    a = O.layernorm(xr).astype(np.float16)
    q = O.linear(a, L.qkv); v = q[:, 2 * h1:].astype(np.float16)
    hres = xr + O.linear(v, L.o)
    a2 = O.layernorm(hres).astype(np.float16)
    u = np.maximum(O.linear(a2, L.fc1), 0).astype(np.float16)
    out16 = hres + O.linear(u, L.fc2)
    print("   oracle-with-fp16-activations vs oracle:", nw(out16, ref), " GPU vs that:", nw(xo.cpu().numpy()[rows], out16))
