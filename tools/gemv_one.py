"""Run one decode GEMV shape a few times (for ncu)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_cluster_zhaowplw25_b200 as sq
n, k, bits, m = (int(a) for a in (sys.argv[1:5] if len(sys.argv) > 4 else (5120, 5120, 4, 1)))
wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
synth.device_weight_f16(wd.data_ptr(), 1234, n, k)
q = sq.QLinear.from_fp16(wd, bits)
x = torch.randn(m, k, device="cuda").half()
y = torch.empty(m, n, device="cuda", dtype=torch.float16)
ws = torch.zeros(sq.sq_linear_workspace_bytes(q, m), dtype=torch.uint8, device="cuda")
xs = sq.sq_xsum(x)
for _ in range(5):
    sq.sq_linear_decode(q, x, y, 0, xsum=xs, ws=ws)
torch.cuda.synchronize()
