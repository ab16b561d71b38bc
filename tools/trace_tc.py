"""Timeline of the tcgen05 decode GEMV on CTA 0 (clock64 per unit): producer W issue (0),
dequant W-ready (1) / slot-ready (5) / done (2), MMA A-ready (3) / issued (4)."""
import sys, os, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["SQ_GEMV_PATH"] = "tc"
import torch, synth
import paper_conf_cluster_zhaowplw25_b200 as sq
n, k, bits, m = (int(a) for a in (sys.argv[1:5] if len(sys.argv) > 4 else (20480, 5120, 4, 32)))
wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
synth.device_weight_f16(wd.data_ptr(), 1234, n, k)
q = sq.QLinear.from_fp16(wd, bits)
x = torch.randn(m, k, device="cuda").half()
y = torch.empty(m, n, device="cuda", dtype=torch.float16)
ws = torch.zeros(sq.sq_linear_workspace_bytes(q, m), dtype=torch.uint8, device="cuda")
tr = torch.zeros(14 * 256, dtype=torch.int64, device="cuda")
sq.lib().sq_debug_trace.argtypes = [ctypes.c_void_p]
for _ in range(3):
    sq.sq_linear_decode(q, x, y, 0, ws=ws)
sq.lib().sq_debug_trace(tr.data_ptr())
sq.sq_linear_decode(q, x, y, 0, ws=ws)
torch.cuda.synchronize()
t = tr.view(14, 256).cpu().numpy().astype("int64")
t0 = t[0, 0]
U = (n // 128) * (k // 128); per = U // 148
print("units on CTA0:", per)
print(" i  Wwait    Wtma  metatma   X0tma   X1tma dq_done mma_Ardy  x0rdy  mma0done  x1rdy mma1done mma_end")
for i in range(min(per, 48)):
    print(f"{i:2d} " + " ".join(f"{(t[e, i] - t0) if t[e, i] else -1:8d}" for e in (0, 6, 7, 8, 9, 2, 3, 10, 11, 12, 13, 4)))
