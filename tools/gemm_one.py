"""Run one prefill GEMM shape a few times and time it (and for ncu)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_cluster_zhaowplw25_b200 as sq
n, k, bits, m = (int(a) for a in (sys.argv[1:5] if len(sys.argv) > 4 else (7168, 7168, 4, 4096)))
wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
synth.device_weight_f16(wd.data_ptr(), 1234, n, k)
q = sq.QLinear.from_fp16(wd, bits)
x = torch.randn(m, k, device="cuda").half()
y = torch.empty(m, n, device="cuda", dtype=torch.float16)
for _ in range(3):
    sq.sq_linear_prefill(q, x, y, 0)
torch.cuda.synchronize()
e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
e0.record()
R = 10
for _ in range(R):
    sq.sq_linear_prefill(q, x, y, 0)
e1.record(); torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / R
print(f"gemm n={n} k={k} bits={bits} m={m}: {ms*1e3:.1f} us  {2*m*n*k/ms/1e9:.1f} TFLOP/s")
