"""Per-CTA timeline of one tcgen05 decode launch (debug build, SQ_TC_DEBUG=1): CTA start, fix-up
start, end (globaltimer, us from the first CTA start), and CTA 0's ramp (clock64: first weight
landed, first dequant done, first MMA issued, relative to the CTA's start).
  SQ_PDL=0 python tools/trace_cta.py n k bits m"""
import os, sys, ctypes
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["SQ_GEMV_PATH"] = "tc"
import numpy as np, torch, synth
import paper_conf_cluster_zhaowplw25_b200 as sq
n, k, bits, m = (int(a) for a in sys.argv[1:5])
wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
synth.device_weight_f16(wd.data_ptr(), 1234, n, k)
q = sq.QLinear.from_fp16(wd, bits)
x = torch.randn(m, k, device="cuda").half()
y = torch.empty(m, n, device="cuda", dtype=torch.float16)
ws = torch.zeros(sq.sq_linear_workspace_bytes(q, m), dtype=torch.uint8, device="cuda")
tr = torch.zeros(16 * 256, dtype=torch.int64, device="cuda")
sq.lib().sq_debug_trace.argtypes = [ctypes.c_void_p]
for _ in range(3):
    sq.sq_linear_decode(q, x, y, 0, ws=ws)
torch.cuda.synchronize()
sq.lib().sq_debug_trace(tr.data_ptr())
sq.sq_linear_decode(q, x, y, 0, ws=ws)
torch.cuda.synchronize()
t = tr.view(16, 256).cpu().numpy().astype(np.int64)
ns = int((t[14] > 0).sum())
g0 = t[14, :ns].min()
st, fx, en = (t[14, :ns] - g0) / 1e3, (t[11, :ns] - g0) / 1e3, (t[15, :ns] - g0) / 1e3
print(f"CTAs {ns}: start max {st.max():.2f} us; fixup start min/med/max {fx.min():.2f}/{np.median(fx):.2f}/{fx.max():.2f}; "
      f"end min/med/max {en.min():.2f}/{np.median(en):.2f}/{en.max():.2f} us")
c0 = t[13, 0]
ghz = 1.9
ev = {"producer past pdl_wait": t[7, 0], "first W landed (dq)": t[1, 0], "first dequant done": t[2, 0],
      "x(0) landed (MMA)": t[6, 0], "MMA ready unit 0": t[3, 0], "first MMA issued": t[4, 0],
      "x(1) landed": t[6, 1], "x(2) landed": t[6, 2]}
print("CTA0 ramp (us from CTA start):", {k: round((v - c0) / ghz / 1e3, 2) for k, v in ev.items() if v})
print("CTA0 pre-issue done per unit (us):", [round((t[0, i] - c0) / ghz / 1e3, 2) for i in range(12) if t[0, i]])
nu = int((t[4] > 0).sum())
if nu > 2:
    print(f"CTA0 units traced {nu}: MMA issue rate {(t[4, nu - 1] - t[4, 1]) / max(nu - 2, 1):.0f} cycles/unit; "
          f"last MMA issued at {(t[4, nu - 1] - c0) / ghz / 1e3:.2f} us")
ac = (t[9, :ns] - g0) / 1e3
if (t[9, :ns] > 0).all():
    print(f"accumulators complete min/med/max {ac.min():.2f}/{np.median(ac):.2f}/{ac.max():.2f} us")
if (t[10, :ns] > 0).all():
    cs = (t[10, :ns] - g0) / 1e3
    print(f"cluster partials in place min/med/max {cs.min():.2f}/{np.median(cs):.2f}/{cs.max():.2f} us")
