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
tr = torch.zeros(16 * 256, dtype=torch.int64, device="cuda")
sq.lib().sq_debug_trace.argtypes = [ctypes.c_void_p]
for _ in range(3):
    sq.sq_linear_decode(q, x, y, 0, ws=ws)
sq.lib().sq_debug_trace(tr.data_ptr())
sq.sq_linear_decode(q, x, y, 0, ws=ws)
torch.cuda.synchronize()
t = tr.view(16, 256).cpu().numpy().astype("int64")
t0 = t[0, 0]
U = (n // 128) * (k // 128); per = U // 148
print("units on CTA0:", per)
cols = [("prodW", 0), ("prodIss", 8), ("dqW", 1), ("dqSlot", 5), ("dqCalc", 12), ("dqDone", 2), ("mmaRdy", 3), ("mmaIss", 4)]
print(" i " + " ".join(f"{c:>8s}" for c, _ in cols))
for i in range(min(per, 64)):
    print(f"{i:2d} " + " ".join(f"{(t[e, i] - t0) if t[e, i] else -1:8d}" for _, e in cols))
ns = min(148, int((t[14] > 0).sum()))
g0 = t[14, :ns].min()
st, en = (t[14, :ns] - g0) / 1e3, (t[15, :ns] - g0) / 1e3
print(f"CTA start us: min {st.min():.2f} max {st.max():.2f}; end us: min {en.min():.2f} med {sorted(en)[ns // 2]:.2f} max {en.max():.2f}")
print("slowest CTAs:", [(int(c), round(float(en[c]), 2)) for c in en.argsort()[-8:]])
print("ends:", " ".join(f"{e:.1f}" for e in en[:40]))
fx = (t[11, :ns] - g0) / 1e3
land = (t[10, :ns] - g0) / 1e3
red = [c for c in range(ns) if t[10, c] > t[14, c]]
print("reducers:", len(red), "fixup start->first tile landed->end us:", [(round(float(fx[c]), 1), round(float(land[c]), 1), round(float(en[c]), 1)) for c in red[:6]])
print("non-reducers fixup start:", [round(float(fx[c]), 1) for c in range(ns) if c not in red][:8])
done = (t[9, :ns] - g0) / 1e3
sync = (t[13, :ns] - g0) / 1e3
print("reducers compute-done / after-sync:", [(round(float(done[c]), 1), round(float(sync[c]), 1)) for c in red[:6]])
l1 = (t[6, :ns] - g0) / 1e3
l3 = (t[7, :ns] - g0) / 1e3
print("reducers tile1/tile3 landed:", [(round(float(l1[c]), 1), round(float(l3[c]), 1)) for c in red[:6]])
