"""Run the attention kernels once at OPT-66B shapes (for ncu): a decode micro-batch of 32 sequences at
position 600 and an 8 x 512-token prefill micro-batch (72 heads x 128)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_cluster_zhaowplw25_b200 as sq
H, dh, B, L = 72, 128, 32, 640
h1 = H * dh
kc = torch.empty((B, L, h1), dtype=torch.float16, device="cuda")
vc = torch.empty_like(kc)
synth.device_fill_f16(kc.data_ptr(), 1, 0, kc.numel(), 0.5, False)
synth.device_fill_f16(vc.data_ptr(), 2, 0, vc.numel(), 1.0, False)
q = torch.randn(B, 3 * h1, device="cuda").half()
o = torch.empty(B, h1, device="cuda", dtype=torch.float16)
qp = torch.randn(8 * 512, 3 * h1, device="cuda").half()
op = torch.empty(8 * 512, h1, device="cuda", dtype=torch.float16)
for _ in range(3):
    sq.sq_attention(q, B, 1, 600, 0, H, kc, vc, o)
    sq.sq_attention(qp, 8, 512, 0, 0, H, kc, vc, op)
torch.cuda.synchronize()
print("ok")
