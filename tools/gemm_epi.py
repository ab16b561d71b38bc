"""Prefill GEMM time per epilogue (F16 vs fp32 residual accumulate) on OPT-66B o / fc2 shapes."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_cluster_zhaowplw25_b200 as sq
for (n, k) in ((9216, 9216), (9216, 36864), (36864, 9216)):
    wd = torch.empty((n, k), dtype=torch.float16, device="cuda"); synth.device_weight_f16(wd.data_ptr(), 5, n, k)
    for bits in (4, 16):
        q = sq.QLinear.from_fp16(wd if bits != 16 else wd.clone(), bits)
        m = 4096
        x = torch.randn(m, k, device="cuda").half()
        for epi in (0, 3):
            y = torch.zeros(m, n, device="cuda", dtype=torch.float32 if epi == 3 else torch.float16)
            sq.sq_linear_prefill(q, x, y, epi); torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            for i in range(5): sq.sq_linear_prefill(q, x, y, epi)
            e1.record(); torch.cuda.synchronize()
            us = e0.elapsed_time(e1) * 1e3 / 5
            print(json.dumps(dict(n=n, k=k, bits=bits, epi=epi, us=round(us, 1), tflops=round(2 * m * n * k / us / 1e6, 1))), flush=True)
