"""Run by test_gpu_linear.test_prefill_cta_pair_bitwise in a subprocess (the tile choice SQ_GEMM_CG is
read once per process): prefill outputs for fixed seeded cases, saved to the .npz named by argv[1]."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_cluster_zhaowplw25_b200 as sq


def main(path):
    out = {}
    for bits in (3, 4, 8, 16):
        for (n, k, m, epi) in ((512, 1280, 300, 0), (1024, 768, 513, 3), (256, 384, 77, 1)):
            w = synth.weight_f16(1200 + n + bits, n, k)
            b = synth.bias_f16(1201 + n, n)
            q = sq.QLinear.from_fp16(torch.from_numpy(w).cuda(), bits, torch.from_numpy(b).cuda())
            x = torch.from_numpy(synth.act_f16(1202 + m, m, k)).cuda()
            if epi == 3:
                y = torch.from_numpy(synth.hidden_f32(1203, m, n)).cuda()
            else:
                y = torch.empty((m, n), dtype=torch.float16, device="cuda")
            sq.sq_linear_prefill(q, x, y, epi)
            torch.cuda.synchronize()
            out[f"b{bits}_n{n}_k{k}_m{m}_e{epi}"] = y.cpu().numpy()
    np.savez(path, **out)


if __name__ == "__main__":
    main(sys.argv[1])
