"""Small launches of every hot-path kernel for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck): quantize + pack, the mma.sync decode GEMV (K2, incl. the cross-CTA fix-up), the tcgen05
decode GEMV (K2c) with the cluster/DSMEM split-k and with the cooperative global fix-up, the prefill
GEMM (K3), a configs[0]-shaped stage and a 2-stage virtual pipeline.  No result checks (the parity
tests do that): the sanitizer's report is the output.

  compute-sanitizer --tool memcheck python tools/sanitize_run.py [mma|tc|all]
"""
from __future__ import annotations

import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main(which: str) -> None:
    import torch
    import synth
    import paper_conf_cluster_zhaowplw25_b200 as sq
    from paper_conf_cluster_zhaowplw25_b200 import runtime as R

    torch.cuda.set_device(0)
    # shapes: split panels (few row tiles, long k) and straddling K2 tiles
    for (n, k) in ((256, 4608), (2048, 1536)):
        w = torch.empty((n, k), dtype=torch.float16, device="cuda")
        synth.device_weight_f16(w.data_ptr(), 5, n, k)
        for bits in (3, 4, 8, 16):
            q = sq.QLinear.from_fp16(w, bits)
            for m in (1, 5, 32):
                x = torch.randn(m, k, device="cuda").half()
                y = torch.empty((m, n), dtype=torch.float16, device="cuda")
                sq.sq_linear_decode(q, x, y, 0)
                ya = torch.zeros((m, n), dtype=torch.float32, device="cuda")
                sq.sq_linear_decode(q, x, ya, sq.SQ_EPI_F32_ACCUM)
            if which in ("all", "gemm"):
                x = torch.randn(300, k, device="cuda").half()
                y = torch.empty((300, n), dtype=torch.float16, device="cuda")
                sq.sq_linear_prefill(q, x, y, 0)
            torch.cuda.synchronize()
    if which == "all":
        bits = [3, 4, 8, 16]
        g = R.build_layers(4, 768, 3072, bits)
        for phase, T in ((0, 32), (1, 1), (1, 8)):
            ws = R.StageWorkspace(g, T)
            xi = torch.randn(T, 768, device="cuda")
            xo = torch.empty_like(xi)
            R.sq_stage_forward(g, phase, xi, xo, ws)
        plan = R.Plan(bits, [0, 0, 1, 1], 768, 3072, 3, 2, 2, 16, 2)
        comm = R.Comm.local(2)
        x0 = torch.randn(3, 16, 768, device="cuda")
        out = torch.zeros(3, 3, 768, device="cuda")
        R.sq_pipeline_run(plan, -1, g, comm, x0, out, R.PipelineWorkspace(plan, g, -1))
        comm.destroy()
    torch.cuda.synchronize()
    print("sanitize_run done", which)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "all")
