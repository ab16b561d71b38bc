"""Decode GEMV on the TP shard shapes of OPT-66B (h1 9216, h2 36864): qkv [3h1/T, h1], o [h1, h1/T],
fc1 [h2/T, h1], fc2 [h1, h2/T] for T = 1, 2, 4, 8; bits 3/4/8; m = 1, 8, 32.  40 back-to-back launches
over > 2 x L2 of weight copies in one CUDA graph, best of 3 (as bench.gemv_sweep).  Run once per
SQ_GEMV_PATH (t = tcgen05 K2c, m = mma.sync K2, unset = the library's choice); prints JSON lines."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
import paper_conf_cluster_zhaowplw25_b200 as sq  # noqa: E402


def main():
    h1, h2 = 9216, 36864
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    tps = [int(t) for t in os.environ.get("TPS", "1,2,4,8").split(",")]
    for T in tps:
        for name, (n, k) in {"qkv": (3 * h1 // T, h1), "o": (h1, h1 // T), "fc1": (h2 // T, h1),
                             "fc2": (h1, h2 // T)}.items():
            wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
            synth.device_weight_f16(wd.data_ptr(), 77, n, k)
            for bits in (3, 4, 8):
                q0 = sq.QLinear.from_fp16(wd, bits)
                R = max(2, int(2 * l2 // q0.nbytes()) + 2)
                qs = [q0] + [sq.QLinear(bits, n, k, q0.packed.clone(), q0.meta.clone()) for _ in range(R - 1)]
                for m in (1, 8, 32):
                    x = torch.randn(m, k, device="cuda").half()
                    y = torch.empty(m, n, device="cuda", dtype=torch.float16)
                    ws = torch.zeros(sq.sq_linear_workspace_bytes(q0, m), dtype=torch.uint8, device="cuda")
                    xs = sq.sq_xsum(x)
                    for i in range(R):
                        sq.sq_linear_decode(qs[i], x, y, 0, xsum=xs, ws=ws)
                    torch.cuda.synchronize()
                    g = torch.cuda.CUDAGraph()
                    with torch.cuda.graph(g):
                        for i in range(40):
                            sq.sq_linear_decode(qs[i % R], x, y, 0, xsum=xs, ws=ws)
                    g.replay()
                    torch.cuda.synchronize()
                    best = 1e9
                    for _ in range(3):
                        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                        e0.record()
                        g.replay()
                        e1.record()
                        torch.cuda.synchronize()
                        best = min(best, e0.elapsed_time(e1))
                    us = best * 1e3 / 40
                    print(json.dumps({"path": os.environ.get("SQ_GEMV_PATH", "auto"), "T": T, "lin": name, "n": n,
                                      "k": k, "bits": bits, "m": m, "us": round(us, 2),
                                      "GBps": round(q0.nbytes() / us / 1e3, 1)}), flush=True)
                    del g
                del qs, q0
            del wd
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
