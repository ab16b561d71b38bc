"""Back-to-back decode GEMV throughput: R distinct copies of one quantized linear (together
> 2 x L2, so every launch streams from HBM) launched in a row on one stream, as consecutive
linears of a decode step are.  One event pair around N launches: per-launch time includes
the launch gaps and ramp/tail of each kernel, but no host time.

  python tools/gemv_rot.py --shapes 5120x5120,36864x9216 --bits 3,4,8,16 --ms 1,8,32
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_cluster_zhaowplw25_b200 as sq


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--bits", default="3,4,8,16")
    ap.add_argument("--ms", default="1,8,32")
    ap.add_argument("--shapes", default="5120x5120,20480x5120,36864x9216")
    ap.add_argument("--n-launch", type=int, default=60)
    ap.add_argument("--min-bytes", type=float, default=400e6)
    ap.add_argument("--graph", action="store_true", help="replay the launches from one CUDA graph (no host time)")
    a = ap.parse_args()
    dev = torch.device("cuda")
    for shp in a.shapes.split(","):
        n, k = map(int, shp.split("x"))
        wd = torch.empty((n, k), dtype=torch.float16, device=dev)
        synth.device_weight_f16(wd.data_ptr(), 1234, n, k)
        for bits in map(int, a.bits.split(",")):
            q0 = sq.QLinear.from_fp16(wd if bits != 16 else wd.clone(), bits)
            R = max(2, int(a.min_bytes // q0.nbytes()) + 1)
            qs = [q0] + [sq.QLinear(bits, n, k, q0.packed.clone(), None if q0.meta is None else q0.meta.clone())
                         for _ in range(R - 1)]
            for m in map(int, a.ms.split(",")):
                x = torch.randn(m, k, device=dev).half()
                y = torch.empty(m, n, device=dev, dtype=torch.float16)
                ws = torch.zeros(sq.sq_linear_workspace_bytes(q0, m), dtype=torch.uint8, device=dev)
                xs = sq.sq_xsum(x)
                for i in range(2 * R):
                    sq.sq_linear_decode(qs[i % R], x, y, 0, xsum=xs, ws=ws)
                torch.cuda.synchronize()
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                if a.graph:
                    g = torch.cuda.CUDAGraph()
                    with torch.cuda.graph(g):
                        for i in range(a.n_launch):
                            sq.sq_linear_decode(qs[i % R], x, y, 0, xsum=xs, ws=ws)
                    g.replay()
                    torch.cuda.synchronize()
                    best = 1e30
                    for _ in range(5):
                        e0.record()
                        g.replay()
                        e1.record()
                        torch.cuda.synchronize()
                        best = min(best, e0.elapsed_time(e1))
                    us = best * 1e3 / a.n_launch
                    del g
                else:
                    torch.cuda._sleep(1_000_000)  # GPU busy while the host enqueues the launches
                    e0.record()
                    for i in range(a.n_launch):
                        sq.sq_linear_decode(qs[i % R], x, y, 0, xsum=xs, ws=ws)
                    e1.record()
                    torch.cuda.synchronize()
                    us = e0.elapsed_time(e1) * 1e3 / a.n_launch
                print(json.dumps({"n": n, "k": k, "bits": bits, "m": m, "copies": R, "us": round(us, 2),
                                  "GBps": round(q0.nbytes() / us / 1e3, 1)}), flush=True)
            del qs, q0
        del wd


if __name__ == "__main__":
    main()
