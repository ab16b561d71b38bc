"""Decode GEMV sweep (configs[1]: OPT-13B linear shapes, bits 3/4/8/16, M 1..32).

L2 flushed between timed reps (read a 2 x L2 buffer); CUDA events on the launch
stream; median of reps.  GB/s = algorithmic bytes (codes + meta) / time.
"""
import argparse
import json
import statistics
import sys
import os

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_cluster_zhaowplw25_b200 as sq


def flush_l2(buf):
    # evict L2 by READING a 2 x L2 buffer: a write flush leaves ~126 MB of dirty lines whose
    # write-back then runs inside the timed kernel (measured: ~13 us on every launch)
    if FLUSH == "write":
        buf.zero_()
    else:
        buf.sum()


FLUSH = "read"


def main():
    global FLUSH
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--bits", default="3,4,8,16")
    ap.add_argument("--ms", default="1,8,32")
    ap.add_argument("--shapes", default="5120x5120,20480x5120,5120x20480")
    ap.add_argument("--flush", default="read", choices=["read", "write"])
    a = ap.parse_args()
    FLUSH = a.flush
    dev = torch.device("cuda")
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    flush = torch.zeros(2 * l2 // 4 + 1024, dtype=torch.float32, device=dev)
    out = []
    for shp in a.shapes.split(","):
        n, k = map(int, shp.split("x"))
        wd = torch.empty((n, k), dtype=torch.float16, device=dev)
        synth.device_weight_f16(wd.data_ptr(), 1234, n, k)
        for bits in map(int, a.bits.split(",")):
            q = sq.QLinear.from_fp16(wd if bits != 16 else wd.clone(), bits)
            nbytes = q.nbytes()
            for m in map(int, a.ms.split(",")):
                x = torch.randn(m, k, device=dev).half()
                y = torch.empty(m, n, device=dev, dtype=torch.float16)
                ws = torch.zeros(sq.sq_linear_workspace_bytes(q, m), dtype=torch.uint8, device=dev)
                xs = sq.sq_xsum(x)
                for _ in range(3):
                    sq.sq_linear_decode(q, x, y, 0, xsum=xs, ws=ws)
                ts = []
                for _ in range(a.reps):
                    flush_l2(flush)
                    # keep the GPU busy while the host marshals the launch, so the events
                    # time the kernel and not the host call
                    torch.cuda._sleep(200_000)
                    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
                    e0.record()
                    sq.sq_linear_decode(q, x, y, 0, xsum=xs, ws=ws)
                    e1.record()
                    torch.cuda.synchronize()
                    ts.append(e0.elapsed_time(e1))
                med = statistics.median(ts)
                rec = {"n": n, "k": k, "bits": bits, "m": m, "us": med * 1e3, "GBps": nbytes / med / 1e6}
                out.append(rec)
                print(json.dumps(rec), flush=True)
            del q
        del wd
    return out


if __name__ == "__main__":
    main()
