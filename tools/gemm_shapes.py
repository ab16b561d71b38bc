"""Prefill GEMM (K3) on OPT-66B shapes at M = 4096 tokens with the stage's epilogues (qkv fp16, o / fc2
fp32 residual, fc1 ReLU), bits 3/4/8/16: median of 5 event-timed launches after 2 warm-up; TFLOP/s
and fraction of the measured sustained bf16 peak.  Prints one JSON line per point."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import synth  # noqa: E402
import paper_conf_cluster_zhaowplw25_b200 as sq  # noqa: E402

pk = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json"))) \
    if os.path.exists("MEASURED_PEAKS.json") else {}
h1, h2 = int(os.environ.get("H1", 9216)), int(os.environ.get("H2", 36864))
M = int(os.environ.get("M", 4096))
x = torch.empty((M, h2), dtype=torch.float16, device="cuda")
synth.device_fill_f16(x.data_ptr(), 9, 0, x.numel(), 1.0, False)
LIN = os.environ.get("LIN", "qkv,o,fc1,fc2").split(",")
EPI = os.environ.get("EPI")
for name, (n, k), epi in (("qkv", (3 * h1, h1), 0), ("o", (h1, h1), 3), ("fc1", (h2, h1), 1), ("fc2", (h1, h2), 3)):
    if name not in LIN:
        continue
    epi = int(EPI) if EPI is not None else epi
    wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
    synth.device_weight_f16(wd.data_ptr(), synth.weight_seed(0, name), n, k)
    xk = x[:, :k].contiguous()
    y = torch.zeros((M, n), dtype=torch.float32 if epi == 3 else torch.float16, device="cuda")
    for bits in [int(b) for b in os.environ.get("BITS", "3,4,8,16").split(",")]:
        q = sq.QLinear.from_fp16(wd, bits)
        for _ in range(2):
            sq.sq_linear_prefill(q, xk, y, epi)
        ts = []
        for _ in range(5):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            sq.sq_linear_prefill(q, xk, y, epi)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        ms = statistics.median(ts)
        tf = 2.0 * M * n * k / (ms / 1e3) / 1e12
        print(json.dumps({"linear": name, "n": n, "k": k, "bits": bits, "epi": epi, "m": M, "us": round(ms * 1e3, 1),
                          "TFLOPs": round(tf, 1)}), flush=True)
        del q
    del wd, xk, y
    torch.cuda.empty_cache()
