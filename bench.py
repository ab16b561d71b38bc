#!/usr/bin/env python
"""bench.py — SplitQuant hot path on B200 (BASELINE.json metric).

Metric: "decode dequant-GEMV GB/s vs HBM peak; pipeline tokens/s at 1/2/4/8 B200".
value = pipeline output tokens/s of the whole job on configs[3] (OPT-66B-shaped,
64 layers, mixed bits 16 x {3,4,8,16}, prompt 512, 128 decode steps, prefill
micro-batch eta = 8, decode micro-batch xi = 32), weak scaling B = 32 * N
(SURVEY.md 8(d) D-4).  A step = one full generation run (prefill + decode) through
sq_pipeline_run, inputs resident in HBM.  The decode dequant-GEMV GB/s (configs[1]
OPT-13B shapes) is reported beside it in "decode_gemv" and as the roofline when it
is the dominant kernel.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
  torchrun --nproc-per-node N bench.py --gpus N ...   (one rank per GPU)

--impl reference times the CPU oracle (oracle/, the only other place this file
executes it) on a bounded sample of the same workload on the host cores.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "decode dequant-GEMV GB/s vs HBM peak; pipeline tokens/s at 1/2/4/8 B200"

WORKLOADS = {
    # BASELINE.json configs[3]
    "opt66b": dict(name="configs[3] OPT-66B-shaped 64 layers, uneven mixed-bit pipeline, prompt 512 + 128 decode tokens",
                   h1=9216, h2=36864, L=64, act=0, eta=8, xi=32, s=512, n_dec=128, b_per_gpu=32, balanced=True),
    # BASELINE.json configs[4]: BLOOM-176B-shaped (d = 14336, fused QKV, GeLU), 70 layers, INT3/INT4 50/50
    "bloom176b": dict(name="configs[4] BLOOM-176B-shaped 70 layers, INT3/INT4-mixed, uneven pipeline with micro-batching",
                      h1=14336, h2=57344, L=70, act=1, eta=8, xi=32, s=512, n_dec=128, b_per_gpu=32, balanced=True,
                      choices=(3, 4)),
    # BASELINE.json configs[0] (small; for quick runs)
    "opt125m": dict(name="configs[0] OPT-125m-shaped 12 layers, bits {3,4,8,16}, prefill 1x32 + 8 decode steps",
                    h1=768, h2=3072, L=12, act=0, eta=1, xi=1, s=32, n_dec=8, b_per_gpu=1, balanced=False),
}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            d = json.load(f)
        return {"hbm_gbs": float(d["hbm_gbs"]), "tflops": float(d["bf16_tflops"]),
                "tflops_sustained": float(d.get("bf16_tflops_sustained", d["bf16_tflops"])), "src": "measured"}
    except Exception:
        return {"hbm_gbs": 6650.0, "tflops": 1590.0, "tflops_sustained": 1400.0, "src": "fallback"}


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


# ------------------------------------------------------------------ clocks sampler
class ClockSampler:
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu, self.proc, self.lines = gpu, None, []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                                          "-lms", "200", "-i", str(self.gpu)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sms, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            p = [x.strip() for x in ln.split(",")]
            if len(p) < 9:
                continue
            try:
                sms.append(float(p[1]))
                mx = float(p[2])
            except ValueError:
                continue
            for nm, v in zip(names, p[5:9]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sms) if sms else None, "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sms)}


# ------------------------------------------------------------------ CPU oracle sample
def cpu_model() -> str:
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:
        pass
    import platform
    return platform.processor() or "unknown"


def oracle_layer_seconds(wl: dict, bits: int, tokens: int, row_frac: int) -> float:
    """Bounded oracle sample: oq_linear (fp64, plain loops) on the first n/row_frac rows of each of the
    4 linears of one layer of the workload at `bits`, `tokens` tokens.  Seconds of host time."""
    import numpy as np
    import synth
    from oracle import oracle as O
    h1, h2 = wl["h1"], wl["h2"]
    dims = {"qkv": (3 * h1, h1), "o": (h1, h1), "fc1": (h2, h1), "fc2": (h1, h2)}
    qws = {}
    for name, (n, k) in dims.items():
        rows = np.arange(n // row_frac)
        qws[name] = O.QWeight(synth.weight_f16(synth.weight_seed(0, name), n, k, rows=rows), bits)
    x1 = synth.act_f16(5, tokens, h1)
    x2 = synth.act_f16(6, tokens, h2)
    t0 = time.perf_counter()
    for name, (n, k) in dims.items():
        O.linear(x1 if k == h1 else x2, qws[name])
    return time.perf_counter() - t0


def workload_bits(wl: dict) -> list[int]:
    import synth
    return [int(b) for b in synth.bits_plan(2, wl["L"], choices=wl.get("choices", (3, 4, 8, 16)),
                                            balanced=wl["balanced"])]


def oracle_tokens_per_s(wl: dict, B: int, per_bit_s: dict, tokens: int, row_frac: int) -> float:
    """Extrapolate per-bit layer samples to the workload: sum over its layers (their own bits) of the
    per-token layer time x the token rows the run processes (B*s prefill + B*n_dec decode)."""
    bits = workload_bits(wl)
    per_token = sum(per_bit_s[b] * row_frac / tokens for b in bits)
    total = per_token * (B * wl["s"] + B * wl["n_dec"])
    return B * (1 + wl["n_dec"]) / total


def cpu_baseline(wl: dict, B: int, tokens: int, row_frac: int, one_thread: bool = True) -> dict:
    """The oracle as it stands, on this host: per bit width present in the workload, at all cores and
    (optionally) at one thread; value = the workload's tokens/s at all cores."""
    from oracle import oracle as O
    ncores = len(os.sched_getaffinity(0))
    present = sorted(set(workload_bits(wl)))
    allc, one = {}, {}
    O.set_threads(ncores)
    for b in present:
        allc[b] = oracle_layer_seconds(wl, b, tokens, row_frac)
    if one_thread:
        O.set_threads(1)
        for b in present:
            one[b] = oracle_layer_seconds(wl, b, tokens, row_frac)
        O.set_threads(ncores)
    out = {"value": oracle_tokens_per_s(wl, B, allc, tokens, row_frac), "unit": "tokens/s", "cores": ncores,
           "kind": "oracle", "cpu": cpu_model(),
           "sample": (f"oq_linear fp64 on the first 1/{row_frac} of the rows of the 4 linears of one layer per bit width "
                      f"{present}, {tokens} tokens; extrapolated over the workload's {wl['L']} layers (their own bits) "
                      f"x (B*s + B*n_dec) token rows"),
           "layer_s_all_cores": {str(b): round(allc[b], 4) for b in present}}
    if one_thread:
        out["value_1_thread"] = oracle_tokens_per_s(wl, B, one, tokens, row_frac)
        out["layer_s_1_thread"] = {str(b): round(one[b], 4) for b in present}
    return out


def run_reference(args, wl):
    rank, world, _ = dist_env()
    if rank != 0:
        return
    from oracle import oracle as O
    ncores = len(os.sched_getaffinity(0))
    O.set_threads(ncores)
    B = wl["b_per_gpu"] * max(1, args.gpus)
    tokens, frac = args.cpu_tokens, args.cpu_row_frac
    present = sorted(set(workload_bits(wl)))

    def one_step():
        t0 = time.perf_counter()
        per = {b: oracle_layer_seconds(wl, b, tokens, frac) for b in present}
        return time.perf_counter() - t0, oracle_tokens_per_s(wl, B, per, tokens, frac)

    for _ in range(args.warmup):
        one_step()
    vals, ts = [], []
    for _ in range(args.steps):
        dt, v = one_step()
        ts.append(dt)
        vals.append(v)
    v = statistics.median(vals)
    sample = (f"per step: oq_linear fp64 on the first 1/{frac} of the rows of the 4 linears of one layer per bit "
              f"width {present}, {tokens} tokens, extrapolated over the workload's {wl['L']} layers x "
              f"(B*s + B*n_dec) token rows")
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "tokens/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * statistics.median(ts),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": wl["name"], "B": B},
            "cpu_baseline": {"value": v, "unit": "tokens/s", "cores": ncores, "kind": "oracle", "sample": sample,
                             "cpu": cpu_model()},
            "e2e": {"value": v, "unit": "tokens/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ decode GEMV sweep (configs[1])
def gemv_sweep(n_launch=40, ms=(1, 2, 4, 8, 16, 32), bit_list=(3, 4, 8, 16)):
    """configs[1]: OPT-13B linear shapes, bits 3/4/8 (+ fp16 as the reference row), micro-batch 1..32.  Each point is a decode
    step's worth of back-to-back linears: n_launch launches cycling over R distinct copies of the
    quantized weight (R copies > 2 x L2, so every launch streams its weights from HBM), captured in
    one CUDA graph (launch gaps hidden by PDL, as in the stage forward); best of 3 replays.
    GB/s = algorithmic bytes (codes + scales/zeros) per launch / time per launch."""
    import torch
    import synth
    import paper_conf_cluster_zhaowplw25_b200 as sq
    pk = peaks()
    dev = torch.device("cuda")
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    out = []
    for (n, k) in ((5120, 5120), (20480, 5120), (5120, 20480)):
        wd = torch.empty((n, k), dtype=torch.float16, device=dev)
        synth.device_weight_f16(wd.data_ptr(), 4242, n, k)
        for bits in bit_list:
            q0 = sq.QLinear.from_fp16(wd, bits)
            R = max(2, int(2 * l2 // q0.nbytes()) + 2)
            qs = [q0] + [sq.QLinear(bits, n, k, q0.packed.clone(), None if q0.meta is None else q0.meta.clone())
                         for _ in range(R - 1)]
            for m in ms:
                x = torch.randn(m, k, device=dev).half()
                y = torch.empty(m, n, device=dev, dtype=torch.float16)
                ws = torch.zeros(sq.sq_linear_workspace_bytes(q0, m), dtype=torch.uint8, device=dev)
                xs = sq.sq_xsum(x)
                for i in range(R):
                    sq.sq_linear_decode(qs[i], x, y, 0, xsum=xs, ws=ws)
                torch.cuda.synchronize()
                g = torch.cuda.CUDAGraph()
                with torch.cuda.graph(g):
                    for i in range(n_launch):
                        sq.sq_linear_decode(qs[i % R], x, y, 0, xsum=xs, ws=ws)
                g.replay()
                torch.cuda.synchronize()
                best = float("inf")
                for _ in range(3):
                    e0 = torch.cuda.Event(enable_timing=True)
                    e1 = torch.cuda.Event(enable_timing=True)
                    e0.record()
                    g.replay()
                    e1.record()
                    torch.cuda.synchronize()
                    best = min(best, e0.elapsed_time(e1))
                us = best * 1e3 / n_launch
                gbs = q0.nbytes() / us / 1e3
                out.append({"n": n, "k": k, "bits": bits, "m": m, "us": round(us, 2), "GBps": round(gbs, 1),
                            "frac": round(gbs / pk["hbm_gbs"], 3)})
                del g
            del qs, q0
        del wd
    return out


def w8a8_decode_sweep(n_launch=40, ms=(1, 32)):
    """f4 W8A8 at configs[1] shapes: per launch the per-token activation quantization + the kind::i8
    linear (split-k + integer reduce for narrow grids), R weight copies > 2 x L2, one CUDA graph of
    n_launch launches, best of 3.  GB/s = weight bytes (n k codes + 2 n scales) / time per launch."""
    import torch
    import synth
    import paper_conf_cluster_zhaowplw25_b200 as sq
    pk = peaks()
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    out = []
    for (n, k) in ((5120, 5120), (20480, 5120), (5120, 20480)):
        wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
        synth.device_weight_f16(wd.data_ptr(), 4243, n, k)
        w0 = sq.W8Linear.from_fp16(wd)
        nbytes = n * k + 2 * n
        R = max(2, int(2 * l2 // nbytes) + 2)
        ws = [w0] + [sq.W8Linear(w0.codes.clone(), w0.scales.clone()) for _ in range(R - 1)]
        for m in ms:
            x = torch.randn(m, k, device="cuda").half()
            y = torch.empty(m, n, device="cuda", dtype=torch.float16)
            wsb = torch.empty(max(1, int(sq.lib().sq_linear_w8a8_workspace_bytes(n, k, m))), dtype=torch.uint8, device="cuda")
            for i in range(R):
                xq, sx = sq.sq_quantize_act8(x)
                sq.sq_linear_w8a8(ws[i], xq, sx, y, 0, ws=wsb)
            torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                for i in range(n_launch):
                    xq, sx = sq.sq_quantize_act8(x)
                    sq.sq_linear_w8a8(ws[i % R], xq, sx, y, 0, ws=wsb)
            g.replay()
            torch.cuda.synchronize()
            best = float("inf")
            for _ in range(3):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                g.replay()
                e1.record()
                torch.cuda.synchronize()
                best = min(best, e0.elapsed_time(e1))
            us = best * 1e3 / n_launch
            gbs = nbytes / us / 1e3
            out.append({"n": n, "k": k, "bits": "w8a8", "m": m, "us": round(us, 2), "GBps": round(gbs, 1),
                        "frac": round(gbs / pk["hbm_gbs"], 3)})
            del g
        del ws, w0, wd
    return out


# ------------------------------------------------------------------ our arm
def run_ours(args, wl):
    import torch
    import synth
    import paper_conf_cluster_zhaowplw25_b200 as sq
    from paper_conf_cluster_zhaowplw25_b200 import runtime as R
    from paper_conf_cluster_zhaowplw25_b200 import plan as PL

    rank, world, local = dist_env()
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}; run `python bench.py --gpus N` "
                         f"(it launches the N ranks itself) or torchrun --nproc-per-node N")
    P = world
    torch.cuda.set_device(local)
    dist = None
    selfcheck = None
    if P > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo")
        # the NCCL pipeline must equal the single-process virtual pipeline bitwise before anything is timed
        from paper_conf_cluster_zhaowplw25_b200.selfcheck import pipeline_bitwise_check
        selfcheck = pipeline_bitwise_check(rank, P, dist)
        if not selfcheck["pipeline_bitwise_ok"]:
            if rank == 0:
                print(json.dumps({"error": "NCCL pipeline differs from the virtual pipeline", **selfcheck}), flush=True)
            raise SystemExit(1)
    pk = peaks()

    B = wl["b_per_gpu"] * P
    L, h1, h2 = wl["L"], wl["h1"], wl["h2"]
    bits = workload_bits(wl)
    costs = PL.phase_costs(bits, h1, h2, B, wl["eta"], wl["xi"], wl["s"], wl["n_dec"], pk["hbm_gbs"],
                           pk["tflops_sustained"])
    sol = PL.partition_layers(costs, P)
    plan = R.Plan(bits, sol, h1, h2, B, wl["eta"], wl["xi"], wl["s"], wl["n_dec"])
    R.sq_plan_check(plan)
    mine = plan.layers_of(rank) if P > 1 else list(range(L))
    layers = R.build_layers(len(mine), h1, h2, [bits[l] for l in mine], act=wl["act"], layer_offset=mine[0])
    arr = R.layer_array(layers)
    first, last = (rank == 0), (rank == P - 1)

    comm = None
    if P > 1:
        uid = [sq.runtime.sq_comm_get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(uid, src=0)
        comm = R.Comm.nccl(uid[0], P, rank)
    ws = R.PipelineWorkspace(plan, layers, rank if P > 1 else 0)
    x0 = out = None
    if first:
        x0 = torch.empty((B, wl["s"], h1), dtype=torch.float32, device="cuda")
        synth.device_fill_f32(x0.data_ptr(), 1, 0, x0.numel(), 1.0, False)
    if last:
        out = torch.zeros((B, 1 + wl["n_dec"], h1), dtype=torch.float32, device="cuda")
    rk = rank if P > 1 else 0

    def step():
        return R.sq_pipeline_run(plan, rk, layers, comm, x0, out, ws, arr=arr)

    def barrier():
        torch.cuda.synchronize()
        if dist:
            dist.barrier()

    def max_over_ranks(v: float) -> float:
        if not dist:
            return v
        t = torch.tensor([v], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sum_over_ranks(v: float) -> float:
        if not dist:
            return v
        t = torch.tensor([v], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return float(t.item())

    for _ in range(args.warmup):
        step()
    # ---------------- timed region: device-resident inputs
    barrier()
    clocks = ClockSampler(local)
    if rank == 0:
        clocks.start()
    launches0 = sq.sq_launch_count()
    e0 = torch.cuda.Event(enable_timing=True)
    e1 = torch.cuda.Event(enable_timing=True)
    barrier()
    e0.record()
    stats = [step() for _ in range(args.steps)]
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    launches = sq.sq_launch_count() - launches0
    clk = clocks.stop() if rank == 0 else None
    ms = max_over_ranks(ms)
    # ---------------- the same K steps again with a CUDA event pair around every kernel launch
    # (per-kernel durations for the roofline; the events cost the launches their PDL overlap,
    # so this pass is slower than the timed one and only its per-kernel split is used)
    barrier()
    sq.sq_profile_enable(True)
    p0 = torch.cuda.Event(enable_timing=True)
    p1 = torch.cuda.Event(enable_timing=True)
    p0.record()
    for _ in range(args.steps):
        step()
    p1.record()
    torch.cuda.synchronize()
    sq.sq_profile_enable(False)
    prof = sq.sq_profile_read()
    prof_ms = max_over_ranks(p0.elapsed_time(p1))
    launches = int(sum_over_ranks(launches))
    tokens = args.steps * B * (1 + wl["n_dec"])
    value = tokens / (ms / 1e3)

    # dominant kernel class on this rank (rank 0 reports)
    kern = {}
    for name, bound in (("gemv", "hbm"), ("gemm", "tensor")):
        d = prof[name]
        if d["launches"] and d["ms"] > 0:
            if bound == "hbm":
                ach = d["bytes"] / (d["ms"] / 1e3) / 1e9
                kern[name] = {"bound": "hbm", "achieved": ach, "peak": pk["hbm_gbs"], "unit": "GB/s",
                              "frac": ach / pk["hbm_gbs"], "launches": d["launches"], "ms": d["ms"],
                              "bytes_per_launch": d["bytes"] / d["launches"]}
            else:
                ach = d["flops"] / (d["ms"] / 1e3) / 1e12
                kern[name] = {"bound": "tensor", "achieved": ach, "peak": pk["tflops_sustained"], "unit": "TFLOP/s",
                              "frac": ach / pk["tflops_sustained"], "launches": d["launches"], "ms": d["ms"],
                              "flops_per_launch": d["flops"] / d["launches"]}
    kern["glue_ms"] = prof["glue"]["ms"]
    kern["profiled_ms_per_step"] = prof_ms / args.steps
    dom = max((k for k in ("gemv", "gemm") if k in kern), key=lambda k: kern[k]["ms"], default=None)
    roof = None
    if dom:
        r = kern[dom]
        roof = {"bound": r["bound"], "achieved": round(r["achieved"], 2), "peak": r["peak"], "unit": r["unit"],
                "frac": round(r["frac"], 4), "traffic": traffic_for(dom, r.get("bytes_per_launch")), "kernel": dom,
                "traffic_src": "profiles/traffic.json (ncu --set full dram bytes / algorithmic bytes of one launch)",
                "peak_src": pk["src"] + (" sustained" if r["bound"] == "tensor" else " copy")}

    # ---------------- e2e: host buffers through the C-ABI, copies inside the timed region.  Every step
    # copies its embeddings host -> device and its outputs device -> host (pinned memory, a copy
    # stream): the next step's H2D and the previous step's D2H run while a step computes (double-
    # buffered device inputs/outputs); the first H2D and the last D2H are exposed.
    e2e = None
    if not args.no_e2e:
        cs = torch.cuda.Stream()
        hx = torch.empty(x0.shape, dtype=torch.float32).pin_memory() if first else None
        if first:
            hx.copy_(x0.cpu())
        x0s = [x0, torch.empty_like(x0)] if first else [None, None]
        outs = [out, torch.empty_like(out)] if last else [None, None]
        houts = [torch.empty(out.shape, dtype=torch.float32).pin_memory() for _ in range(2)] if last else None
        ev_in = [torch.cuda.Event(), torch.cuda.Event()]
        barrier()
        f0 = torch.cuda.Event(enable_timing=True)
        f1 = torch.cuda.Event(enable_timing=True)
        cur = torch.cuda.current_stream()
        f0.record()
        cs.wait_stream(cur)
        if first:
            with torch.cuda.stream(cs):
                x0s[0].copy_(hx, non_blocking=True)
                ev_in[0].record(cs)
        for i in range(args.steps):
            b = i % 2
            if first:
                cur.wait_event(ev_in[b])
                if i + 1 < args.steps:  # buffer (i+1)%2 was last read by step i-1, which has returned
                    with torch.cuda.stream(cs):
                        x0s[1 - b].copy_(hx, non_blocking=True)
                        ev_in[1 - b].record(cs)
            R.sq_pipeline_run(plan, rk, layers, comm, x0s[b], outs[b], ws, arr=arr)
            if last:
                cs.wait_stream(cur)
                with torch.cuda.stream(cs):
                    houts[b].copy_(outs[b], non_blocking=True)
        cur.wait_stream(cs)
        f1.record()
        torch.cuda.synchronize()
        ems = max_over_ranks(f0.elapsed_time(f1))
        e2e = {"value": tokens / (ems / 1e3), "unit": "tokens/s",
               "h2d_bytes_per_step": int(sum_over_ranks(x0.numel() * 4 if first else 0)),
               "d2h_bytes_per_step": int(sum_over_ranks(out.numel() * 4 if last else 0)),
               "copies": "every step: pinned host -> device embeddings and device -> pinned host outputs through "
                         "sq_pipeline_run's public API, on a copy stream overlapping the neighbouring steps' compute "
                         "(double-buffered device tensors); first H2D and last D2H exposed"}
        del x0s, outs

    # ---------------- side measurements on rank 0 at N = 1
    extra = {}
    cpu = None
    if rank == 0 and P == 1:
        if not args.no_gemv_sweep:
            extra["decode_gemv"] = {"workload": "configs[1] OPT-13B linear shapes, m = 1..32, bits 3/4/8 (+16); 40 back-to-back launches over > 2 x L2 of distinct weight copies in one CUDA graph, best of 3",
                                    "results": gemv_sweep(), "w8a8": w8a8_decode_sweep()}
        if not args.no_gemm_sweep:
            extra["prefill_gemm"] = {"workload": "configs[2] OPT-30B linear shapes (fused qkv 21504x7168, o 7168^2, fc1 28672x7168, fc2 7168x28672) at M = 8 x 512 = 4096 tokens, bits 3/4/8/16; median of 5 event-timed launches after 2 warm-up",
                                     "results": gemm_sweep(pk)}
        if not args.no_configs0:
            extra["configs0"] = configs0_latency()
        if not args.no_attention:
            del ws
            torch.cuda.empty_cache()
            extra["attention"] = attention_run(wl, plan, layers, arr, x0, pk)
        if not args.no_tp and args.workload == "opt66b":
            layers.clear()
            torch.cuda.empty_cache()
            extra["tp_stage"] = tp_run()
        if not args.no_bloom and args.workload == "opt66b":
            layers.clear()  # the OPT-66B model's HBM goes to the BLOOM-176B-shaped one
            torch.cuda.empty_cache()
            extra["configs4"] = bloom_run(pk)
        if not args.no_cpu:
            cpu = cpu_baseline(wl, B, args.cpu_tokens, args.cpu_row_frac)
    if rank == 0:
        st = stats[-1]
        line = {
            "metric": METRIC, "value": value, "unit": "tokens/s", "n_gpus": P, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f16", "data": "synthetic",
            "config": {"workload": wl["name"], "B": B, "eta": wl["eta"], "xi": wl["xi"], "prompt_len": wl["s"],
                       "n_decode": wl["n_dec"], "layers": L, "hidden": h1, "ffn": h2,
                       "bits_histogram": {str(b): bits.count(b) for b in (3, 4, 8, 16)},
                       "stage_sizes": [sol.count(s) for s in range(P)],
                       "weights_GB": round(sum(PL.layer_bytes(h1, h2, b) for b in bits) / 1e9, 2),
                       "l2": "inputs larger than L2: every step streams all packed weights (tens of GB)",
                       "parallelism": f"pp{P}"},
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches, "clocks": clk,
            "kernels": kern,
            "phase_ms_rank0": {"prefill": st["t_prefill_ms"], "decode": st["t_decode_ms"]},
            "gpus_active": P,
        }
        if selfcheck is not None:
            line["pipeline_bitwise_ok"] = selfcheck["pipeline_bitwise_ok"]
            line["selfcheck"] = selfcheck
        line.update(extra)
        print(json.dumps(line), flush=True)
    if comm:
        comm.destroy()
    if dist:
        dist.barrier()
        dist.destroy_process_group()


def spawn_ranks(n: int) -> None:
    """`python bench.py --gpus N` without torchrun: re-exec under torch.distributed.run with one rank per
    GPU (never silently measure fewer GPUs than asked for)."""
    import socket
    import torch
    have = torch.cuda.device_count()
    if have < n:
        print(json.dumps({"metric": METRIC, "error": f"--gpus {n} requested but only {have} CUDA device(s) visible",
                          "n_gpus": n, "gpus_active": have}), flush=True)
        raise SystemExit(1)
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    os.execv(sys.executable, cmd)


# ------------------------------------------------------------------ prefill GEMM sweep (configs[2])
def gemm_sweep(pk: dict, reps: int = 5):
    """configs[2]: OPT-30B linear shapes at M = eta * s = 8 * 512 = 4096 tokens, bits 3/4/8/16.  TFLOP/s =
    2 M N K / event-timed launch duration (median of `reps` after 2 warm-up launches); fractions of the
    measured bf16 dense peaks (burst and sustained)."""
    import torch
    import synth
    import paper_conf_cluster_zhaowplw25_b200 as sq
    h1, h2, M = 7168, 28672, 4096
    out = []
    x = torch.empty((M, h2), dtype=torch.float16, device="cuda")
    synth.device_fill_f16(x.data_ptr(), 9, 0, x.numel(), 1.0, False)
    for name, (n, k) in (("qkv", (3 * h1, h1)), ("o", (h1, h1)), ("fc1", (h2, h1)), ("fc2", (h1, h2))):
        wd = torch.empty((n, k), dtype=torch.float16, device="cuda")
        synth.device_weight_f16(wd.data_ptr(), synth.weight_seed(0, name), n, k)
        xk = x[:, :k].contiguous()
        y = torch.empty((M, n), dtype=torch.float16, device="cuda")
        for bits in (3, 4, 8, 16):
            q = sq.QLinear.from_fp16(wd, bits)
            for _ in range(2):
                sq.sq_linear_prefill(q, xk, y, 0)
            ts = []
            for _ in range(reps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                sq.sq_linear_prefill(q, xk, y, 0)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            ms = statistics.median(ts)
            tf = 2.0 * M * n * k / (ms / 1e3) / 1e12
            out.append({"linear": name, "n": n, "k": k, "bits": bits, "m": M, "us": round(ms * 1e3, 1),
                        "TFLOPs": round(tf, 1), "frac_burst": round(tf / pk["tflops"], 3),
                        "frac_sustained": round(tf / pk["tflops_sustained"], 3)})
            del q
        # f4 W8A8 (kind::i8 tensor cores, per-token activation quantization included in the timing);
        # INT8 dense peak = the measured bf16 peak x 2 (the guide's nominal ratio)
        w8 = sq.W8Linear.from_fp16(wd)
        ts = []
        for r in range(2 + reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            xq, sx = sq.sq_quantize_act8(xk)
            sq.sq_linear_w8a8(w8, xq, sx, y, 0)
            e1.record()
            torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
        ms = statistics.median(ts)
        tf = 2.0 * M * n * k / (ms / 1e3) / 1e12
        out.append({"linear": name, "n": n, "k": k, "bits": "w8a8", "m": M, "us": round(ms * 1e3, 1), "TFLOPs": round(tf, 1),
                    "frac_int8_peak": round(tf / (2 * pk["tflops"]), 3), "peak_note": "int8 dense = 2 x measured bf16 (burst)"})
        del w8
        del wd, xk, y
    return out


# ------------------------------------------------------------------ configs[0] latency
def configs0_latency(runs: int = 20):
    """BASELINE.json configs[0] (OPT-125m shapes, 12 layers, bits {3,4,8,16}, G = 128, one sequence: prefill
    1 x 32 tokens + 8 decode steps, 1 GPU): per-run latency through sq_pipeline_run, and the decode step
    (all 12 layers at 1 token) captured in one CUDA graph."""
    import torch
    import synth
    from paper_conf_cluster_zhaowplw25_b200 import runtime as R
    wl = WORKLOADS["opt125m"]
    h1, h2, L = wl["h1"], wl["h2"], wl["L"]
    bits = workload_bits(wl)
    g = R.build_layers(L, h1, h2, bits)
    plan = R.Plan(bits, [0] * L, h1, h2, 1, 1, 1, wl["s"], wl["n_dec"])
    ws = R.PipelineWorkspace(plan, g, 0)
    x0 = torch.empty((1, wl["s"], h1), dtype=torch.float32, device="cuda")
    synth.device_fill_f32(x0.data_ptr(), 1, 0, x0.numel(), 1.0, False)
    out = torch.zeros((1, 1 + wl["n_dec"], h1), dtype=torch.float32, device="cuda")
    arr = R.layer_array(g)
    for _ in range(3):
        R.sq_pipeline_run(plan, 0, g, None, x0, out, ws, arr=arr)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(runs):
        R.sq_pipeline_run(plan, 0, g, None, x0, out, ws, arr=arr)
    e1.record()
    torch.cuda.synchronize()
    run_ms = e0.elapsed_time(e1) / runs
    # decode step (12 layers, 1 token) as one CUDA graph
    sw = R.StageWorkspace(g, 1)
    xi = torch.zeros((1, h1), dtype=torch.float32, device="cuda")
    xo = torch.empty_like(xi)
    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(side):
        R.sq_stage_forward(g, 1, xi, xo, sw, arr=arr)
    torch.cuda.current_stream().wait_stream(side)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph):
        R.sq_stage_forward(g, 1, xi, xo, sw, arr=arr)
    graph.replay()
    torch.cuda.synchronize()
    e0.record()
    for _ in range(100):
        graph.replay()
    e1.record()
    torch.cuda.synchronize()
    step_us = e0.elapsed_time(e1) / 100 * 1e3
    return {"workload": wl["name"], "bits": bits, "ms_per_run": round(run_ms, 3),
            "tokens_per_s": round((1 + wl["n_dec"]) / (run_ms / 1e3), 1),
            "decode_step_us_cuda_graph": round(step_us, 1),
            "note": "one sequence; per-run = prefill 32 tokens + 8 decode steps through sq_pipeline_run (P = 1)"}


# ------------------------------------------------------------------ configs[4] side line
def bloom_run(pk: dict, steps: int = 1):
    """BASELINE.json configs[4] on ONE B200: BLOOM-176B-shaped (d = 14336, fused QKV, GeLU), 70 layers,
    INT3/INT4 50/50 (80.9 GB), B = 32, eta = 8, xi = 32, prompt 512 + 128 decode tokens (the paper's
    8-way pipeline needs 8 GPUs; this is its 1-GPU point).  One warm-up run, `steps` timed runs."""
    import torch
    import synth
    from paper_conf_cluster_zhaowplw25_b200 import runtime as R
    from paper_conf_cluster_zhaowplw25_b200 import plan as PL
    wl = WORKLOADS["bloom176b"]
    L, h1, h2, B = wl["L"], wl["h1"], wl["h2"], wl["b_per_gpu"]
    bits = workload_bits(wl)
    g = R.build_layers(L, h1, h2, bits, act=wl["act"])
    plan = R.Plan(bits, [0] * L, h1, h2, B, wl["eta"], wl["xi"], wl["s"], wl["n_dec"])
    ws = R.PipelineWorkspace(plan, g, 0)
    arr = R.layer_array(g)
    x0 = torch.empty((B, wl["s"], h1), dtype=torch.float32, device="cuda")
    synth.device_fill_f32(x0.data_ptr(), 1, 0, x0.numel(), 1.0, False)
    out = torch.zeros((B, 1 + wl["n_dec"], h1), dtype=torch.float32, device="cuda")
    R.sq_pipeline_run(plan, 0, g, None, x0, out, ws, arr=arr)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(steps):
        st = R.sq_pipeline_run(plan, 0, g, None, x0, out, ws, arr=arr)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    res = {"workload": wl["name"] + " (1 GPU)", "B": B, "weights_GB": round(sum(PL.layer_bytes(h1, h2, b) for b in bits) / 1e9, 1),
           "bits_histogram": {str(b): bits.count(b) for b in (3, 4)}, "ms_per_step": round(ms, 1),
           "tokens_per_s": round(B * (1 + wl["n_dec"]) / (ms / 1e3), 1),
           "phase_ms": {"prefill": round(st["t_prefill_ms"], 1), "decode": round(st["t_decode_ms"], 1)}}
    del g, ws, x0, out
    torch.cuda.empty_cache()
    return res


# ------------------------------------------------------------------ f4: tensor-parallel stages
def tp_run(reps: int = 5, tps=(2, 4, 8)):
    """SURVEY 8(f) f4 intra-node TP: 4 OPT-66B-shaped layers (bits 4/3/4/8) as one stage,
    unsharded (sq_stage_forward) and split T ways (sq_stage_forward_tp, virtual: the T shard sets run
    one after the other on this GPU, so time / T is one TP rank's compute).  Decode micro-batch 32 and a
    2048-token prefill item; each call captured in a CUDA graph, median of `reps` replays.
    eff = t(TP1) / t(TP T virtual): 1.0 means the 1/T-wide kernels keep the unsharded kernels' efficiency,
    i.e. T ranks would run the stage T x faster before the all-reduce (not measurable on one GPU; its
    algorithmic volume per rank is 2 x layers x tokens x h1 x 4 bytes per step, reported)."""
    import statistics
    import torch
    import synth
    from paper_conf_cluster_zhaowplw25_b200 import runtime as R
    L, h1, h2 = 4, 9216, 36864
    bits = [4, 3, 4, 8]
    cases = (("decode", 1, 32), ("prefill", 0, 2048))

    def timed(fn):
        fn()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            fn()
        g.replay()
        torch.cuda.synchronize()
        ts = []
        for _ in range(reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            g.replay()
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        del g
        return statistics.median(ts)

    res = {"workload": "4 OPT-66B layers (h1 9216, h2 36864), bits 4/3/4/8; decode m = 32, prefill 2048 tokens",
           "results": []}
    base = {}
    g1 = R.build_layers(L, h1, h2, bits)
    for name, phase, T_tok in cases:
        x = torch.empty((T_tok, h1), dtype=torch.float32, device="cuda")
        synth.device_fill_f32(x.data_ptr(), 5, 0, x.numel(), 1.0, False)
        y = torch.empty_like(x)
        ws = R.StageWorkspace(g1, T_tok)
        arr = R.layer_array(g1)
        base[name] = timed(lambda: R.sq_stage_forward(g1, phase, x, y, ws, arr=arr))
        res["results"].append({"tp": 1, "phase": name, "ms": round(base[name], 3)})
        del ws
    del g1
    torch.cuda.empty_cache()
    for T in tps:
        sets = R.build_tp_layers(L, h1, h2, bits, T)
        for name, phase, T_tok in cases:
            x = torch.empty((T_tok, h1), dtype=torch.float32, device="cuda")
            synth.device_fill_f32(x.data_ptr(), 5, 0, x.numel(), 1.0, False)
            y = torch.empty_like(x)
            ws = R.TpWorkspace(sets, T_tok)
            ms = timed(lambda: R.sq_stage_forward_tp(sets, phase, x, y, ws, T))
            res["results"].append({"tp": T, "phase": name, "ms_all_shards": round(ms, 3),
                                   "ms_per_rank": round(ms / T, 3), "eff": round(base[name] / ms, 3),
                                   "allreduce_MB_per_rank": round(2 * L * T_tok * h1 * 4 / 1e6, 1)})
            del ws
        del sets
        torch.cuda.empty_cache()
    return res


# ------------------------------------------------------------------ f3: the same run with real attention
def attention_run(wl: dict, plan0, layers, arr, x0, pk: dict, steps: int = 1):
    """the configs[3] generation with causal attention over a KV cache (head_dim 128,
    h1 / 128 heads; KV cache 2 x B x (s + n_dec) x h1 fp16 per layer inside the pipeline workspace)
    in place of the R12 stub; same layers, plan and inputs.  One warm-up run, `steps` timed runs, then a
    profiled run for the attention kernels' own rooflines (decode: KV-cache GB/s vs HBM; prefill: causal
    TFLOP/s)."""
    import torch
    import paper_conf_cluster_zhaowplw25_b200 as sq
    from paper_conf_cluster_zhaowplw25_b200 import runtime as R
    heads = wl["h1"] // 128
    plan = R.Plan(plan0.bits, plan0.stage_of_layer, plan0.hidden, plan0.ffn, plan0.B, plan0.eta, plan0.xi,
                  plan0.prompt_len, plan0.n_decode, n_heads=heads, kappa=1)
    R.sq_plan_check(plan)
    ws = R.PipelineWorkspace(plan, layers, 0)
    out = torch.zeros((plan.B, 1 + plan.n_decode, plan.hidden), dtype=torch.float32, device="cuda")
    R.sq_pipeline_run(plan, 0, layers, None, x0, out, ws, arr=arr)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    st = None
    for _ in range(steps):
        st = R.sq_pipeline_run(plan, 0, layers, None, x0, out, ws, arr=arr)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / steps
    sq.sq_profile_enable(True)
    R.sq_pipeline_run(plan, 0, layers, None, x0, out, ws, arr=arr)
    torch.cuda.synchronize()
    sq.sq_profile_enable(False)
    prof = sq.sq_profile_read()
    ad, ap_ = prof["attn_decode"], prof["attn_prefill"]
    kv_gb = 2 * plan.B * (plan.prompt_len + plan.n_decode) * plan.hidden * 2 * len(layers) / 1e9
    res = {"workload": wl["name"] + ", with causal attention over a KV cache (f3)", "n_heads": heads, "head_dim": 128,
           "kv_cache_GB": round(kv_gb, 2), "ms_per_step": round(ms, 1),
           "tokens_per_s": round(plan.B * (1 + plan.n_decode) / (ms / 1e3), 1),
           "phase_ms": {"prefill": round(st["t_prefill_ms"], 1), "decode": round(st["t_decode_ms"], 1)},
           "gpu_launches_per_step": st["gpu_launches"]}
    if ad["launches"] and ad["ms"] > 0:
        gbs = ad["bytes"] / (ad["ms"] / 1e3) / 1e9
        res["decode_attention"] = {"bound": "hbm", "achieved": round(gbs, 1), "peak": pk["hbm_gbs"], "unit": "GB/s",
                                   "frac": round(gbs / pk["hbm_gbs"], 3), "launches": ad["launches"],
                                   "ms_per_step": round(ad["ms"], 1),
                                   "bytes_per_launch": ad["bytes"] / ad["launches"]}
    if ap_["launches"] and ap_["ms"] > 0:
        tf = ap_["flops"] / (ap_["ms"] / 1e3) / 1e12
        res["prefill_attention"] = {"bound": "tensor", "achieved": round(tf, 1), "unit": "TFLOP/s",
                                    "peak_mma_sync_note": "mma.sync path; the tcgen05 peak is " + str(pk["tflops"]),
                                    "launches": ap_["launches"], "ms_per_step": round(ap_["ms"], 1)}
    del ws
    torch.cuda.empty_cache()
    return res


def traffic_for(kernel: str, per_launch: float | None = None):
    """DRAM bytes per launch of the dominant kernel from the committed ncu --set full capture
    (profiles/traffic.json): the captured launch's dram/algorithmic ratio applied to this run's
    algorithmic bytes per launch (so `traffic` and `achieved` count the same launches)."""
    try:
        with open(os.path.join(ROOT, "profiles", "traffic.json")) as f:
            t = json.load(f).get(kernel)
    except Exception:
        return None
    if not t:
        return None
    if per_launch is not None and t.get("ratio"):
        return round(t["ratio"] * per_launch)
    return t.get("dram_bytes")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", choices=sorted(WORKLOADS), default="opt66b")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-gemv-sweep", action="store_true")
    ap.add_argument("--no-gemm-sweep", action="store_true")
    ap.add_argument("--no-configs0", action="store_true")
    ap.add_argument("--no-attention", action="store_true")
    ap.add_argument("--no-bloom", action="store_true")
    ap.add_argument("--no-tp", action="store_true")
    ap.add_argument("--cpu-tokens", type=int, default=8)
    ap.add_argument("--cpu-row-frac", type=int, default=8)
    args = ap.parse_args()
    wl = WORKLOADS[args.workload]
    if args.impl == "ours" and args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        spawn_ranks(args.gpus)  # does not return
    if args.impl == "reference":
        run_reference(args, wl)
    else:
        run_ours(args, wl)


if __name__ == "__main__":
    main()
