"""f1 + f2 end to end on one B200: fit the phase-aware latency cost model to this GPU,
compute the variance indicator omega (eq. 3) of every layer with the library's kernels, solve the
bit-width / partition problem (eq. 4) for 1/2/4/8 B200, and check the model against a measured
run of the 1-GPU plan (cost-model fidelity, "< 6 %").

  python tools/plan_flow.py [--model opt66b|opt13b] [--theta T] [--out profiles/r01_planner.json]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
from paper_conf_cluster_zhaowplw25_b200 import costmodel as CM
from paper_conf_cluster_zhaowplw25_b200 import indicator as IND
from paper_conf_cluster_zhaowplw25_b200 import planner as PL
from paper_conf_cluster_zhaowplw25_b200 import runtime as R

MODELS = {"opt66b": dict(h1=9216, h2=36864, L=64), "opt13b": dict(h1=5120, h2=20480, L=40),
          "opt125m": dict(h1=768, h2=3072, L=12)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--model", default="opt66b", choices=sorted(MODELS))
    ap.add_argument("--theta", type=float, default=None, help="default: balance latency and quality scales")
    ap.add_argument("--eta", type=int, default=8)
    ap.add_argument("--xi", type=int, default=32)
    ap.add_argument("--s", type=int, default=512)
    ap.add_argument("--n", type=int, default=129, help="generated tokens (prefill token + n - 1 decode steps)")
    ap.add_argument("--mem-gb", type=float, default=170.0, help="M_j per B200 for weights + KV (180 GB HBM3e minus context/workspace)")
    ap.add_argument("--omega-layers", type=int, default=0, help="layers to compute omega for (0 = all)")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    mdl = MODELS[a.model]
    h1, h2, L = mdl["h1"], mdl["h2"], mdl["L"]
    out = {"model": a.model, "h1": h1, "h2": h2, "layers": L}

    # ---- 1. latency cost model: fit on profiled points, validate on unseen workloads
    t0 = time.time()
    # train and unseen points measured interleaved in one random order (same thermal / clock mix)
    sets = CM.profile_interleaved(h1, h2, {
        "train": {"pre": ((1, 128), (1, 512), (2, 256), (2, 1024), (4, 128), (4, 512), (8, 256), (8, 512), (16, 256),
                          (6, 640)),
                  "dec": ((1, 256), (2, 1024), (4, 512), (6, 128), (8, 512), (12, 256), (16, 384), (24, 900),
                          (32, 640), (32, 1024))},
        "unseen": {"pre": ((3, 384), (5, 256), (6, 448), (12, 320)),
                   "dec": ((3, 384), (5, 700), (12, 768), (20, 200), (28, 512))}})
    train, unseen = sets["train"], sets["unseen"]
    model = CM.LatencyModel.fit(train, {"gpu": torch.cuda.get_device_name(0), "h1": h1, "h2": h2})
    err_tr, err_un = model.errors(train), model.errors(unseen)
    out["costmodel"] = {"coef": json.loads(model.to_json())["coef"], "train_points": len(train),
                        "train_err_mean": float(np.mean(err_tr)), "unseen_points": len(unseen),
                        "unseen_err_mean": float(np.mean(err_un)), "unseen_err_max": float(np.max(err_un)),
                        "unseen": [dict(r, pred=model.predict(r)) for r in unseen], "profile_s": round(time.time() - t0, 1)}
    print(json.dumps({k: v for k, v in out["costmodel"].items() if k not in ("coef", "unseen")}), flush=True)

    # ---- 2. variance indicator per layer (synthetic weights + synthetic calibration tokens)
    t0 = time.time()
    nl = L if a.omega_layers <= 0 else min(L, a.omega_layers)
    omegas = []
    for l in range(nl):
        t = IND.layer_terms(l, h1, h2, calib_tokens=128)
        omegas.append({b: IND.omega(t, b) for b in (3, 4, 8, 16)})
    while len(omegas) < L:
        omegas.append(omegas[len(omegas) % nl])
    out["omega"] = {"layers_computed": nl, "mean": {b: float(np.mean([o[b] for o in omegas])) for b in (3, 4, 8)},
                    "cv": {b: float(np.std([o[b] for o in omegas]) / np.mean([o[b] for o in omegas])) for b in (3, 4, 8)},
                    "seconds": round(time.time() - t0, 1)}
    print(json.dumps(out["omega"]), flush=True)
    torch.cuda.empty_cache()

    # ---- 3. plans for 1/2/4/8 B200 (weak scaling B = 32 N)
    plans = {}
    for N in (1, 2, 4, 8):
        B = 32 * N
        l_pre = {b: model.t_pre(b, a.eta, a.s) for b in (3, 4, 8, 16)}
        l_dec = {b: model.t_dec(b, a.xi, a.s + a.n // 2) for b in (3, 4, 8, 16)}
        mem = {b: PL.layer_memory(h1, h2, b, B, a.s, a.n) for b in (3, 4, 8, 16)}
        lat_scale = (a.n - 1) * L * l_dec[4]
        theta = a.theta if a.theta is not None else 0.05 * lat_scale / max(L * omegas[0][4], 1e-30)
        p = PL.Problem(L, N, (3, 4, 8, 16), l_pre, l_dec, mem, omegas, theta, B, a.eta, a.xi, a.n, a.mem_gb * 1e9)
        t0 = time.time()
        sol = PL.solve(p)
        tokens = B * a.n
        plans[N] = {"B": B, "theta": theta, "bits_histogram": {b: sol.bits.count(b) for b in (3, 4, 8, 16)},
                    "stage_sizes": [sol.stage_of_layer.count(j) for j in range(N)], "bits": sol.bits,
                    "stage_of_layer": sol.stage_of_layer, "objective": sol.objective,
                    "predicted_latency_s": sol.latency, "predicted_tokens_per_s": tokens / sol.latency,
                    "quality_term": sol.quality, "solve_s": round(time.time() - t0, 2), "iterations": len(sol.log)}
        print(json.dumps({k: v for k, v in plans[N].items() if k not in ("bits", "stage_of_layer")}), flush=True)
    out["plans"] = plans

    # ---- 4. fidelity: run the 1-GPU plan (all stages on this GPU) and compare with the model
    pl = plans[1]
    plan = R.Plan(pl["bits"], pl["stage_of_layer"], h1, h2, pl["B"], a.eta, a.xi, a.s, a.n - 1)
    layers = R.build_layers(L, h1, h2, pl["bits"])
    ws = R.PipelineWorkspace(plan, layers, 0)
    x0 = torch.empty((pl["B"], a.s, h1), dtype=torch.float32, device="cuda")
    synth.device_fill_f32(x0.data_ptr(), 1, 0, x0.numel(), 1.0, False)
    y = torch.zeros((pl["B"], a.n, h1), dtype=torch.float32, device="cuda")
    arr = R.layer_array(layers)
    R.sq_pipeline_run(plan, 0, layers, None, x0, y, ws, arr=arr)
    st = R.sq_pipeline_run(plan, 0, layers, None, x0, y, ws, arr=arr)
    meas = st["t_total_ms"] / 1e3
    out["fidelity_1gpu"] = {"measured_s": meas, "predicted_s": pl["predicted_latency_s"],
                            "rel_err": abs(pl["predicted_latency_s"] - meas) / meas,
                            "measured_prefill_s": st["t_prefill_ms"] / 1e3, "measured_decode_s": st["t_decode_ms"] / 1e3}
    print(json.dumps(out["fidelity_1gpu"]), flush=True)
    if a.out:
        with open(a.out, "w") as f:
            json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
