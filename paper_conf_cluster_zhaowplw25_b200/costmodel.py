"""f1 — SplitQuant's phase-aware latency cost model (Sec. IV-A), fitted to THIS B200.

The paper models the execution time of ONE decoder layer per precision and phase by linear
regression over profiled sample points:

  prefill (compute-bound, "a function of FLOPs"):   t_pre(v, s)      ~ [1, v, s, v s, v s^2]
  decode  (memory-bound, "MOPs"):                    t_dec(v, t + s)  ~ [1, v, v (t+s), (t+s)]

with v the micro-batch size, s the prompt length and t + s the past sequence length.  Here the
samples are our own kernels (``sq_stage_forward`` on an 8-layer synthetic stage, CUDA events), fitted per
bit width by least squares; the model error on unseen workloads is reported like the paper's
< 6 %.  The attention stub (reading R12) has no KV cache, so the (t+s) terms fit to ~0 on
this path; they are kept so the model has the paper's form.

Profiling needs the GPU (``profile``); fitting / prediction are plain host code.
"""
from __future__ import annotations

import json
import statistics

import numpy as np

PRE_FEATURES = ("1", "v", "s", "v*s", "v*s^2")
DEC_FEATURES = ("1", "v", "v*(t+s)", "(t+s)")


def pre_features(v: float, s: float) -> np.ndarray:
    return np.array([1.0, v, s, v * s, v * s * s], np.float64)


def dec_features(v: float, ctx: float) -> np.ndarray:
    return np.array([1.0, v, v * ctx, ctx], np.float64)


class LatencyModel:
    """Per-bit, per-phase linear regression of one layer's time (seconds)."""

    def __init__(self, coef: dict | None = None, meta: dict | None = None):
        self.coef = coef or {}  # {"pre": {bits: [..]}, "dec": {bits: [..]}}
        self.meta = meta or {}

    # ---------------------------------------------------------------- fit / predict
    @staticmethod
    def _lstsq(X: np.ndarray, y: np.ndarray) -> np.ndarray:
        # relative least squares (errors weighted by 1/y): the paper reports relative errors
        w = 1.0 / np.maximum(y, 1e-12)
        c, *_ = np.linalg.lstsq(X * w[:, None], y * w, rcond=None)
        return c

    @classmethod
    def fit(cls, samples: list[dict], meta: dict | None = None) -> "LatencyModel":
        """samples: {"phase": "pre"|"dec", "bits": b, "v": v, "s": s, "ctx": t+s, "t": seconds}."""
        coef = {"pre": {}, "dec": {}}
        for phase, feat in (("pre", lambda r: pre_features(r["v"], r["s"])),
                            ("dec", lambda r: dec_features(r["v"], r["ctx"]))):
            for b in sorted({r["bits"] for r in samples if r["phase"] == phase}):
                rows = [r for r in samples if r["phase"] == phase and r["bits"] == b]
                X = np.stack([feat(r) for r in rows])
                y = np.array([r["t"] for r in rows])
                coef[phase][int(b)] = cls._lstsq(X, y).tolist()
        return cls(coef, meta)

    def t_pre(self, bits: int, v: float, s: float) -> float:
        return float(pre_features(v, s) @ np.array(self.coef["pre"][int(bits)]))

    def t_dec(self, bits: int, v: float, ctx: float) -> float:
        return float(dec_features(v, ctx) @ np.array(self.coef["dec"][int(bits)]))

    def predict(self, r: dict) -> float:
        return self.t_pre(r["bits"], r["v"], r["s"]) if r["phase"] == "pre" else self.t_dec(r["bits"], r["v"], r["ctx"])

    def errors(self, samples: list[dict]) -> list[float]:
        """|predicted - measured| / measured per sample."""
        return [abs(self.predict(r) - r["t"]) / r["t"] for r in samples]

    # ---------------------------------------------------------------- persistence
    def to_json(self) -> str:
        return json.dumps({"coef": {p: {str(b): c for b, c in d.items()} for p, d in self.coef.items()},
                           "meta": self.meta}, indent=1)

    @classmethod
    def from_json(cls, txt: str) -> "LatencyModel":
        d = json.loads(txt)
        return cls({p: {int(b): c for b, c in v.items()} for p, v in d["coef"].items()}, d.get("meta"))


# ---------------------------------------------------------------- profiling (GPU)
def profile(h1: int, h2: int, bits_set=(3, 4, 8, 16), pre_points=((1, 128), (1, 512), (2, 256), (4, 512), (8, 512)),
            dec_points=((1, 256), (8, 512), (16, 384), (32, 640), (32, 1024)), reps: int = 5, act: int = 0,
            n_layers: int = 8) -> list[dict]:
    """Time sq_stage_forward per bit width on a stage of ``n_layers`` synthetic layers (so the
    per-layer time includes the steady-state launch overlap of consecutive layers, as in a real
    stage) and divide by n_layers: prefill v sequences x s tokens, decode v tokens (past length
    ctx).  Distinct layers: every weight byte streams from HBM."""
    import torch
    from . import SQ_DECODE, SQ_PREFILL
    from .runtime import StageWorkspace, build_layers, layer_array, sq_stage_forward
    out = []
    for b in bits_set:
        copies = build_layers(n_layers, h1, h2, [b] * n_layers, act=act)
        arr = layer_array(copies)
        max_tok = max(v * s for v, s in pre_points)
        ws = StageWorkspace(copies, max_tok)
        x = torch.randn(max_tok, h1, device="cuda")
        y = torch.empty_like(x)
        for phase, pts in (("pre", pre_points), ("dec", dec_points)):
            for (v, s_or_ctx) in pts:
                tokens = v * s_or_ctx if phase == "pre" else v
                ph = SQ_PREFILL if phase == "pre" else SQ_DECODE
                ts = []
                for rep in range(reps + 1):
                    e0 = torch.cuda.Event(enable_timing=True)
                    e1 = torch.cuda.Event(enable_timing=True)
                    e0.record()
                    sq_stage_forward(copies, ph, x[:tokens], y[:tokens], ws, arr=arr)
                    e1.record()
                    torch.cuda.synchronize()
                    if rep:
                        ts.append(e0.elapsed_time(e1) / 1e3 / len(copies))
                rec = {"phase": phase, "bits": int(b), "v": int(v), "t": statistics.median(ts)}
                if phase == "pre":
                    rec.update(s=int(s_or_ctx), ctx=int(s_or_ctx))
                else:
                    rec.update(s=int(s_or_ctx), ctx=int(s_or_ctx))
                out.append(rec)
        del copies, ws
        torch.cuda.empty_cache()
    return out


def profile_interleaved(h1: int, h2: int, point_sets: dict, bits_set=(3, 4, 8, 16), reps: int = 5, dec_reps: int = 25,
                        act: int = 0, n_layers: int = 8, seed: int = 0) -> dict:
    """As ``profile``, for several named point sets at once ({"train": {"pre": [...], "dec": [...]}, "unseen":
    ...}), every (set, bits, phase, point) measured in one seeded random order with all bit widths'
    stages resident.  The board runs at its power limit and the clock drifts with the load history
    (1275-1965 MHz), so profiling one set after the other puts a clock difference
    between the fit and its validation; interleaving gives both sets the same mix of thermal states.
    Returns {set name: [samples]}."""
    import random
    import torch
    from . import SQ_DECODE, SQ_PREFILL
    from .runtime import StageWorkspace, build_layers, layer_array, sq_stage_forward
    max_tok = max(v * s for d in point_sets.values() for v, s in d.get("pre", ()))
    stages = {}
    for b in bits_set:
        copies = build_layers(n_layers, h1, h2, [b] * n_layers, act=act)
        stages[b] = (copies, layer_array(copies), StageWorkspace(copies, max_tok))
    x = torch.randn(max_tok, h1, device="cuda")
    y = torch.empty_like(x)
    jobs = [(name, b, ph, pt) for name, d in point_sets.items() for b in bits_set for ph in ("pre", "dec")
            for pt in d.get(ph, ())]
    random.Random(seed).shuffle(jobs)
    out = {name: [] for name in point_sets}
    for name, b, phase, (v, s_or_ctx) in jobs:
        copies, arr, ws = stages[b]
        tokens = v * s_or_ctx if phase == "pre" else v
        ph = SQ_PREFILL if phase == "pre" else SQ_DECODE
        run = lambda: sq_stage_forward(copies, ph, x[:tokens], y[:tokens], ws, arr=arr)
        if phase == "dec":
            # decode steps replay from CUDA graphs in sq_pipeline_run: time them the same way (the
            # ~6 launches per layer would otherwise be host-enqueue bound)
            run()
            torch.cuda.synchronize()
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                run()
            run = g.replay
        ts = []
        # a decode step of the 8-layer stage is ~1-3 ms: more repetitions than a prefill point so the
        # median spans the power-capped clock's swings
        for rep in range((reps if phase == "pre" else dec_reps) + 1):
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            run()
            e1.record()
            torch.cuda.synchronize()
            if rep:
                ts.append(e0.elapsed_time(e1) / 1e3 / len(copies))
        out[name].append({"phase": phase, "bits": int(b), "v": int(v), "s": int(s_or_ctx), "ctx": int(s_or_ctx),
                          "t": statistics.median(ts)})
    del stages
    torch.cuda.empty_cache()
    return out

