"""Host-side plan helpers (the planner is an INPUT of the hot path, BASELINE.json north_star).

``partition_layers`` is the θ = 0, bits-fixed special case of SplitQuant's
eq. (4): choose a contiguous partition (eqs. 15-16) of
L layers into P stages minimising the slowest stage's phase-aware cost
    T_j = sum_{l in stage j} ( mu_pre * t_pre(l) + n_dec * mu_dec * t_dec(l) )
(eqs. 5-6).  With uniform devices (8 x B200 over NVSwitch) the
device-ordering enumeration of the paper is moot.  Exact O(P L^2) DP.
"""
from __future__ import annotations

import math


def layer_bytes(h1: int, h2: int, bits: int, group: int = 128) -> int:
    """Decode-streamed bytes of one layer: codes + fp16 scale/zero per group."""
    params = 4 * h1 * h1 + 2 * h1 * h2
    if bits == 16:
        return 2 * params
    return params * bits // 8 + (params // group) * 4


def layer_flops(h1: int, h2: int, tokens: int) -> float:
    return 2.0 * tokens * (4 * h1 * h1 + 2 * h1 * h2)


def phase_costs(bits: list[int], h1: int, h2: int, B: int, eta: int, xi: int, s: int, n_dec: int,
                hbm_gbs: float = 6550.4, tflops: float = 1382.0) -> list[float]:
    """Per-layer phase-aware cost (seconds) from the roofline model (HBM for decode, tensor for prefill)."""
    mu_pre, mu_dec = math.ceil(B / eta), math.ceil(B / xi)
    out = []
    for b in bits:
        t_pre = layer_flops(h1, h2, eta * s) / (tflops * 1e12)
        t_dec = layer_bytes(h1, h2, b) / (hbm_gbs * 1e9)
        out.append(mu_pre * t_pre + n_dec * mu_dec * t_dec)
    return out


def partition_layers(costs: list[float], P: int) -> list[int]:
    """Exact min-max contiguous partition of ``costs`` into P non-empty stages -> stage_of_layer."""
    L = len(costs)
    if not 1 <= P <= L:
        raise ValueError("need 1 <= P <= L")
    pre = [0.0]
    for c in costs:
        pre.append(pre[-1] + c)
    INF = float("inf")
    # best[p][i] = min over partitions of first i layers into p stages of the max stage cost
    best = [[INF] * (L + 1) for _ in range(P + 1)]
    arg = [[-1] * (L + 1) for _ in range(P + 1)]
    best[0][0] = 0.0
    for p in range(1, P + 1):
        for i in range(p, L + 1):
            for j in range(p - 1, i):
                v = max(best[p - 1][j], pre[i] - pre[j])
                if v < best[p][i] - 1e-15:
                    best[p][i], arg[p][i] = v, j
    cuts = []
    i = L
    for p in range(P, 0, -1):
        j = arg[p][i]
        cuts.append((j, i))
        i = j
    stage_of_layer = [0] * L
    for s, (a, b) in enumerate(reversed(cuts)):
        for l in range(a, b):
            stage_of_layer[l] = s
    return stage_of_layer


def stage_costs(costs: list[float], stage_of_layer: list[int]) -> list[float]:
    P = max(stage_of_layer) + 1
    out = [0.0] * P
    for c, s in zip(costs, stage_of_layer):
        out[s] += c
    return out


def pipeline_latency_model(stage_pre: list[float], stage_dec: list[float], mu_pre: int, mu_dec: int,
                           n_dec: int) -> float:
    """Eq. (4) first term: all stages + (mu - 1) x slowest, per phase (n_dec decode steps)."""
    pre = sum(stage_pre) + (mu_pre - 1) * max(stage_pre)
    dec = n_dec * (sum(stage_dec) + (mu_dec - 1) * max(stage_dec))
    return pre + dec
