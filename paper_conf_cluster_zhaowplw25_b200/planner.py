"""f1 — SplitQuant's joint bit-width / layer-partition planner (Sec. IV-C, eqs. 4-16)
for a single node of uniform B200s (host-side; its output is the hot path's plan input).

Objective (eq. 4 with reading R18 of DESIGN.md -- the decode terms count the n - 1 decode steps,
P:204 "the decode time of the remaining n - 1 tokens"):

    J = (mu_pre - 1) Tmax_pre + T_pre + (n - 1) [ (mu_dec - 1) Tmax_dec + T_dec ] + theta sum_i omega_{i, b_i}

    T_pre,j = sum_{i in stage j} l_pre(b_i)   (eq. 5, one prefill micro-batch of eta sequences)
    T_dec,j = sum_{i in stage j} l_dec(b_i)   (eq. 6, one decode micro-batch of xi tokens at the
                                                average past length s + n/2)
    Tmax_* >= T_*,j and >= the stage-boundary transfer time P_* / f (eq. 7), T_* = sum_j T_*,j (eq. 8)
    each layer one bit width and one stage (eqs. 9-11); stage memory <= M_j, the first stage also
    holds M_emb (eqs. 12-13); stages are contiguous and non-empty (eqs. 15-16).

With identical devices the paper's device-ordering enumeration is moot.  ``solve`` follows
the paper's bitwidth-transfer heuristic: start from the quality-optimal bit widths
that fit the memory ("adabits"), partition exactly (min-max DP over contiguous stages), then
repeatedly apply transformations on the straggler stage (lower / raise one layer's precision,
re-partition) while the objective improves.  ``brute_force`` enumerates everything (tiny
instances; the test oracle of the heuristic).
"""
from __future__ import annotations

import itertools
import math
from dataclasses import dataclass, field

import numpy as np


@dataclass
class Problem:
    n_layers: int
    n_stages: int
    bits_set: tuple                      # BITs, e.g. (3, 4, 8, 16)
    l_pre: dict                          # bits -> seconds per layer per prefill micro-batch
    l_dec: dict                          # bits -> seconds per layer per decode micro-batch
    mem: dict                            # bits -> bytes per layer (weights + KV + activations)
    omega: list                          # [n_layers] of {bits: omega_{i,b}}
    theta: float
    B: int
    eta: int
    xi: int
    n_tokens: int                        # n (generated tokens, eq. 4)
    mem_cap: float                       # M_j (uniform devices)
    mem_emb: float = 0.0                 # M_emb on the first device (eq. 13)
    xfer_pre: float = 0.0                # P_pre / f (eq. 7), seconds
    xfer_dec: float = 0.0                # P_dec / f

    @property
    def mu_pre(self) -> int:
        return math.ceil(self.B / self.eta)

    @property
    def mu_dec(self) -> int:
        return math.ceil(self.B / self.xi)


@dataclass
class Solution:
    bits: list
    stage_of_layer: list
    objective: float
    latency: float
    quality: float
    feasible: bool = True
    log: list = field(default_factory=list)


def evaluate(p: Problem, bits: list, stage_of_layer: list) -> Solution:
    """Objective (4) of a complete assignment; infeasible (memory / contiguity) -> inf."""
    N, L = p.n_stages, p.n_layers
    ok = len(bits) == L and len(stage_of_layer) == L and stage_of_layer[0] == 0 and stage_of_layer[-1] == N - 1
    ok = ok and all(0 <= stage_of_layer[i + 1] - stage_of_layer[i] <= 1 for i in range(L - 1))
    pre, dec, mem = [0.0] * N, [0.0] * N, [0.0] * N
    if ok:
        for i, (b, j) in enumerate(zip(bits, stage_of_layer)):
            pre[j] += p.l_pre[b]
            dec[j] += p.l_dec[b]
            mem[j] += p.mem[b]
        mem[0] += p.mem_emb
        ok = all(m <= p.mem_cap for m in mem)
    q = p.theta * sum(p.omega[i][b] for i, b in enumerate(bits))
    if not ok:
        return Solution(list(bits), list(stage_of_layer), math.inf, math.inf, q, False)
    tmax_pre = max(max(pre), p.xfer_pre)
    tmax_dec = max(max(dec), p.xfer_dec)
    lat = (p.mu_pre - 1) * tmax_pre + sum(pre) + (p.n_tokens - 1) * ((p.mu_dec - 1) * tmax_dec + sum(dec))
    return Solution(list(bits), list(stage_of_layer), lat + q, lat, q, True)


def _minmax_pre(p: Problem, cp, cd, cm, cap: float):
    """min over N-stage contiguous partitions with every stage's decode sum <= cap (and memory
    <= M_j) of the largest stage prefill sum; (value, stage_of_layer) or (inf, None)."""
    L, N = p.n_layers, p.n_stages
    INF = math.inf
    f = np.full((N + 1, L + 1), INF)
    arg = np.full((N + 1, L + 1), -1, np.int64)
    f[0, 0] = 0.0
    tol = cap * (1 + 1e-12) + 1e-18
    for k in range(1, N + 1):
        for i in range(k, L - (N - k) + 1):
            j = np.arange(k - 1, i)
            ok = (cd[i] - cd[j] <= tol) & (cm[i] - cm[j] + np.where(j == 0, p.mem_emb, 0.0) <= p.mem_cap)
            ok &= np.isfinite(f[k - 1, j])
            if not ok.any():
                continue
            v = np.where(ok, np.maximum(f[k - 1, j], cp[i] - cp[j]), INF)
            t = int(np.argmin(v))
            f[k, i], arg[k, i] = v[t], j[t]
    if not np.isfinite(f[N, L]):
        return INF, None
    cuts, i = [], L
    for k in range(N, 0, -1):
        j = int(arg[k, i])
        cuts.append((j, i))
        i = j
    sol = [0] * L
    for st, (a, b) in enumerate(reversed(cuts)):
        for l in range(a, b):
            sol[l] = st
    return float(f[N, L]), sol


def partition(p: Problem, bits: list) -> list | None:
    """Exact contiguous partition for fixed bits: minimises (mu_pre - 1) max_j pre_j +
    (n - 1)(mu_dec - 1) max_j dec_j subject to stage memory (T_pre, T_dec and the quality term do
    not depend on the partition).  The decode bottleneck is enumerated over the candidate stage
    sums in increasing order (pruned once (n - 1)(mu_dec - 1) cap alone exceeds the best value),
    with a min-max DP on the prefill cost under each cap."""
    L = p.n_layers
    if p.n_stages == 1:
        return [0] * L if sum(p.mem[b] for b in bits) + p.mem_emb <= p.mem_cap else None
    cp = np.concatenate([[0.0], np.cumsum([p.l_pre[b] for b in bits])])
    cd = np.concatenate([[0.0], np.cumsum([p.l_dec[b] for b in bits])])
    cm = np.concatenate([[0.0], np.cumsum([p.mem[b] for b in bits])])
    a_pre, a_dec = p.mu_pre - 1, (p.n_tokens - 1) * (p.mu_dec - 1)
    caps = np.unique(np.concatenate([cd[i + 1:] - cd[i] for i in range(L)]))
    lo_cap = max(p.l_dec[b] for b in bits)
    caps = caps[caps >= lo_cap * (1 - 1e-12)]
    # smallest feasible cap by bisection (feasibility is monotone in the cap)
    lo, hi = 0, len(caps) - 1
    if _minmax_pre(p, cp, cd, cm, float(caps[hi]))[1] is None:
        return None
    while lo < hi:
        mid = (lo + hi) // 2
        if _minmax_pre(p, cp, cd, cm, float(caps[mid]))[1] is None:
            lo = mid + 1
        else:
            hi = mid
    if a_dec == 0:  # the decode bottleneck is not in the objective: no cap
        return _minmax_pre(p, cp, cd, cm, float(caps[-1]))[1]
    best, best_sol = math.inf, None
    for cap in caps[lo:]:
        if a_dec * cap >= best:
            break
        v, sol = _minmax_pre(p, cp, cd, cm, float(cap))
        if sol is None:
            continue
        val = a_pre * v + a_dec * float(cap)
        if val < best - 1e-15:
            best, best_sol = val, sol
    return best_sol


def adabits(p: Problem) -> list:
    """Quality-optimal bit widths that fit the total memory (latency ignored, P:252 'adabits'):
    start from each layer's best-quality width and lower, one step at a time, the layer whose
    step costs the least quality per byte saved until the model fits N devices."""
    order = sorted(p.bits_set)
    bits = [min(order, key=lambda b: (p.omega[i][b], -b)) for i in range(p.n_layers)]
    budget = p.n_stages * p.mem_cap - p.mem_emb
    while sum(p.mem[b] for b in bits) > budget:
        best, arg = math.inf, None
        for i, b in enumerate(bits):
            k = order.index(b)
            if k == 0:
                continue
            nb = order[k - 1]
            saved = p.mem[b] - p.mem[nb]
            if saved <= 0:
                continue
            cost = (p.omega[i][nb] - p.omega[i][b]) / saved
            if cost < best:
                best, arg = cost, (i, nb)
        if arg is None:
            break
        bits[arg[0]] = arg[1]
    return bits


def solve(p: Problem, max_iter: int = 200) -> Solution:
    """Bitwidth-transfer heuristic around the exact partition."""
    bits = adabits(p)
    sol = partition(p, bits)
    cur = evaluate(p, bits, sol) if sol else Solution(bits, [0] * p.n_layers, math.inf, math.inf, math.inf, False)
    log = [("adabits", cur.objective)]

    def best_move(cand_layers, top: int = 6):
        # transfers: one layer to another width, or every candidate layer of width b to width nb
        # (the paper's rules (b_st, b_pi, num_s) move several layers at once); score each on
        # the current partition (cheap), re-partition the `top` most promising exactly, keep the
        # best improving one
        cand_layers = list(cand_layers)
        moves = [[(i, nb)] for i in cand_layers for nb in p.bits_set if nb != cur.bits[i]]
        for b in set(cur.bits[i] for i in cand_layers):
            group = [i for i in cand_layers if cur.bits[i] == b]
            if len(group) > 1:
                moves += [[(i, nb) for i in group] for nb in p.bits_set if nb != b]
        scored = []
        for mv in moves:
            trial = list(cur.bits)
            for i, nb in mv:
                trial[i] = nb
            ev = evaluate(p, trial, cur.stage_of_layer)
            key = ev.objective if ev.feasible else 1e300 + sum(p.mem[b] for b in trial)
            scored.append((key, len(scored), mv))
        scored.sort()
        improved = None
        for _, _, mv in scored[:top]:
            trial = list(cur.bits)
            for i, nb in mv:
                trial[i] = nb
            s2 = partition(p, trial)
            if s2 is None:
                continue
            ev = evaluate(p, trial, s2)
            if ev.objective < (improved.objective if improved else cur.objective) - 1e-12:
                improved = ev
        return improved

    for _ in range(max_iter):
        improved = None
        if cur.feasible:
            # straggler first: the stage with the largest weighted phase cost
            pre = [0.0] * p.n_stages
            dec = [0.0] * p.n_stages
            for i, (b, j) in enumerate(zip(cur.bits, cur.stage_of_layer)):
                pre[j] += p.l_pre[b]
                dec[j] += p.l_dec[b]
            w = [(p.mu_pre - 1) * a + (p.n_tokens - 1) * (p.mu_dec - 1) * d for a, d in zip(pre, dec)]
            st = max(range(p.n_stages), key=lambda j: w[j])
            improved = best_move([i for i, j in enumerate(cur.stage_of_layer) if j == st])
        if improved is None:  # no straggler move helps (or infeasible): any single-layer transfer
            improved = best_move(range(p.n_layers))
        if improved is None:
            break
        cur = improved
        log.append(("transfer", cur.objective))
    cur.log = log
    return cur


def brute_force(p: Problem) -> Solution:
    """Every bit assignment x every contiguous partition (|BITS|^L C(L-1, N-1)): tiny instances."""
    L, N = p.n_layers, p.n_stages
    best = Solution([], [], math.inf, math.inf, math.inf, False)
    parts = []
    for cuts in itertools.combinations(range(1, L), N - 1):
        sol, s, c = [], 0, list(cuts) + [L]
        for i in range(L):
            while i >= c[s]:
                s += 1
            sol.append(s)
        parts.append(sol)
    for bits in itertools.product(p.bits_set, repeat=L):
        for sol in parts:
            ev = evaluate(p, list(bits), sol)
            if ev.objective < best.objective:
                best = ev
    return best


def layer_memory(h1: int, h2: int, bits: int, v: int, s: int, n: int, group: int = 128, bit_kv: int = 16) -> float:
    """Memory cost model: quantized linear weights (4 h1^2 + 2 h1 h2) bit/8 + scale/zero
    metadata + LayerNorm vectors, plus the KV cache 2 v (s + n) h1 bit_kv / 8 of one layer."""
    params = 4 * h1 * h1 + 2 * h1 * h2
    wbytes = 2 * params if bits == 16 else params * bits / 8 + params / group * 4
    return wbytes + 4 * h1 * 2 + 2 * v * (s + n) * h1 * bit_kv / 8
