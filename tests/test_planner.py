"""f1 — planner (eqs. 4-16) and latency cost model, host-side.

The planner's exact partition is pinned against brute force over every contiguous partition, the
bitwidth-transfer heuristic against brute force over every (bits, partition) pair on tiny
instances, and its limits against closed forms (theta = 0 -> fastest widths that fit; huge theta
-> highest quality that fits; memory caps respected).  The cost model recovers known
coefficients from synthetic samples exactly.
"""
from __future__ import annotations

import itertools
import math
import random

import numpy as np
import pytest

from paper_conf_cluster_zhaowplw25_b200 import costmodel as CM
from paper_conf_cluster_zhaowplw25_b200 import planner as PL


def _problem(L=6, N=2, theta=1.0, B=8, eta=2, xi=4, n=9, mem_cap=1e9, seed=0, bits_set=(3, 4, 8, 16)):
    rng = random.Random(seed)
    l_pre = {3: 1.10, 4: 1.05, 8: 1.02, 16: 1.00}
    l_dec = {3: 0.21, 4: 0.26, 8: 0.50, 16: 1.00}
    mem = {3: 0.41, 4: 0.53, 8: 1.03, 16: 2.0}
    omega = [{3: 4.6 * a, 4: a, 8: a / 289.0, 16: 0.0} for a in (rng.uniform(0.5, 2.0) for _ in range(L))]
    return PL.Problem(L, N, tuple(bits_set), {b: l_pre[b] for b in bits_set}, {b: l_dec[b] for b in bits_set},
                      {b: mem[b] for b in bits_set}, omega, theta, B, eta, xi, n, mem_cap)


def _all_partitions(L, N):
    for cuts in itertools.combinations(range(1, L), N - 1):
        c, s, sol = list(cuts) + [L], 0, []
        for i in range(L):
            while i >= c[s]:
                s += 1
            sol.append(s)
        yield sol


@pytest.mark.parametrize("seed", range(6))
def test_partition_is_exact(seed):
    rng = random.Random(100 + seed)
    p = _problem(L=7, N=3, seed=seed, mem_cap=rng.choice([1e9, 3.0, 2.2]))
    bits = [rng.choice((3, 4, 8, 16)) for _ in range(p.n_layers)]
    sol = PL.partition(p, bits)
    best = min((PL.evaluate(p, bits, s).objective for s in _all_partitions(p.n_layers, p.n_stages)), default=math.inf)
    if sol is None:
        assert best == math.inf
    else:
        assert PL.evaluate(p, bits, sol).objective == pytest.approx(best, rel=1e-12)


@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("theta", [0.0, 0.05, 1.0])
def test_heuristic_matches_brute_force_on_tiny_instances(seed, theta):
    p = _problem(L=5, N=2, theta=theta, seed=seed, mem_cap=2.6)
    bf = PL.brute_force(p)
    h = PL.solve(p)
    assert h.feasible and bf.feasible
    assert h.objective <= bf.objective * (1 + 0.03) + 1e-12  # near-optimal ("near-optimal")
    assert h.objective >= bf.objective - 1e-12


def test_theta_limits_and_memory():
    # theta = 0: latency only -> the fastest decode width everywhere (memory permitting)
    p = _problem(L=6, N=2, theta=0.0, mem_cap=1e9)
    assert set(PL.solve(p).bits) == {3}
    # huge theta: quality first -> fp16 (omega = 0) when it fits ...
    p = _problem(L=6, N=2, theta=1e6, mem_cap=1e9)
    assert set(PL.solve(p).bits) == {16}
    # ... and the best quality that fits when it does not: 6 layers x 2.0 > 2 x 5.0
    p = _problem(L=6, N=2, theta=1e6, mem_cap=5.0)
    s = PL.solve(p)
    assert s.feasible and sum(p.mem[b] for b in s.bits) <= 2 * 5.0
    assert all(sum(p.mem[b] for b, j in zip(s.bits, s.stage_of_layer) if j == st) <= 5.0 for st in range(2))


def test_evaluate_matches_eq4_by_hand():
    p = _problem(L=2, N=2, theta=0.5, B=8, eta=2, xi=4, n=9)
    ev = PL.evaluate(p, [3, 16], [0, 1])
    mu_pre, mu_dec = 4, 2
    pre = [1.10, 1.00]
    dec = [0.21, 1.00]
    lat = (mu_pre - 1) * max(pre) + sum(pre) + (9 - 1) * ((mu_dec - 1) * max(dec) + sum(dec))
    assert ev.latency == pytest.approx(lat, rel=1e-15)
    assert ev.objective == pytest.approx(lat + 0.5 * (p.omega[0][3] + p.omega[1][16]), rel=1e-15)
    assert PL.evaluate(p, [3, 16], [0, 0]).objective == math.inf  # stage 1 empty (eq. 15)


def test_costmodel_recovers_coefficients():
    rng = np.random.default_rng(0)
    true_pre, true_dec = [1e-4, 2e-5, 3e-7, 4e-8, 1e-12], [5e-5, 1e-6, 0.0, 0.0]
    samples = []
    for b in (4, 8):
        for v, s in ((1, 128), (2, 256), (4, 512), (8, 512), (8, 1024), (3, 300)):
            samples.append({"phase": "pre", "bits": b, "v": v, "s": s, "ctx": s,
                            "t": float(CM.pre_features(v, s) @ np.array(true_pre)) * (b / 4)})
        for v, c in ((1, 256), (8, 512), (16, 384), (32, 640), (4, 100)):
            samples.append({"phase": "dec", "bits": b, "v": v, "s": c, "ctx": c,
                            "t": float(CM.dec_features(v, c) @ np.array(true_dec)) * (b / 4)})
    m = CM.LatencyModel.fit(samples)
    assert max(m.errors(samples)) < 1e-9
    assert m.t_pre(8, 5, 700) == pytest.approx(2 * float(CM.pre_features(5, 700) @ np.array(true_pre)), rel=1e-9)
    m2 = CM.LatencyModel.from_json(m.to_json())
    assert m2.t_dec(4, 7, 333) == pytest.approx(m.t_dec(4, 7, 333), rel=1e-15)
    del rng


def test_layer_memory_matches_p160():
    # (4 h1^2 + 2 h1 h2) bit/8 + metadata + 4 h1 LN (fp16) + KV 2 v (s+n) h1 * 2 B
    h1, h2 = 768, 3072
    params = 4 * h1 * h1 + 2 * h1 * h2
    assert PL.layer_memory(h1, h2, 4, 0, 0, 0) == params / 2 + params / 128 * 4 + 8 * h1
    assert PL.layer_memory(h1, h2, 16, 2, 10, 6) == 2 * params + 8 * h1 + 2 * 2 * 16 * h1 * 2
