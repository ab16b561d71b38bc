"""Host plan helpers: exact min-max contiguous partition (eqs. 15-16), pinned by brute force."""
import itertools
import random

from paper_conf_cluster_zhaowplw25_b200 import plan as PL


def brute(costs, P):
    L = len(costs)
    best = None
    for cuts in itertools.combinations(range(1, L), P - 1):
        b = (0,) + cuts + (L,)
        m = max(sum(costs[b[i]:b[i + 1]]) for i in range(P))
        best = m if best is None else min(best, m)
    return best


def test_partition_matches_bruteforce():
    rnd = random.Random(5)
    for _ in range(200):
        L = rnd.randint(1, 9)
        P = rnd.randint(1, L)
        costs = [rnd.choice([1.0, 1.3, 2.6, 5.0]) * rnd.random() for _ in range(L)]
        sol = PL.partition_layers(costs, P)
        assert sol[0] == 0 and sol[-1] == P - 1
        assert all(b - a in (0, 1) for a, b in zip(sol, sol[1:]))  # contiguous, non-empty
        got = max(PL.stage_costs(costs, sol))
        assert abs(got - brute(costs, P)) < 1e-12


def test_uneven_partition_for_mixed_bits():
    # OPT-66B mixed bits: cheaper (low-bit) layers pack more per stage -> uneven stage sizes
    bits = [3] * 16 + [16] * 16 + [4] * 16 + [8] * 16
    c = PL.phase_costs(bits, 9216, 36864, B=256, eta=8, xi=32, s=512, n_dec=128)
    sol = PL.partition_layers(c, 8)
    sizes = [sol.count(s) for s in range(8)]
    assert sum(sizes) == 64 and len(set(sizes)) > 1


def test_layer_bytes_matches_paper_memory_model():
    # P:160 codes term + group metadata
    h1, h2 = 9216, 36864
    assert PL.layer_bytes(h1, h2, 16) == 2 * (4 * h1 * h1 + 2 * h1 * h2)
    assert PL.layer_bytes(h1, h2, 4) == (4 * h1 * h1 + 2 * h1 * h2) // 2 + (4 * h1 * h1 + 2 * h1 * h2) // 128 * 4


def test_latency_model_eq4():
    # all stages + (mu - 1) x slowest
    assert PL.pipeline_latency_model([1, 2, 3], [0.1, 0.2, 0.3], 4, 3, 2) == (6 + 3 * 3) + 2 * (0.6 + 2 * 0.3)
