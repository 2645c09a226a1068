"""Pins of the application oracles (oracle/apps_oracle.cpp) — CPU only.

Knapsack: the best-first branch and bound (the method of P:477-479) against the textbook DP
and exhaustive enumeration on random instances of every generator class, plus closed forms
(everything fits; nothing fits; one item).  A*: against Dijkstra on random obstacle grids,
and the closed form on an obstacle-free grid (orthogonal 1 / diagonal 2 -> cost = Manhattan
distance, reading R24), and unreachable targets.
"""
import numpy as np
import pytest

import oracle
import synth


@pytest.mark.parametrize("kind", ["strong", "weak", "uncorrelated"])
def test_ks_bnb_vs_dp_and_brute(kind):
    for seed in range(12):
        n = 6 + seed
        w, p, C = synth.knapsack_items(n, 100 + seed, kind)
        opt = oracle.ks_dp(w, p, C)
        assert oracle.ks_brute(w, p, C) == opt
        assert oracle.ks_bnb(w, p, C)["optimum"] == opt


@pytest.mark.parametrize("kind", ["strong", "weak", "uncorrelated"])
def test_ks_bnb_vs_dp_medium(kind):
    for seed in range(4):
        w, p, C = synth.knapsack_items(60, 200 + seed, kind)
        assert oracle.ks_bnb(w, p, C)["optimum"] == oracle.ks_dp(w, p, C)


def test_ks_closed_forms():
    w = np.array([5, 3, 9, 1], np.uint32)
    p = np.array([10, 1, 7, 3], np.uint32)
    for fn in (oracle.ks_dp, oracle.ks_brute, lambda *a: oracle.ks_bnb(*a)["optimum"]):
        assert fn(w, p, int(w.sum())) == int(p.sum())      # everything fits
        assert fn(w, p, 0) == 0                              # nothing fits
        assert fn(w[:1], p[:1], 5) == 10 and fn(w[:1], p[:1], 4) == 0
        assert fn(w, p, 6) == 13                             # {5, 1}: 10 + 3


def test_ks_c4_instance_shape():
    """C4 (BASELINE configs[3]): the 1000-item instance; the DP optimum is the value every
    GPU run must reach."""
    w, p, C = synth.knapsack_items(1000, synth.SEEDS["C4"])
    assert len(w) == 1000 and w.min() >= 1 and w.max() <= 1000 and np.all(p == w + 100)
    assert oracle.ks_dp(w, p, C) == 320455


def test_astar_vs_dijkstra_random_grids():
    for seed, (N, M, rate) in enumerate([(40, 40, 0.1), (60, 35, 0.2), (80, 80, 0.3), (5, 200, 0.1), (1, 50, 0.0)]):
        g = synth.grid(N, M, rate, 300 + seed)
        a = oracle.astar(g, (0, 0), (N - 1, M - 1))
        assert a["cost"] == oracle.dijkstra(g, (0, 0), (N - 1, M - 1))


def test_astar_closed_forms():
    g = np.zeros((30, 45), np.uint8)
    for (sr, sc, tr, tc) in [(0, 0, 29, 44), (5, 7, 5, 7), (29, 0, 0, 44), (3, 40, 20, 2)]:
        want = abs(sr - tr) + abs(sc - tc)
        assert oracle.astar(g, (sr, sc), (tr, tc))["cost"] == want
        assert oracle.dijkstra(g, (sr, sc), (tr, tc)) == want
    # a wall of obstacles separating the target: unreachable for both
    g = np.zeros((10, 10), np.uint8)
    g[:, 5] = 1
    assert oracle.astar(g, (0, 0), (9, 9))["cost"] == oracle.UNREACHABLE
    assert oracle.dijkstra(g, (0, 0), (9, 9)) == oracle.UNREACHABLE
    # a diagonal squeeze: only the diagonal move (cost 2) passes between two obstacles
    g = np.zeros((2, 2), np.uint8)
    g[0, 1] = g[1, 0] = 1
    assert oracle.astar(g, (0, 0), (1, 1))["cost"] == 2


def test_astar_expands_fewer_than_grid():
    g = synth.grid(300, 300, 0.1, 5)
    a = oracle.astar(g, (0, 0), (299, 299))
    assert a["cost"] == oracle.dijkstra(g, (0, 0), (299, 299))
    assert a["expanded"] < 300 * 300 // 2  # the heuristic focuses the search
