"""GPU parity of the applications (csrc/bgpq_apps.cu through include/bgpq_apps.h) against the
application oracles: the knapsack optimum must equal the DP optimum (and the sequential
best-first B&B's), the A* path cost must equal the sequential A*'s (pinned by Dijkstra).
-m gpu.  (readings R23-R25.)"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    from paper_conf_icpp_chenhjz21_b200 import apps


@pytest.mark.parametrize("kind", ["strong", "weak", "uncorrelated"])
@pytest.mark.parametrize("K", [64, 1024])
def test_knapsack_small_vs_dp(kind, K):
    for seed, n in [(1, 20), (2, 40), (3, 60), (4, 90)]:
        w, p, C = synth.knapsack_items(n, 500 + seed, kind)
        s = apps.KnapsackSearch(w, p, C, K=K, capacity=1 << 22)
        s.seed()
        inc, _, _ = apps.run_search(s)
        st = s.stats()
        assert inc == oracle.ks_dp(w, p, C), (kind, K, n)
        assert st["pending"] == 0 and s.size() == 0
        assert st["inserted"] + 1 >= st["pops"]
        s.close()


def test_knapsack_c4_full():
    """C4 (BASELINE configs[3]): the 1000-item strongly correlated instance, K = 1024."""
    w, p, C = synth.knapsack_items(1000, synth.SEEDS["C4"])
    s = apps.KnapsackSearch(w, p, C, K=1024, capacity=1 << 28)
    s.seed()
    inc, _, _ = apps.run_search(s)
    assert inc == oracle.ks_dp(w, p, C) == 320455
    st = s.stats()
    print("C4 knapsack stats", st)
    assert st["pending"] == 0 and s.size() == 0
    s.close()


def _astar_case(N, M, rate, seed, K, src=None, dst=None):
    g = synth.grid(N, M, rate, seed)
    src = src or (0, 0)
    dst = dst or (N - 1, M - 1)
    s = apps.AStarSearch(g, src, dst, K=K, capacity=min(max(1 << 20, 4 * N * M), 1 << 30))
    s.seed()
    inc, _, _ = apps.run_search(s)
    want = oracle.astar(g, src, dst)["cost"]
    st = s.stats()
    s.close()
    return inc, want, st, g


@pytest.mark.parametrize("K", [64, 1024])
def test_astar_small_vs_oracle(K):
    for seed, (N, M, rate) in enumerate([(50, 50, 0.1), (64, 40, 0.2), (100, 100, 0.3), (3, 300, 0.1), (1, 1, 0.0)]):
        inc, want, st, g = _astar_case(N, M, rate, 700 + seed, K)
        assert want != oracle.UNREACHABLE
        assert inc == want, (N, M, rate)
        assert inc == oracle.dijkstra(g, (0, 0), (N - 1, M - 1))
        assert st["pending"] == 0


def test_astar_unreachable_and_interior_endpoints():
    g = np.zeros((40, 40), np.uint8)
    g[:, 20] = 1
    s = apps.AStarSearch(g, (0, 0), (39, 39), K=64, capacity=1 << 20)
    s.seed()
    inc, _, _ = apps.run_search(s)
    assert inc == apps.AStarSearch.INF                    # no path (oracle: UNREACHABLE)
    assert oracle.astar(g, (0, 0), (39, 39))["cost"] == oracle.UNREACHABLE
    s.close()
    g = synth.grid(80, 90, 0.2, 9)
    g[10, 70] = 0
    g[60, 5] = 0
    s = apps.AStarSearch(g, (10, 70), (60, 5), K=64, capacity=1 << 20)
    s.seed()
    inc, _, _ = apps.run_search(s)
    assert inc == oracle.dijkstra(g, (10, 70), (60, 5))
    s.close()


@pytest.mark.parametrize("rate", [0.1, 0.2])
def test_astar_2000_grid(rate):
    inc, want, st, _ = _astar_case(2000, 2000, rate, synth.SEEDS["C5"], 1024)
    assert inc == want
    print("A* 2000^2", rate, st)


@pytest.mark.parametrize("rate", [0.1, 0.2])
def test_astar_c5_full(rate):
    """C5 (BASELINE configs[4]): 20000 x 20000 grid at 10% / 20% obstacles, K = 1024."""
    inc, want, st, _ = _astar_case(20000, 20000, rate, synth.SEEDS["C5"], 1024)
    assert want != oracle.UNREACHABLE
    assert inc == want
    print("A* C5", rate, st)
