"""Quick application runs with progress output (run under `timeout`): python tools/app_debug.py ks|astar ..."""
import sys, time
sys.path.insert(0, ".")
import numpy as np, torch
import synth, oracle
from paper_conf_icpp_chenhjz21_b200 import apps
app = sys.argv[1]
if app == "ks":
    n, K, kind = int(sys.argv[2]), int(sys.argv[3]), sys.argv[4] if len(sys.argv) > 4 else "strong"
    w, p, C = synth.knapsack_items(n, synth.SEEDS["C4"] if n == 1000 else 500 + n, kind)
    s = apps.KnapsackSearch(w, p, C, K=K, capacity=1 << 27)
    s.seed(); torch.cuda.synchronize()
    print("seeded size", s.size(), flush=True)
    for r in range(int(sys.argv[5]) if len(sys.argv) > 5 else 1):
        t = time.time(); s.run(int(sys.argv[6]) if len(sys.argv) > 6 else apps.UNBOUNDED); torch.cuda.synchronize()
        print("round", r, "%.3fs" % (time.time() - t), s.stats(), "size", s.size(), flush=True)
    print("dp", oracle.ks_dp(w, p, C))
else:
    N, rate, K = int(sys.argv[2]), float(sys.argv[3]), int(sys.argv[4])
    g = synth.grid(N, N, rate, synth.SEEDS["C5"])
    s = apps.AStarSearch(g, (0, 0), (N - 1, N - 1), K=K, capacity=int(sys.argv[5]) if len(sys.argv) > 5 else 1 << 26)
    s.seed(); torch.cuda.synchronize()
    t = time.time(); s.run(); torch.cuda.synchronize()
    print("astar %.3fs" % (time.time() - t), s.stats(), flush=True)
    print("oracle", oracle.astar(g, (0, 0), (N - 1, N - 1)))
