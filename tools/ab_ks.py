"""One C4 knapsack solve on one GPU (time to solution): python tools/ab_ks.py"""
import sys, time
sys.path.insert(0, ".")
import torch, synth
import paper_conf_icpp_chenhjz21_b200.apps as apps
w, p, C = synth.knapsack_items(1000, synth.SEEDS["C4"])
s = apps.KnapsackSearch(w, p, C, K=1024, capacity=1 << 28, ctas=int(sys.argv[1]) if len(sys.argv) > 1 else None)
s.seed(); torch.cuda.synchronize()
t0 = time.perf_counter()
inc, _, _ = apps.run_search(s)
torch.cuda.synchronize()
print("knapsack s %.2f inc %d expanded %d" % (time.perf_counter() - t0, inc, s.stats().get("expanded", -1)))
