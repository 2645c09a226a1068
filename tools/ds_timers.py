"""Per-role cycle timers of the cluster DELETEMIN engine: python tools/ds_timers.py lg [K]"""
import sys
sys.path.insert(0, ".")
import numpy as np, torch
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
pkg.set_debug(1024 | (int(sys.argv[3]) if len(sys.argv) > 3 else 0))
lg = int(sys.argv[1]); K = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
n = 1 << lg
keys = synth.keys(n, seed=2)
q = pkg.BGPQ(capacity=n, K=K, values=False)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
q.insert(dk); torch.cuda.synchronize()
t0 = q.timers().astype(np.float64)
e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
e[0].record(); q.deletemin(n, out); e[1].record(); torch.cuda.synchronize()
d = q.timers().astype(np.float64) - t0
ops = n // K
print("del ms %.2f  us/op %.3f" % (e[0].elapsed_time(e[1]), e[0].elapsed_time(e[1]) * 1e3 / ops))
names = ["total", "wait-above", "wait-children/staging", "split", "wait-b", "sends"]
for r in range(5):
    print("R%d" % r, "  ".join("%s %.0f" % (names[k], d[6 * r + k] / ops) for k in range(6)), "cyc/op")
print("sorted", np.array_equal(out.cpu().numpy().view(np.uint32), np.sort(keys)))
print("walker first level (go -> release start node): %.0f cyc avg over %d" % (d[30] / max(d[31], 1), d[31]))
