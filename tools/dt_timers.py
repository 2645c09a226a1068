"""Top-CTA timers of the deletemin execution: python tools/dt_timers.py [lg] [K]"""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
pkg.set_debug(8)
lg = int(sys.argv[1]) if len(sys.argv) > 1 else 24
K = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
n = 1 << lg
keys = synth.keys(n, seed=2)
q = pkg.BGPQ(capacity=n, K=K, values=False)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
def raw():
    o = np.zeros(32, np.uint64)
    o[:] = q.timers()
    return o.astype(np.float64)
q.insert(dk); torch.cuda.synchronize()
t1 = raw()
e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
e[0].record(); q.deletemin(n, out); e[1].record(); torch.cuda.synchronize()
d = raw() - t1
slots = max(d[21], 1)
print("del ms %.2f us/op %.2f slots %d conflicts %d" % (e[0].elapsed_time(e[1]), e[0].elapsed_time(e[1]) * 1e3 / (n // K), d[21], d[22]))
for i, nm in enumerate(["plan/decisions", "phaseA(wait)", "G2 wait|flush", "data waits", "phaseB"]):
    print("  %-14s %8.0f cyc/slot" % (nm, d[16 + i] / slots))
print("  helper lock wait %8.0f cyc/slot" % (d[23] / slots))
print("  G0 out+merge %8.0f  G1 merge %8.0f  G2 wait+merge %8.0f  rounds/slot %.2f" % (d[24] / slots, d[25] / slots, d[26] / slots, d[27] / slots))
print("  stage cycles/slot:", {nm: round(d[k] / slots) for k, nm in enumerate(["fast:loads+tests", "fast:lag commit", "fast:rest", "plan:to refill", "plan:refill enq", "plan:m1+stage enq", "plan:writeback", "B waits", "-", "-", "-", "-"])})
print("sorted", bool(np.array_equal(out.cpu().numpy().view(np.uint32), np.sort(keys))))
