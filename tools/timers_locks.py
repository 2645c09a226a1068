"""Phase timers of the default (lock-ahead) execution: BGPQ_DEBUG=8 python tools/timers_locks.py [lg] [K]"""
import os, sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
NAMES = ["DEL_TOTAL", "DEL_ROOTACQ", "DEL_ROOTHOLD", "DEL_ROOTLOAD", "DEL_TWAIT", "DEL_PWAIT",
         "DEL_MERGE", "DEL_STORE", "DEL_LEVELS", "INS_TOTAL", "INS_SORT", "INS_ROOTACQ",
         "INS_ROOTHOLD", "INS_PWAIT", "INS_MERGE", "INS_STORE", "INS_TARWAIT", "P_LOCKWAIT",
         "T_LOCKWAIT", "T_TOTAL", "R1", "R2", "R3", "R4", "R5", "R6", "R7"]
lg = int(sys.argv[1]) if len(sys.argv) > 1 else 24
K = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
n = 1 << lg
keys = synth.keys(n, seed=2)
q = pkg.BGPQ(capacity=n, K=K)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
def raw():
    o = np.zeros(32, np.uint64)
    pkg.lib().bgpq_timers(q._h, o.ctypes.data_as(pkg._vp))
    return o.astype(np.float64)
e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
t0 = raw()
e[0].record(); q.insert(dk); e[1].record(); torch.cuda.synchronize()
t1 = raw()
q.deletemin(n, out); e[2].record(); torch.cuda.synchronize()
t2 = raw()
nops = n // K
print("ins ms %.2f del ms %.2f  per-op us: ins %.2f del %.2f" % (e[0].elapsed_time(e[1]), e[1].elapsed_time(e[2]),
      e[0].elapsed_time(e[1]) * 1e3 / nops, e[1].elapsed_time(e[2]) * 1e3 / nops))
d = t2 - t1
print("DELETEMIN phase, cycles per op:")
for i, nm in enumerate(NAMES):
    if d[i]: print("  %-12s %10.0f" % (nm, d[i] / nops))
print("stats", q.stats())
print("sorted", bool(np.array_equal(out.cpu().numpy().view(np.uint32), np.sort(keys))))
