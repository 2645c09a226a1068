"""Phase timers of the lock-ahead execution (bgpq_locks.cuh, BGPQ_DEBUG=8): average cycles
per operation for phased insert-all / deletemin-all.  python tools/prof_locks.py [lg] [K] [grid]"""
import ctypes
import os
import sys

os.environ["BGPQ_DEBUG"] = "8"
import numpy as np  # noqa: E402
import torch  # noqa: E402

sys.path.insert(0, ".")
import synth  # noqa: E402
import paper_conf_icpp_chenhjz21_b200 as pkg  # noqa: E402

NAMES = ["del_total", "del_rootacq", "del_roothold", "del_rootload", "del_twait", "del_pwait",
         "del_merge", "del_store", "del_levels(n)", "ins_total", "ins_sort", "ins_rootacq",
         "ins_roothold", "ins_pwait", "ins_merge", "ins_store", "ins_tarwait", "P_lockwait",
         "T_lockwait", "T_total", "R1_hdr+post", "R2_twait", "R3_L0pwait", "R4_L0merge", "R5_xstore+rel",
         "R6_cy+rootstore", "R7_rootrel"]

lg = int(sys.argv[1]) if len(sys.argv) > 1 else 24
K = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
grid = int(sys.argv[3]) if len(sys.argv) > 3 else 0
n = 1 << lg
keys = synth.keys(n, seed=2)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
q = pkg.BGPQ(capacity=n, K=K, values=False)
if grid:
    q.set_grid(grid)
L = pkg.lib()


def timers():
    a = np.zeros(32, np.uint64)
    L.bgpq_timers(q._h, a.ctypes.data_as(ctypes.c_void_p))
    return a[:len(NAMES)].astype(np.float64)


e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
e[0].record(); q.insert(dk); e[1].record(); torch.cuda.synchronize()
t1 = timers()
e[1].record(); q.deletemin(n, out); e[2].record(); torch.cuda.synchronize()
t2 = timers() - t1
ops = n // K
print(f"grid {q.grid()}  K {K}  n 2^{lg}  ops {ops}: insert {e[0].elapsed_time(e[1]):.1f} ms, "
      f"deletemin {e[1].elapsed_time(e[2]):.1f} ms")
print("insert phase, cycles per op:")
for i, nm in enumerate(NAMES):
    if t1[i]:
        print(f"  {nm:14s} {t1[i] / ops:10.0f}")
print("deletemin phase, cycles per op:")
for i, nm in enumerate(NAMES):
    if t2[i]:
        print(f"  {nm:14s} {t2[i] / ops:10.0f}")
print("stats", q.stats())
print("sorted", bool(np.array_equal(out.cpu().numpy().view(np.uint32), np.sort(keys))))
