"""Per-stage take-wait of the INSERT level pipeline: python tools/pipe_timers.py [lg]"""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
lg = int(sys.argv[1]) if len(sys.argv) > 1 else 27
n = 1 << lg
keys = synth.keys(n, seed=2)
q = pkg.BGPQ(capacity=n, K=1024, values=False)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
q.insert(dk); q.deletemin(n, out); torch.cuda.synchronize()   # reused-heap state, like the bench
extra = int(sys.argv[2]) if len(sys.argv) > 2 else 0   # 16384: per-stage H2 request-ring waits instead of totals; 65536: merge cycles instead of take-waits (131072: the split between its barriers)
pkg.set_debug(128 | extra)
t0 = q.timers().astype(np.float64)
e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
e[0].record(); q.insert(dk); e[1].record(); torch.cuda.synchronize()
pkg.set_debug(0)
d = q.timers().astype(np.float64) - t0
ops = n // 1024
print("insert ms %.1f   (cycles per op)" % e[0].elapsed_time(e[1]))
for l in range(16):
    print("stage %2d: %s %7.0f  %s %7.0f" % (l, "split" if extra & 131072 else "merge" if extra & 65536 else "take-wait", d[l] / ops,
                                             "h2-wait" if extra & 16384 else "total", d[16 + l] / ops))
print("root H1 (minus the stage 13-15 totals): wait icons %.0f  wait sorted batch %.0f  wait slot %.0f" % ((d[29]-d[16]) / ops, (d[30]-d[16]) / ops, (d[31]-d[16]) / ops))
