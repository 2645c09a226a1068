"""Per-level INSERT pipeline timers: python tools/pipe_timers.py [lg]"""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
pkg.set_debug(128)
lg = int(sys.argv[1]) if len(sys.argv) > 1 else 27
n = 1 << lg
keys = synth.keys(n, seed=2)
q = pkg.BGPQ(capacity=n, K=1024, values=False)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
e[0].record(); q.insert(dk); e[1].record(); torch.cuda.synchronize()
o = np.zeros(32, np.uint64); o[:] = q.timers()
print("insert ms %.1f  (cycles, Mcyc)" % e[0].elapsed_time(e[1]))
levels = list(range(1, 10)) + [14, 15, 16]
for idx, l in enumerate(levels):
    k = 3 * l if l < 10 else 3 * (l - 4)
    if k + 2 < 32:
        print("level %2d: take-wait %7.1f  merge %7.1f  total %7.1f" % (l, o[k] / 1e6, o[k + 1] / 1e6, o[k + 2] / 1e6))
