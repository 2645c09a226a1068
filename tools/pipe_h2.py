"""INSERT pipeline: per-stage H2 costs (debug 262144): flow-control wait, wait_group, publish,
cycles per op: python tools/pipe_h2.py [lg]"""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
lg = int(sys.argv[1]) if len(sys.argv) > 1 else 27
n = 1 << lg
keys = synth.keys(n, seed=2)
q = pkg.BGPQ(capacity=n, K=1024, values=False)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
q.insert(dk); q.deletemin(n, out); torch.cuda.synchronize()
off = int(sys.argv[2]) if len(sys.argv) > 2 else 0   # 8: stages 8..23
pkg.set_debug(262144 | (524288 if off else 0))
t0 = q.timers()
e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
e[0].record(); q.insert(dk); e[1].record(); torch.cuda.synchronize()
pkg.set_debug(0)
d = q.timers() - t0
ops = n // 1024
print("insert ms %.1f" % e[0].elapsed_time(e[1]))
for l in range(16):
    lo, hi = int(d[l]) & 0xFFFFFFFF, int(d[l]) >> 32
    print("stage %2d: H2 flow-control %6.0f  wait_group %6.0f  publish %6.0f  cycles/op" % (l + off, lo / ops, hi / ops, d[16 + l] / ops))
