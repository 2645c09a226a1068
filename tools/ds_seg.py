"""R1's per-segment cycles per op on a C2-size DELETEMIN (debug 2097152): python tools/ds_seg.py [lg]"""
import sys
sys.path.insert(0, ".")
import numpy as np, torch
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
lg = int(sys.argv[1]) if len(sys.argv) > 1 else 27
n = 1 << lg
keys = synth.keys(n, seed=2)
q = pkg.BGPQ(capacity=n, K=1024, values=False)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
q.insert(dk); q.deletemin(n, out); q.insert(dk); torch.cuda.synchronize()
pkg.set_debug(2097152)
t0 = q.timers().astype(np.float64)
q.deletemin(n, out); torch.cuda.synchronize()
pkg.set_debug(0)
d = q.timers().astype(np.float64) - t0
ops = n // 1024
names = ["recv a", "children pend", "decide+send a", "barrier 1", "split", "post-split bookkeeping",
         "push up", "send b", "recv b", "barrier 2", "", "", "", "", "", "loop/other"]
for k in range(16):
    if names[k]:
        print("%-24s %7.0f" % (names[k], d[k] / ops))
print("sum %.0f cycles per op" % (d[:16].sum() / ops))
