"""Time the C2 INSERT call (reused heap, like the bench): python tools/ab_ins.py [lg] [reps]"""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
lg = int(sys.argv[1]) if len(sys.argv) > 1 else 27
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
n = 1 << lg
keys = synth.keys(n, seed=2)
q = pkg.BGPQ(capacity=n, K=1024, values=False)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
q.insert(dk); q.deletemin(n, out); torch.cuda.synchronize()
ms = []
for r in range(reps):
    e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    e[0].record(); q.insert(dk); e[1].record(); torch.cuda.synchronize()
    ms.append(e[0].elapsed_time(e[1]))
    q.deletemin(n, out); torch.cuda.synchronize()
    if r == 0:
        assert np.array_equal(out.cpu().numpy().view(np.uint32), np.sort(keys))
print("insert ms %s  min %.1f" % (" ".join("%.1f" % x for x in ms), min(ms)))
