"""Insert-call timing probe with a debug switch on fresh heaps: python tools/ins_probe.py bits [lg] [reps]"""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
bits = int(sys.argv[1]); lg = int(sys.argv[2]) if len(sys.argv) > 2 else 27
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
n = 1 << lg
dk = torch.from_numpy(synth.keys(n, seed=2).view(np.int32)).cuda()
res = {0: [], bits: []}
for r in range(reps):
    for b in (0, bits):
        q = pkg.BGPQ(capacity=n, K=1024, values=False)
        pkg.set_debug(b)
        torch.cuda.synchronize()
        e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        e[0].record(); q.insert(dk); e[1].record(); torch.cuda.synchronize()
        pkg.set_debug(0)
        res[b].append(e[0].elapsed_time(e[1]))
        q.close()
for b, v in res.items():
    print("debug %d: insert ms %s  min %.1f" % (b, " ".join("%.1f" % x for x in v), min(v)))
