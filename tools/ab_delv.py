"""A/B of a debug switch on the C2 DELETEMIN call: python tools/ab_del.py bits [lg] [reps]"""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
bits = int(sys.argv[1]); lg = int(sys.argv[2]) if len(sys.argv) > 2 else 27
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
n = 1 << lg
keys = synth.keys(n, seed=2)
q = pkg.BGPQ(capacity=n, K=1024, values=True)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda"); outv = torch.empty(n, dtype=torch.int32, device="cuda"); dv = torch.arange(n, dtype=torch.int32, device="cuda")
res = {0: [], bits: []}
for r in range(reps):
    for b in (0, bits):
        pkg.set_debug(b)
        q.insert(dk, dv); torch.cuda.synchronize()
        e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        e[0].record(); q.deletemin(n, out, outv); e[1].record(); torch.cuda.synchronize()
        res[b].append(e[0].elapsed_time(e[1]))
        if r == 0:
            assert np.array_equal(out.cpu().numpy().view(np.uint32), np.sort(keys)), b
pkg.set_debug(0)
for b, v in res.items():
    print("debug %d: deletemin ms %s  median %.1f" % (b, " ".join("%.1f" % x for x in v), float(np.median(v))))
