"""Cluster DELETEMIN engine check: python tools/ds_check.py lg K [values] [debugbits]"""
import sys, time
sys.path.insert(0, ".")
import numpy as np, torch
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
lg = int(sys.argv[1]); K = int(sys.argv[2]); vals = len(sys.argv) > 3 and sys.argv[3] == "1"
dbg = int(sys.argv[4]) if len(sys.argv) > 4 else 0
pkg.set_debug(dbg)
n = 1 << lg
keys = synth.keys(n, seed=2)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
dv = torch.arange(n, dtype=torch.int32, device="cuda") if vals else None
q = pkg.BGPQ(capacity=n, K=K, values=vals)
out = torch.empty(n, dtype=torch.int32, device="cuda")
ov = torch.empty(n, dtype=torch.int32, device="cuda") if vals else None
srt = np.sort(keys)
for rep in range(3):
    q.insert(dk, dv); torch.cuda.synchronize()
    s0 = q.stats()
    e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    e[0].record(); q.deletemin(n, out, ov); e[1].record(); torch.cuda.synchronize()
    s1 = q.stats()
    o = out.cpu().numpy().view(np.uint32)
    ok = np.array_equal(o, srt)
    bad = np.nonzero(o != srt)[0]
    print("rep", rep, "del ms %.2f" % e[0].elapsed_time(e[1]), "sorted", ok, "first bad", bad[:5], "size", q.size(),
          {k: s1[k] - s0[k] for k in ("del_ops", "del_levels", "del_cy_swap", "keys_out")}, flush=True)
    if vals:
        v = ov.cpu().numpy().view(np.uint32)
        print("  pairing", np.array_equal(keys[v], o))
