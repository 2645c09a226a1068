import sys, json, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
K = int(sys.argv[1]); lg = int(sys.argv[2]); V = sys.argv[3] == "v"
n = 1 << lg
keys = synth.keys(n, seed=2)
q = pkg.BGPQ(capacity=n, K=K, values=V, locks=(len(sys.argv) > 4 and sys.argv[4] == "locks"))
dk = torch.from_numpy(keys.view(np.int32)).cuda()
dv = torch.arange(n, dtype=torch.int32, device="cuda") if V else None
out = torch.empty(n, dtype=torch.int32, device="cuda")
e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
e[0].record(); q.insert(dk, dv); e[1].record(); t_ins_timers = None
torch.cuda.synchronize(); t1 = q.timers() if not q.locks else {}
e[1].record(); q.deletemin(n, out); e[2].record(); torch.cuda.synchronize()
t2 = q.timers() if not q.locks else {}
print("grid", q.grid(), "ins ms", e[0].elapsed_time(e[1]), "del ms", e[1].elapsed_time(e[2]))
print("ins timers (Mcyc)", {k: round(v / 1e6, 2) if "_n" not in k else v for k, v in t1.items()})
d = {k: t2[k] - t1.get(k, 0) for k in t2}
print("del timers (Mcyc)", {k: round(v / 1e6, 2) if "_n" not in k else v for k, v in d.items()})
print("stats", q.stats())
print("sorted", bool(np.array_equal(out.cpu().numpy().view(np.uint32), np.sort(keys))))
