import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
K = int(sys.argv[1]) if len(sys.argv) > 1 else 64
n = int(sys.argv[2]) if len(sys.argv) > 2 else 300 * K + 37
V = (sys.argv[3] == "v") if len(sys.argv) > 3 else True
keys = synth.keys(n, seed=3)
q = pkg.BGPQ(capacity=n, K=K, values=V)
print("grid", q.grid(), flush=True)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
dv = torch.arange(n, dtype=torch.int32, device="cuda") if V else None
q.insert(dk, dv)
torch.cuda.synchronize()
print("size", q.size(), n, q.stats(), flush=True)
ok, ov = q.deletemin(n)
torch.cuda.synchronize()
out = ok.cpu().numpy().view(np.uint32)
print("sorted ok:", np.array_equal(out, np.sort(keys)), q.size(), flush=True)
