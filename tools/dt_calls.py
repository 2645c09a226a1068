"""Deletemin-all of 2^lg keys split into `parts` calls: python tools/dt_calls.py lg parts..."""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
lg = int(sys.argv[1]); n = 1 << lg; K = 1024
keys = synth.keys(n, seed=3)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
q = pkg.BGPQ(capacity=n, K=K, values=False)
for parts in [int(x) for x in sys.argv[2:]]:
    ei = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    ei[0].record(); q.insert(dk); ei[1].record(); torch.cuda.synchronize()
    print(f"insert ms {ei[0].elapsed_time(ei[1]):.1f}", flush=True)
    e = [torch.cuda.Event(enable_timing=True) for _ in range(parts + 1)]
    step = n // parts
    e[0].record()
    for p in range(parts):
        q.deletemin(step, out[p * step:(p + 1) * step]); e[p + 1].record()
    torch.cuda.synchronize()
    ok = np.array_equal(out.cpu().numpy().view(np.uint32), np.sort(keys))
    print(f"parts={parts} total_ms={e[0].elapsed_time(e[-1]):.1f} per-part ms={[round(e[p].elapsed_time(e[p+1]),1) for p in range(parts)]} sorted={ok}", flush=True)
