"""A/B of debug switches on the C2 phased step, same box: python tools/ab_insert.py bitsA bitsB [reps]"""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
n, K = 1 << 27, 1024
keys = synth.keys(n, seed=2)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
q = pkg.BGPQ(capacity=n, K=K, values=False)
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
for r in range(reps):
    for bits in (int(sys.argv[1]), int(sys.argv[2])):
        pkg.set_debug(bits)
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record(); q.insert(dk); e[1].record(); q.deletemin(n, out); e[2].record(); torch.cuda.synchronize()
        print("bits %5d  insert %.1f ms  deletemin %.1f ms" % (bits, e[0].elapsed_time(e[1]), e[1].elapsed_time(e[2])), flush=True)
pkg.set_debug(0)
