"""Time one C2-shaped mixed call (prefill 2^23 after a drain, pairs): python tools/ab_mix.py [pairs_lg]"""
import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
npairs = 1 << (int(sys.argv[1]) if len(sys.argv) > 1 else 16)
K, P = 1024, 1 << 23
q = pkg.BGPQ(capacity=P + npairs * K + K, K=K, values=False)
pre = torch.from_numpy(synth.keys(P, seed=synth.SEEDS["C2_mix"]).view(np.int32)).cuda()
drain = torch.empty(P + npairs * K + K, dtype=torch.int32, device="cuda")
types, sizes = synth.mixed_ops(npairs, K, seed=synth.SEEDS["C2_mix"])
in_off = np.zeros(2 * npairs, np.uint64); in_off[0::2] = np.arange(npairs, dtype=np.uint64) * K
keys = torch.from_numpy(synth.keys(npairs * K, seed=synth.SEEDS["C2"]).view(np.int32)).cuda()
dt, ds = torch.from_numpy(types).cuda(), torch.from_numpy(sizes.view(np.int32)).cuda()
do = torch.from_numpy(in_off.view(np.int64)).cuda()
out = torch.empty(2 * npairs * K, dtype=torch.int32, device="cuda")
cnt = torch.zeros(2 * npairs, dtype=torch.int32, device="cuda")
ms = []
for r in range(2):
    sz = q.size()
    if sz: q.deletemin(sz, drain)
    q.insert(pre); torch.cuda.synchronize()
    e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    e[0].record(); q.run_mixed(dt, ds, do, keys, None, out, None, cnt); e[1].record(); torch.cuda.synchronize()
    ms.append(e[0].elapsed_time(e[1]))
print("mixed ms %s  min %.1f" % (" ".join("%.1f" % x for x in ms), min(ms)))
