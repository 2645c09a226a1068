"""One C2 mixed call (prefill 2^23 from a drained heap, then 131072 (INSERT(K), DELETEMIN(K))
pairs) for ncu: python tools/mix_once.py [prefill_lg] [pairs_lg]"""
import sys
sys.path.insert(0, ".")
import numpy as np, torch
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
plg = int(sys.argv[1]) if len(sys.argv) > 1 else 23
npairs = 1 << (int(sys.argv[2]) if len(sys.argv) > 2 else 17)
K = 1024
P = 1 << plg
q = pkg.BGPQ(capacity=P + npairs * K + K, K=K, values=False)
pre = torch.from_numpy(synth.keys(P, seed=synth.SEEDS["C2_mix"]).view(np.int32)).cuda()
q.insert(pre); q.deletemin(P, torch.empty(P, dtype=torch.int32, device="cuda")); q.insert(pre)
types, sizes = synth.mixed_ops(npairs, K, seed=synth.SEEDS["C2_mix"])
in_off = np.zeros(2 * npairs, np.uint64); in_off[0::2] = np.arange(npairs, dtype=np.uint64) * K
keys = torch.from_numpy(synth.keys(npairs * K, seed=synth.SEEDS["C2"]).view(np.int32)).cuda()
out = torch.empty(2 * npairs * K, dtype=torch.int32, device="cuda")
cnt = torch.zeros(2 * npairs, dtype=torch.int32, device="cuda")
q.run_mixed(torch.from_numpy(types).cuda(), torch.from_numpy(sizes.view(np.int32)).cuda(),
            torch.from_numpy(in_off.view(np.int64)).cuda(), keys, None, out, None, cnt)
torch.cuda.synchronize()
print("mixed call done; pairs", npairs, "stats", q.stats())
