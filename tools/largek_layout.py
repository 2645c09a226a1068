import sys; sys.path.insert(0, ".")
import numpy as np, torch, synth, oracle, paper_conf_icpp_chenhjz21_b200 as pkg
K = int(sys.argv[1]); nodes = int(sys.argv[2]); reps = int(sys.argv[3])
n = nodes * K
keys = synth.keys(n, seed=5)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
for rep in range(reps):
    q = pkg.BGPQ(capacity=2 * n, K=K, values=False)
    seq = oracle.SeqBGPQ(K, q.slots() - 1)
    for r2 in range(2):
        q.insert(dk)
        for off in range(0, n, K):
            seq.insert(keys[off:off + K])
        nk, _, meta, h = q.dump()
        sk, _, sst = seq.dump()
        sh = seq.header()
        bad = [i for i in range(1, h["heapSize"] + 1) if not np.array_equal(nk[i, :K if i > 1 else h["rootSize"]], sk[i, :K if i > 1 else sh["rootSize"]])]
        print("rep", rep, "call", r2, "hdr", h, "seq", sh, "bad nodes", bad[:10], len(bad), flush=True)
        if bad:
            i = bad[0]
            g, s_ = nk[i], sk[i]
            print("  node", i, "gpu min/max", g.min(), g.max(), "seq", s_.min(), s_.max(), "sorted gpu", bool(np.all(g[1:] >= g[:-1])),
                  "diff pos", np.nonzero(g != s_)[0][:8], flush=True)
    q.close()
