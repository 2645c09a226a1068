import sys; sys.path.insert(0, ".")
import numpy as np, torch, synth, oracle, paper_conf_icpp_chenhjz21_b200 as pkg
K = int(sys.argv[1]); nodes = int(sys.argv[2]); reps = int(sys.argv[3])
n = nodes * K + 37
keys = synth.keys(n, seed=synth.SEEDS["C3"] + K)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
q = pkg.BGPQ(capacity=n, K=K, values=False)
seq = oracle.SeqBGPQ(K, q.slots() - 1)
for rep in range(reps):
    q.insert(dk)
    for off in range(0, n, K):
        seq.insert(keys[off:min(off + K, n)])
    nk, _, meta, h = q.dump()
    sk, _, sst = seq.dump()
    sh = seq.header()
    bad = [i for i in range(2, h["heapSize"] + 1) if not np.array_equal(nk[i], sk[i])]
    rb = not np.array_equal(nk[1, :h["rootSize"]], sk[1, :sh["rootSize"]])
    pbb = not np.array_equal(nk[0, :h["pbSize"]], sk[0, :sh["pbSize"]])
    print("rep", rep, "hdr", h, "seq", sh, "bad nodes", bad[:10], len(bad), "root bad", rb, "pb bad", pbb, flush=True)
    if bad:
        i = bad[0]
        g, s_ = nk[i], sk[i]
        d = np.nonzero(g != s_)[0]
        print("  node", i, "state", meta[i], "diff pos", d[:8], len(d), "gpu vals", g[d[:4]], "seq", s_[d[:4]], flush=True)
        # where did the GPU's wrong keys come from?
        print("  gpu node sorted", bool(np.all(g[1:] >= g[:-1])), "gpu keys in input", np.isin(g[d[:8]], keys).tolist(), flush=True)
    q.deletemin(n)
    out = np.concatenate([seq.deletemin(K)[0] for _ in range((n + K - 1) // K)])
    torch.cuda.synchronize()
