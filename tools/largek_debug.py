import sys; sys.path.insert(0, ".")
import numpy as np, torch, synth, oracle, paper_conf_icpp_chenhjz21_b200 as pkg
K = int(sys.argv[1]); nodes = int(sys.argv[2])
n = nodes * K + 37
keys = synth.keys(n, seed=synth.SEEDS["C3"] + K)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
for locks in (True, False):
    q = pkg.BGPQ(capacity=n, K=K, values=False, locks=locks)
    for rep in range(3):
        q.insert(dk)
        nk, _, meta, h = q.dump()
        seq_ok = None
        ok, _ = q.deletemin(n)
        o = ok.cpu().numpy().view(np.uint32)
        srt = np.sort(keys)
        bad = np.nonzero(o != srt)[0]
        print("locks", locks, "rep", rep, "hdr", h, "sorted", len(bad) == 0, "first bad", bad[:3], "nbad", len(bad),
              "multiset", np.array_equal(np.sort(o), srt), flush=True)
