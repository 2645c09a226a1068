import sys; sys.path.insert(0, ".")
import numpy as np, torch, synth, paper_conf_icpp_chenhjz21_b200 as pkg
K = int(sys.argv[1]); nodes = int(sys.argv[2]); bits = int(sys.argv[3]); reps = int(sys.argv[4])
pkg.set_debug(bits)
n = nodes * K + 37
keys = synth.keys(n, seed=synth.SEEDS["C3"] + K)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
srt = np.sort(keys)
q = pkg.BGPQ(capacity=n, K=K, values=False)
bad = 0
for rep in range(reps):
    q.insert(dk)
    nk, _, meta, h = q.dump()
    hs, rs, ps = h["heapSize"], h["rootSize"], h["pbSize"]
    parts = [nk[1, :rs], nk[0, :ps]] + ([nk[2:hs + 1].ravel()] if hs >= 2 else [])
    ms_ok = np.array_equal(np.sort(np.concatenate(parts)), srt)
    ok, _ = q.deletemin(n)
    o = ok.cpu().numpy().view(np.uint32)
    if not (ms_ok and np.array_equal(o, srt)):
        bad += 1
        print("rep", rep, "insert multiset ok", ms_ok, "drain ok", np.array_equal(o, srt), flush=True)
print("K", K, "bits", bits, "bad reps", bad, "of", reps, flush=True)
