"""Repeated insert-all / deletemin-all with invariant checks between: python tools/race_hunt.py lg reps"""
import sys, time, numpy as np, torch
sys.path.insert(0, ".")
import synth, oracle, paper_conf_icpp_chenhjz21_b200 as pkg
lg, reps = int(sys.argv[1]), int(sys.argv[2])
n = 1 << lg
keys = synth.keys(n, seed=2)
srt = np.sort(keys)
q = pkg.BGPQ(capacity=n, K=1024, values=False)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
bad = 0
for r in range(reps):
    q.insert(dk); torch.cuda.synchronize()
    nk, _, meta, h = q.dump()
    inv = oracle.check_invariants(q.K, q.slots() - 1, h["heapSize"], h["rootSize"], h["pbSize"], nk,
                                  pkg.to_oracle_states(meta[:, 1]))
    # multiset after the insert: root (rs) + pBuffer (ps) + nodes 2..heapSize
    K = q.K
    hs, rs, ps = h["heapSize"], h["rootSize"], h["pbSize"]
    nk2 = nk.reshape(-1, K)
    parts = [nk2[1, :rs], nk2[0, :ps]] + ([nk2[2:hs + 1].ravel()] if hs >= 2 else [])
    ms_ok = np.array_equal(np.sort(np.concatenate(parts)), srt)
    q.deletemin(n, out); torch.cuda.synchronize()
    o = out.cpu().numpy().view(np.uint32)
    ok = np.array_equal(o, srt)
    msg = ""
    if not ok:
        bad += 1
        d = np.nonzero(o != srt)[0]
        msg = f" first_bad={d[0]} n_bad={len(d)} batch={d[0] // 1024} sorted_out={bool(np.all(o[1:] >= o[:-1]))} multiset_ok={np.array_equal(np.sort(o), srt)}"
    print(f"rep {r}: insert_invariants={inv} insert_multiset={ms_ok} drain_ok={ok}{msg}", flush=True)
print("bad", bad, "of", reps)
