import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, oracle, paper_conf_icpp_chenhjz21_b200 as pkg
K = int(sys.argv[1]); n = int(sys.argv[2]); V = sys.argv[3] == "v"; step = int(sys.argv[4])
seed = int(sys.argv[5]) if len(sys.argv) > 5 else 3
keys = synth.keys(n, seed=seed)
q = pkg.BGPQ(capacity=n, K=K, values=V)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
dv = torch.arange(n, dtype=torch.int32, device="cuda") if V else None
srt = np.sort(keys)
def inv():
    nk, _, meta, h = q.dump()
    st = pkg.to_oracle_states(meta[:, 1])
    return oracle.check_invariants(K, q.slots() - 1, h["heapSize"], h["rootSize"], h["pbSize"], nk, st), h
istep = int(sys.argv[6]) if len(sys.argv) > 6 else n
for off in range(0, n, istep):
    q.insert(dk[off:off+istep], None if dv is None else dv[off:off+istep])
    iv, h = inv()
    if iv[0] != 0:
        print("INSERT BAD after", off, iv, h, flush=True); break
print("after insert", inv(), q.stats(), flush=True)
pos = 0
while pos < n:
    m = min(step, n - pos)
    ok, _ = q.deletemin(m)
    out = ok.cpu().numpy().view(np.uint32)[:m]
    good = np.array_equal(out, srt[pos:pos + m])
    iv, h = inv()
    if not good or iv[0] != 0:
        print("FIRST BAD at pos", pos, "op", pos // K, "good", good, "inv", iv, h, q.stats(), flush=True)
        bad = np.nonzero(out != srt[pos:pos+m])[0]
        print(" bad idx", bad[:10], out[bad[:5]], srt[pos + bad[:5]])
        break
    pos += m
print("done pos", pos, flush=True)
