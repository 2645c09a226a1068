"""Quick check of the deletemin execution: phased insert-all / deletemin-all vs np.sort.
python tools/dt_quick.py [log2_n K [v]]"""
import sys
import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
import paper_conf_icpp_chenhjz21_b200 as pkg  # noqa: E402

cases = [(1 << 12, 64, False), (1 << 14, 64, True), (1 << 16, 64, False), (100_003, 128, True),
         (1 << 18, 1024, False), (1 << 20, 1024, True), (1 << 22, 1024, False), (1 << 24, 1024, False)]
if len(sys.argv) > 1:
    cases = [(1 << int(sys.argv[1]), int(sys.argv[2]), len(sys.argv) > 3)]
for n, K, V in cases:
    keys = synth.keys(n, seed=3)
    q = pkg.BGPQ(capacity=n, K=K, values=V)
    dk = torch.from_numpy(keys.view(np.int32)).cuda()
    dv = torch.arange(n, dtype=torch.int32, device="cuda") if V else None
    q.insert(dk, dv)
    torch.cuda.synchronize()
    out = torch.empty(n, dtype=torch.int32, device="cuda")
    outv = torch.empty(n, dtype=torch.int32, device="cuda") if V else None
    e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    # two calls: half, then the rest (exercises the call-boundary write-back)
    h = (n // 2 // K) * K
    e[0].record()
    q.deletemin(h, out[:h], outv[:h] if V else None)
    q.deletemin(n - h, out[h:], outv[h:] if V else None)
    e[1].record()
    torch.cuda.synchronize()
    o = out.cpu().numpy().view(np.uint32)
    ok = np.array_equal(o, np.sort(keys))
    okv = True
    if V:
        ov = outv.cpu().numpy().view(np.uint32)
        okv = np.array_equal(keys[ov], o) and np.array_equal(np.sort(ov), np.arange(n, dtype=np.uint32))
    ms = e[0].elapsed_time(e[1])
    print(f"n={n} K={K} V={V}: sorted={ok} values={okv} size_after={q.size()} del_ms={ms:.2f} "
          f"us/op={ms * 1e3 / max(1, n // K):.2f} stats={q.stats()}", flush=True)
    q.close()
