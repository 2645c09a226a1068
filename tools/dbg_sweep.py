import sys, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
for V in (False, True):
    for K in (64, 128, 256, 512, 1024):
        for mult in (40, 300, 3000):
            n = mult * K + 37
            keys = synth.keys(n, seed=3)
            q = pkg.BGPQ(capacity=n, K=K, values=V)
            dk = torch.from_numpy(keys.view(np.int32)).cuda()
            dv = torch.arange(n, dtype=torch.int32, device="cuda") if V else None
            q.insert(dk, dv)
            sz = q.size()
            ok, ov = q.deletemin(n)
            out = ok.cpu().numpy().view(np.uint32)
            srt = np.sort(keys)
            good = np.array_equal(out, srt)
            bad = np.nonzero(out != srt)[0]
            print(f"V={V} K={K} n={n} size={sz} ok={good} first_bad={bad[:3]} nbad={len(bad)} st={q.stats()['marked']}", flush=True)
            q.close()
