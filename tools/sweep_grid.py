"""Grid-size sweep of the paper-literal (locks) execution: phased insert / deletemin times
at 2^lg keys (default 2^24), K = 1024, keys only.  python tools/sweep_grid.py [lg]"""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import synth  # noqa: E402
import paper_conf_icpp_chenhjz21_b200 as pkg  # noqa: E402

lg = int(sys.argv[1]) if len(sys.argv) > 1 else 24
K = 1024
n = 1 << lg
keys = synth.keys(n, seed=2)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
out = torch.empty(n, dtype=torch.int32, device="cuda")
srt = torch.sort(dk.to(torch.int64) & 0xFFFFFFFF)[0]
for grid in (4, 8, 16, 32, 64, 148):
    q = pkg.BGPQ(capacity=n, K=K, values=False, locks=True)
    q.set_grid(grid)
    e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
    e[0].record(); q.insert(dk); e[1].record(); q.deletemin(n, out); e[2].record()
    torch.cuda.synchronize()
    ok = torch.equal(out.to(torch.int64) & 0xFFFFFFFF, srt)
    print(f"grid {grid:4d}: insert {e[0].elapsed_time(e[1]):8.1f} ms  deletemin {e[1].elapsed_time(e[2]):8.1f} ms"
          f"  sorted={ok}  spins={q.stats()['root_spins']}", flush=True)
    q.close()
