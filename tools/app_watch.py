"""Watch an application run's state words from a second stream while the kernel runs (debug)."""
import sys, time
sys.path.insert(0, ".")
import numpy as np, torch
import synth, oracle
from paper_conf_icpp_chenhjz21_b200 import apps
n, K = int(sys.argv[1]), int(sys.argv[2])
budget = int(sys.argv[3]) if len(sys.argv) > 3 else apps.UNBOUNDED
w, p, C = synth.knapsack_items(n, 500 + n, "strong")
s = apps.KnapsackSearch(w, p, C, K=K, capacity=1 << 24)
s.seed(); torch.cuda.synchronize()
s.state[apps.ST_PENDING] = s.size(); torch.cuda.synchronize()
main = torch.cuda.Stream(); side = torch.cuda.Stream()
host = torch.empty(8, dtype=torch.int64).pin_memory()
hdr = torch.empty(4, dtype=torch.int32).pin_memory()
from paper_conf_icpp_chenhjz21_b200 import lib
import ctypes
v = apps._bind()
view = (ctypes.c_byte * 64)()
with torch.cuda.stream(main):
    from paper_conf_icpp_chenhjz21_b200 import _ptr
    apps._check(v.bgpq_ks_run(s.q._h, ctypes.byref(s.ks), _ptr(s.state), budget, ctypes.c_void_p(main.cuda_stream)))
for i in range(20):
    time.sleep(0.5)
    with torch.cuda.stream(side):
        host.copy_(s.state, non_blocking=True)
    side.synchronize()
    print(i, dict(zip(apps.STATE_NAMES, host.tolist())), "done" if main.query() else "", flush=True)
    if main.query():
        break
print("dp", oracle.ks_dp(w, p, C), flush=True)
