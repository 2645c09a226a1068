"""Per-role cycle timers of the cluster engine on a mixed call of (INSERT(K), DELETEMIN(K))
pairs: python tools/dsm_timers.py [prefill_lg] [pairs] [K] [extra debug bits]"""
import sys
sys.path.insert(0, ".")
import numpy as np, torch
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
plg = int(sys.argv[1]) if len(sys.argv) > 1 else 23
npairs = int(sys.argv[2]) if len(sys.argv) > 2 else 16384
K = int(sys.argv[3]) if len(sys.argv) > 3 else 1024
extra = int(sys.argv[4]) if len(sys.argv) > 4 else 0
P = 1 << plg
q = pkg.BGPQ(capacity=P + npairs * K + K, K=K, values=False)
pre = torch.from_numpy(synth.keys(P, seed=22).view(np.int32)).cuda()
q.insert(pre); q.deletemin(P, torch.empty(P, dtype=torch.int32, device="cuda")); q.insert(pre)
types, sizes = synth.mixed_ops(npairs, K, seed=22)
in_off = np.zeros(2 * npairs, np.uint64); in_off[0::2] = np.arange(npairs, dtype=np.uint64) * K
keys = torch.from_numpy(synth.keys(npairs * K, seed=2).view(np.int32)).cuda()
dt = torch.from_numpy(types).cuda(); ds = torch.from_numpy(sizes.view(np.int32)).cuda()
do = torch.from_numpy(in_off.view(np.int64)).cuda()
out = torch.empty(2 * npairs * K, dtype=torch.int32, device="cuda")
cnt = torch.zeros(2 * npairs, dtype=torch.int32, device="cuda")
torch.cuda.synchronize()
pkg.set_debug(1024 | extra)
t0 = q.timers().astype(np.float64)
st0 = q.stats()
e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
e[0].record(); q.run_mixed(dt, ds, do, keys, None, out, None, cnt); e[1].record(); torch.cuda.synchronize()
pkg.set_debug(0)
d = q.timers().astype(np.float64) - t0
st = {k: v - st0[k] for k, v in q.stats().items()}
print("mixed ms %.2f  us/pair %.3f" % (e[0].elapsed_time(e[1]), e[0].elapsed_time(e[1]) * 1e3 / npairs))
names = ["total", "wait-above", "wait-children/staging", "split", "wait-b", "sends"]
for r in range(5):
    print("R%d" % r, "  ".join("%s %.0f" % (names[k], d[6 * r + k] / npairs) for k in range(6)), "cyc/pair")
print("stats per pair:", {k: round(v / npairs, 3) for k, v in st.items() if v})
print("walker first level (go -> release start node): %.0f cyc avg over %d" % (d[30] / max(d[31], 1), d[31]))
