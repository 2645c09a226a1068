import sys, ctypes, numpy as np, torch
sys.path.insert(0, ".")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
L = pkg.lib()
for trial in range(int(sys.argv[4]) if len(sys.argv) > 4 else 10):
    K = int(sys.argv[1]); n = int(sys.argv[2]); V = sys.argv[3] == "v"
    keys = synth.keys(n, seed=3 + trial)
    q = pkg.BGPQ(capacity=n, K=K, values=V)
    dk = torch.from_numpy(keys.view(np.int32)).cuda()
    q.insert(dk)
    rec = np.zeros(4, np.uint32)
    L.bgpq_debug_record(q._h, rec.ctypes.data_as(ctypes.c_void_p))
    ok, _ = q.deletemin(n)
    out = ok.cpu().numpy().view(np.uint32)
    rec2 = np.zeros(4, np.uint32)
    L.bgpq_debug_record(q._h, rec2.ctypes.data_as(ctypes.c_void_p))
    srt = np.sort(keys)
    bad = np.nonzero(out != srt)[0]
    print(f"trial {trial} ok={len(bad)==0} first_bad_op={bad[0]//K if len(bad) else -1} ins_rec={rec} del_rec(op+1,node,kind,hs)={rec2}", flush=True)
    q.close()
