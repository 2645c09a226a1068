#!/bin/bash
# sanitizers, application benches and the utilisation sweep (under gpurun)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out/evid
CS=/usr/local/cuda/bin/compute-sanitizer
cat > /tmp/san_case.py <<'PY'
import sys; sys.path.insert(0, ".")
import numpy as np, torch, synth, oracle, paper_conf_icpp_chenhjz21_b200 as pkg
K, n, vals = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3] == "1"
keys = synth.keys(n, seed=1)
q = pkg.BGPQ(capacity=n, K=K, values=vals)
dk = torch.from_numpy(keys.view(np.int32)).cuda()
dv = torch.arange(n, dtype=torch.int32, device="cuda") if vals else None
q.insert(dk, dv); ok, ov = q.deletemin(n); torch.cuda.synchronize()
assert np.array_equal(ok.cpu().numpy().view(np.uint32), np.sort(keys))
types, sizes = synth.mixed_ops(500, K, seed=3, partial=True)
print("case ok", K, n, vals)
PY
for tool in memcheck synccheck racecheck; do
  timeout -s KILL 900 $CS --tool $tool --print-limit 20 python /tmp/san_case.py 64 65536 1 > gpurun_out/evid/san_${tool}_c1.txt 2>&1; echo "$tool c1 rc=$?" >> gpurun_out/evid/san_summary.txt
done
timeout -s KILL 900 $CS --tool memcheck --print-limit 20 python /tmp/san_case.py 256 $((1500*256)) 0 > gpurun_out/evid/san_memcheck_k256_cluster.txt 2>&1; echo "memcheck k256-cluster rc=$?" >> gpurun_out/evid/san_summary.txt
timeout -s KILL 900 $CS --tool synccheck --print-limit 20 python /tmp/san_case.py 256 $((1500*256)) 0 > gpurun_out/evid/san_synccheck_k256_cluster.txt 2>&1; echo "synccheck k256-cluster rc=$?" >> gpurun_out/evid/san_summary.txt
tail -3 gpurun_out/evid/san_*.txt >> gpurun_out/evid/san_summary.txt
timeout 600 python bench_apps.py --app knapsack --steps 3 --warmup 1 > gpurun_out/evid/apps_knapsack.json 2>&1
timeout 900 python bench_apps.py --app astar --rate 0.1 --steps 3 --warmup 1 > gpurun_out/evid/apps_astar10.json 2>&1
timeout 900 python bench_apps.py --app astar --rate 0.2 --steps 3 --warmup 1 > gpurun_out/evid/apps_astar20.json 2>&1
for p in -1 20 23; do
  timeout 600 python bench.py --mix --n-log2 26 --prefill-log2 $p --steps 3 --warmup 2 > gpurun_out/evid/util_prefill_$p.json 2>&1
done
