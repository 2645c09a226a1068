#!/bin/bash
# Late round-2 evidence (under gpurun): C3 x K sweep, utilisation sweep (mix at three prefills),
# application benches, w = 8 bench
cd "$GRAFT_REPO_ROOT"; O=${OUT:-gpurun_out/late2}; mkdir -p $O
: > $O/sweep_c3.jsonl
for d in uniform ascending descending gaussian; do
  for k in 128 256 512 1024 2048 4096; do
    timeout 300 python bench.py --n-log2 26 --K $k --dist $d --steps 3 --warmup 2 --no-cpu-baseline --no-e2e --no-mix 2>/dev/null | tail -1 >> $O/sweep_c3.jsonl
  done
done
echo "c3 lines $(wc -l < $O/sweep_c3.jsonl)"
for p in -1 20 23; do
  timeout 600 python bench.py --mix --n-log2 26 --prefill-log2 $p --steps 3 --warmup 2 > $O/util_prefill_$p.json 2>&1
done
echo "util done"
timeout 900 python bench.py --steps 3 --warmup 3 --values --no-cpu-baseline > $O/bench_w8.log 2>&1; echo "w8 rc=$?"
timeout 600 python bench_apps.py --app knapsack --steps 3 --warmup 1 > $O/apps_knapsack.json 2>&1; echo "ks rc=$?"
timeout 900 python bench_apps.py --app astar --rate 0.1 --steps 3 --warmup 1 > $O/apps_astar10.json 2>&1; echo "a10 rc=$?"
timeout 900 python bench_apps.py --app astar --rate 0.2 --steps 3 --warmup 1 > $O/apps_astar20.json 2>&1; echo "a20 rc=$?"
