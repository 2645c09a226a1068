#!/usr/bin/env python
"""bench_apps.py — the paper's applications on BGPQ:
time to solution of the C4 knapsack (1000 strongly correlated items) and the C5 A* (20000^2
grid, 10% / 20% obstacles), one BGPQ per GPU, at N GPUs (torchrun, NCCL between rounds:
incumbent all-reduce, size all-gather, K-batch rebalancing).

    python bench_apps.py --app knapsack|astar [--rate 0.1] [--steps 3] [--warmup 1]
    torchrun --nproc-per-node N bench_apps.py --app ...

Prints one JSON line (rank 0): time per solve (max over ranks, CUDA-synchronized wall time
around the whole multi-round search), the reached optimum, device counters, and a
cpu_baseline (the sequential oracle, 1 core) unless --no-cpu-baseline.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--app", choices=["knapsack", "astar"], default="knapsack")
    ap.add_argument("--n-items", type=int, default=1000)
    ap.add_argument("--grid", type=int, default=20000)
    ap.add_argument("--rate", type=float, default=0.1)
    ap.add_argument("--K", type=int, default=1024)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=1)
    ap.add_argument("--budget", type=int, default=64, help="DELETEMINs per CTA per round (N > 1)")
    ap.add_argument("--ctas", type=int, default=None,
                    help="CTAs of the application kernel (0: all co-resident; default: the app's DEFAULT_CTAS)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    args = ap.parse_args()

    import torch
    import synth
    from paper_conf_icpp_chenhjz21_b200 import apps

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    comm, dist = None, None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        comm = apps.TorchComm(dist, "cuda")

    if args.app == "knapsack":
        w, p, C = synth.knapsack_items(args.n_items, synth.SEEDS["C4"])
        make = lambda: apps.KnapsackSearch(w, p, C, K=args.K, capacity=1 << 29, ctas=args.ctas)
        workload = f"C4 knapsack B&B, {args.n_items} strongly correlated items, C={C}, K={args.K}"
    else:
        N = args.grid
        grid = synth.grid(N, N, args.rate, synth.SEEDS["C5"])
        dgrid = torch.from_numpy(grid).cuda()
        make = lambda: apps.AStarSearch(None, (0, 0), (N - 1, N - 1), K=args.K, capacity=1 << 30, dgrid=dgrid,
                                        ctas=args.ctas)
        workload = f"C5 A* {N}x{N} grid, {int(args.rate * 100)}% obstacles, K={args.K}"

    times, result, st_sum = [], None, None
    for i in range(args.warmup + args.steps):
        s = make()
        if rank == 0:
            s.seed()
        elif args.app == "astar":
            s.reset_g()
        torch.cuda.synchronize()
        if dist: dist.barrier()
        t0 = time.perf_counter()
        inc, rounds, moved = apps.run_search(s, comm, budget=args.budget)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        if dist:
            t = torch.tensor([dt], dtype=torch.float64, device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            dt = float(t.item())
        st = s.stats()
        if i >= args.warmup:
            times.append(dt)
            st_sum = st if st_sum is None else {k: st_sum[k] + st[k] for k in st}
        result = (inc, rounds, moved)
        s.close()
        del s
    if rank == 0:
        line = {"app": args.app, "metric": "time to solution (s)", "value": float(np.median(times)),
                "unit": "s", "higher_is_better": False, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "times_s": times, "optimum": result[0], "rounds": result[1],
                "bytes_moved_between_gpus": result[2], "dtype": "u32", "data": "synthetic",
                "config": {"workload": workload, "budget_per_round": args.budget if world > 1 else None,
                           "app_ctas": (args.ctas if args.ctas is not None else
                                        (apps.KnapsackSearch if args.app == "knapsack" else apps.AStarSearch).DEFAULT_CTAS),
                           "parallelism": f"one BGPQ per GPU x{world}, NCCL incumbent all-reduce + rebalancing"},
                "counters_per_solve": {k: v // args.steps for k, v in st_sum.items()}}
        if not args.no_cpu_baseline:
            import oracle
            t0 = time.perf_counter()
            if args.app == "knapsack":
                ref = oracle.ks_bnb(w, p, C)
                opt = ref["optimum"]
            else:
                ref = oracle.astar(grid, (0, 0), (args.grid - 1, args.grid - 1))
                opt = ref["cost"]
            line["cpu_baseline"] = {"value": time.perf_counter() - t0, "unit": "s", "cores": 1, "kind": "oracle",
                                    "sample": "the full instance, sequential best-first search (oracle/apps_oracle.cpp)",
                                    "optimum": opt, "counters": ref}
            line["parity_optimum_equal"] = opt == result[0]
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
