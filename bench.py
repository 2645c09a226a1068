#!/usr/bin/env python
"""bench.py — BGPQ hot-path benchmark (BASELINE.json metric) on B200.

Default workload (config C2, phased; BASELINE.json configs[1]): insert 2^27 uniform uint32
keys into an empty BGPQ with K = 1024 (keys only, w = 4 B), then DELETEMIN all of them.
One step = one pass of the whole hot path (all INSERT batches then all DELETEMIN batches).
Metric: keys/s = keys / (t_insert + t_deletemin), device-timed with CUDA events.  The same
line carries the C2 50/50 concurrent mix (the other half of configs[1]) as "mix" (skip with
--no-mix), the e2e number through the host-buffer C ABI, the roofline of the dominant kernel
with its critical-path bound, and the CPU baselines.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--values] [--dist uniform|ascending|descending|gaussian] [--K 1024]
                    [--n-log2 27] [--mix] [--mode default|locks]

Multi-GPU: the linearizable heap does not shard: N ranks run N independent
replicas ("scaling": "weak"), timed as the max over ranks.
--impl reference runs the CPU oracle (oracle/, std::multiset) on a bounded sample of the
same workload on the host cores (rank 0 only).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import platform
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "keys/sec insert & deletemin (128M keys, K=1024) on 1 B200; % HBM roofline"
SM_MHZ = 1965.0  # B200 max SM clock (MEASURED_PEAKS.json sm_max_mhz); cycle <-> time conversions
# Critical-path floor of the DELETEMIN chain: every DELETEMIN's depth-0 step
# reads the node the previous one's depth-1 step produced (Alg.3 l.10-15), so a drain is a
# chain of one link per batch; a link needs at least one 2K-entry SORT_SPLIT on one SM
# (bitonic split, 920 cycles keys-only at K = 1024, profiles/r1/micro_merge.txt) plus the
# decision on its result (~680 cycles: co-rank of the next path node + two shared-memory
# hand-offs) = 1,600 cycles per batch.
CHAIN_FLOOR_CYCLES = {1024: 1600}


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, burst copy)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""
    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines: list[str] = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        self.proc.wait()
        sm, smax, reasons = [], [], set()
        names = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0])); smax.append(float(f[1]))
            except ValueError:
                continue
            for nm, v in zip(names, f[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None,
                "sm_max_mhz": max(smax) if smax else None,
                "samples": len(sm), "reasons": sorted(reasons)}


def byte_model(st: dict, K: int, w: int) -> dict:
    """Algorithmic bytes of Alg.1-3, from device counters.
    INSERT: K·w input read + 2K·w per intermediate path level + K·w target write.
    DELETEMIN: K·w output + K·w read of the last node + 4K·w per heapify level + K·w final
    write of the node the sinking keys stop in.
    B_eff: B_alg minus the node traffic of INSERT levels whose SORT_SPLIT is a no-op (the
    cached-min/max fast path moves nothing there)."""
    ins = st["ins_ops"] * K * w + st["ins_levels"] * 2 * K * w + st["ins_heapify_ops"] * K * w
    dele = st["keys_out"] * w + st["del_refill_ops"] * K * w + st["del_levels"] * 4 * K * w \
        + st["del_refill_ops"] * K * w
    skipped = st["ins_noop"] * 2 * K * w
    return {"insert": ins, "deletemin": dele, "total": ins + dele, "insert_noop_skipped": skipped,
            "insert_eff": ins - skipped, "total_eff": ins + dele - skipped}


def max_over_ranks(ms: float, dist=None, device: str = "cpu") -> float:
    """Max of a per-rank time over all ranks (replicas: the job ends with its slowest GPU)."""
    if dist is None:
        return ms
    import torch
    t = torch.tensor([float(ms)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def job_throughput(n_keys: int, steps: int, world: int, total_ms: float) -> float:
    """Whole-job keys/s: every rank processes n_keys per step (weak scaling, replicas)."""
    return world * n_keys * steps / (total_ms / 1e3)


def _dist_setup():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def _cpu_info():
    model = platform.processor() or ""
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                model = ln.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model, "threads": 1}


def _pin_one_core():
    try:
        os.sched_setaffinity(0, {sorted(os.sched_getaffinity(0))[0]})
        return True
    except (AttributeError, OSError):
        return False


def _config(args):
    w = 8 if args.values else 4
    ex = ({"insert": "level pipeline (bgpq_ins_pipe2_kernel: root stage, one stage CTA per heap depth, sorter CTAs)",
           "deletemin": ("cluster engine (bgpq_dsys_kernel: 5-CTA cluster over depths 0-4, walker CTAs "
                         "below) + the call's tail on the top CTA (bgpq_dtop_kernel)")} if args.mode == "default" else
          {"insert": "per-node locks (bgpq_locks_kernel, FLAG_LOCKS)",
           "deletemin": "per-node locks (bgpq_locks_kernel, FLAG_LOCKS)"})
    return {"workload": (f"C2 phased: insert 2^{args.n_log2} {args.dist} uint32 keys into an empty BGPQ "
                         f"then deletemin all, K={args.K}, {'key+value' if args.values else 'keys only'} "
                         f"(w={w} B)"),
            "n_keys": 1 << args.n_log2, "K": args.K, "w_bytes": w, "dist": args.dist, "mode": args.mode,
            "execution": ex,
            "l2": f"inputs and heap ({(1 << args.n_log2) * w * 3 >> 20} MiB) larger than the 126 MB L2; no flush"}


def cpu_baseline(args, n_log2_sample=None):
    """The oracle as it stands on one pinned host core (std::multiset batched PQ, the
    reference arm), plus a textbook binary heap and std::sort on the same phased workload."""
    import oracle
    import synth
    oracle.build()
    pinned = _pin_one_core()
    lg = n_log2_sample or args.ref_log2
    n = 1 << lg
    keys = synth.keys(n, seed=synth.SEEDS["C2"], dist=args.dist)
    t0 = time.perf_counter()
    out = oracle.pq_phased(keys, args.K)
    dt = time.perf_counter() - t0
    assert len(out) == n
    lg2 = min(args.base_log2, args.n_log2)
    keys2 = synth.keys(1 << lg2, seed=synth.SEEDS["C2"], dist=args.dist)
    t0 = time.perf_counter(); oracle.binheap_phased(keys2); t_heap = time.perf_counter() - t0
    t0 = time.perf_counter(); oracle.sort_phased(keys2); t_sort = time.perf_counter() - t0
    # n log n extrapolation of the multiset to the full workload (stated, not measured)
    N = 1 << args.n_log2
    extrap = n / dt * (lg / args.n_log2)
    return {"value": n / dt, "unit": "keys/s", "cores": 1, "kind": "oracle",
            "sample": (f"phased insert-all/deletemin-all of 2^{lg} keys (K={args.K}) through the std::multiset "
                       f"oracle (OracleBPQ), 1 pinned host core, {dt:.1f} s"),
            "pinned": pinned, **_cpu_info(),
            "extrapolated_full_keys_per_s": extrap,
            "extrapolation": f"n log n from 2^{lg} to 2^{args.n_log2}: value * {lg}/{args.n_log2}",
            "legs": {
                "std_priority_queue": {"value": (1 << lg2) / t_heap, "unit": "keys/s", "n_log2": lg2,
                                       "seconds": t_heap, "what": "textbook binary heap, one key per op"},
                "std_sort": {"value": (1 << lg2) / t_sort, "unit": "keys/s", "n_log2": lg2, "seconds": t_sort,
                             "what": "closed form of the phased output"}}}


def run_reference(args, world, rank):
    """Reference arm: the CPU oracle (std::multiset, oracle/) on a bounded sample of the same
    workload on one host core (rank 0 only; other ranks exit 0 without work)."""
    if rank != 0:
        return
    import oracle
    import synth
    oracle.build()
    n_sample = 1 << args.ref_log2
    keys = synth.keys(n_sample, seed=synth.SEEDS["C2"], dist=args.dist)
    _pin_one_core()
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        out = oracle.pq_phased(keys, args.K)
        dt = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(dt)
    assert np.array_equal(out[:1024], np.sort(keys)[:1024])
    t = float(np.mean(times))
    v = n_sample / t
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "keys/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": _config(args),
            "cpu_baseline": {"value": v, "unit": "keys/s", "cores": 1, "kind": "oracle", **_cpu_info(),
                             "sample": f"phased insert-all/deletemin-all of 2^{args.ref_log2} keys "
                                       f"(K={args.K}) through the std::multiset oracle, 1 pinned core"},
            "e2e": {"value": v, "unit": "keys/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def measure_mix(args, world, rank, local, dist, q_factory=None):
    """C2 mix: prefill 2^prefill keys (stream 22), then
    bgpq_run_mixed over n/K insert(K) + n/K deletemin(K) ops interleaved as pairs.
    keys/s = (keys inserted + keys deleted) / 2 / t.  Each step re-builds the
    prefilled heap untimed (drain + prefill insert), then times the mixed call only."""
    import torch
    import synth
    import paper_conf_icpp_chenhjz21_b200 as pkg

    n, K, P = 1 << args.mix_log2, args.K, (1 << args.prefill_log2) if args.prefill_log2 >= 0 else 0
    w = 8 if args.values else 4
    n_pairs = n // K
    types, sizes = synth.mixed_ops(n_pairs, K, seed=synth.SEEDS["C2_mix"])
    in_off = np.zeros(2 * n_pairs, np.uint64)
    in_off[0::2] = np.arange(n_pairs, dtype=np.uint64) * K
    keys = synth.keys(n, seed=synth.SEEDS["C2"] + rank, dist=args.dist)
    pre = synth.keys(max(P, 1), seed=synth.SEEDS["C2_mix"] + rank, dist=args.dist)[:P]
    d_types = torch.from_numpy(types).cuda()
    d_sizes = torch.from_numpy(sizes.view(np.int32)).cuda()
    d_off = torch.from_numpy(in_off.view(np.int64)).cuda()
    dk = torch.from_numpy(keys.view(np.int32)).cuda()
    dpre = torch.from_numpy(pre.view(np.int32)).cuda()
    dv = torch.arange(n, dtype=torch.int32, device="cuda") if args.values else None
    dpv = torch.arange(P, dtype=torch.int32, device="cuda") if args.values else None
    out_k = torch.empty(2 * n_pairs * K, dtype=torch.int32, device="cuda")
    out_v = torch.empty(2 * n_pairs * K, dtype=torch.int32, device="cuda") if args.values else None
    cnt = torch.zeros(2 * n_pairs, dtype=torch.int32, device="cuda")
    drain = torch.empty(n + P + K, dtype=torch.int32, device="cuda")
    drain_v = torch.empty(n + P + K, dtype=torch.int32, device="cuda") if args.values else None
    q = pkg.BGPQ(capacity=n + P + K, K=K, values=args.values)
    if args.grid:
        q.set_grid(args.grid)
    stream = torch.cuda.current_stream()

    def reset():
        sz = q.size(stream=stream)
        if sz:
            q.deletemin(sz, drain, drain_v, stream=stream)
        if P:
            q.insert(dpre, dpv, stream=stream)

    def mixed():
        q.run_mixed(d_types, d_sizes, d_off, dk, dv, out_k, out_v, cnt, None, stream=stream)

    for _ in range(args.warmup):
        reset(); mixed()
    torch.cuda.synchronize()
    # parity of the last warm-up step at full size: the key multiset is conserved (mix
    # outputs + what is left in the heap == prefill + inserted keys); with a prefill every
    # deletemin also returned K keys (with an empty heap early deletemins may find fewer)
    left = q.size(stream=stream)
    if left:
        q.deletemin(left, drain, drain_v, stream=stream)
    torch.cuda.synchronize()
    mask = 0xFFFFFFFF
    outs = out_k.view(2 * n_pairs, K)[1::2]
    cnts = cnt[1::2].to(torch.int64)
    sel = torch.arange(K, device="cuda").unsqueeze(0) < cnts.unsqueeze(1)
    got = torch.cat([outs[sel], drain[:left]]).to(torch.int64) & mask
    want = torch.cat([dk, dpre]).to(torch.int64) & mask
    ok_parity = bool(torch.equal(torch.sort(got)[0], torch.sort(want)[0]))
    if P:
        ok_parity = ok_parity and bool((cnt[1::2] == K).all().item())
    del got, want, outs, sel

    ms, launches, acc = [], 0, None
    for _ in range(args.steps):
        reset()
        st0 = q.stats()  # synchronizes; counters bracket the mixed call only
        l0 = pkg.launch_count()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        if dist: dist.barrier()
        torch.cuda.synchronize()
        e0.record(stream); mixed(); e1.record(stream)
        torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
        launches += pkg.launch_count() - l0
        st1 = q.stats()
        d = {k: st1[k] - st0[k] for k in st1}
        acc = d if acc is None else {k: acc[k] + d[k] for k in d}
    q.close()
    total_ms = max_over_ranks(float(np.sum(ms)), dist, device="cuda")
    ms_per_step = total_ms / args.steps
    value = job_throughput(n, args.steps, world, total_ms)
    dst = {k: v // args.steps for k, v in acc.items()}
    bm = byte_model(dst, K, w)
    peak, peak_src = _peaks()
    achieved = bm["total"] / (ms_per_step / 1e3) / 1e9
    return {
        "metric": METRIC + " — C2 50/50 concurrent mix", "value": value, "unit": "keys/s",
        "ms_per_step": ms_per_step, "steps": args.steps, "warmup": args.warmup,
        "config": {"workload": (f"C2 mix: prefill 2^{args.prefill_log2} then {n_pairs} insert(K) + "
                                f"{n_pairs} deletemin(K) ops as pairs, 2^{args.mix_log2} {args.dist} "
                                f"keys, K={K}, w={w} B; keys/s = (in + out)/2/t") if P else
                   (f"C2 mix: empty heap, {n_pairs} insert(K) + {n_pairs} deletemin(K) pairs"),
                   "n_keys": n, "K": K, "w_bytes": w, "prefill": P, "dist": args.dist,
                   "execution": ("bgpq_run_mixed: the leading (INSERT(K), DELETEMIN(K)) pairs on the cluster "
                                 "engine (bgpq_msort_kernel sorts the batches, bgpq_dsys_kernel runs each pair "
                                 "as the MARKED hand-off at the root, reading R26), the rest of the call on the "
                                 "per-node-lock engine (bgpq_locks_kernel)"),
                   "l2": "heap and inputs larger than the 126 MB L2; no flush"},
        "roofline": {"bound": "hbm", "kernel": "bgpq_dsys_kernel (the mixed call's pairs)", "achieved": achieved,
                     "peak": peak, "unit": "GB/s", "frac": achieved / peak, "traffic": None,
                     "peak_source": peak_src, "alg_bytes_per_launch": bm["total"]},
        "counters_per_step": dst, "gpu_launches": launches,
        "parity_warmup_multiset_conserved": ok_parity,
    }


def run_mix_only(args, world, rank, local):
    import torch
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    clk = ClockSampler(local)
    clk.start()
    res = measure_mix(args, world, rank, local, dist)
    clocks = clk.stop()
    if rank == 0:
        line = dict(res)
        line.update({"metric": METRIC, "n_gpus": world, "higher_is_better": True, "scaling": "weak",
                     "vs_baseline": None, "dtype": "u32", "data": "synthetic", "clocks": clocks,
                     "parallelism": "replicas only (one linearizable heap per GPU)", "e2e": None})
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--K", type=int, default=1024)
    ap.add_argument("--n-log2", type=int, default=27)
    ap.add_argument("--values", action="store_true")
    ap.add_argument("--dist", default="uniform")
    ap.add_argument("--ref-log2", type=int, default=22, help="multiset oracle sample (cpu_baseline / reference arm)")
    ap.add_argument("--base-log2", type=int, default=24, help="std::priority_queue / std::sort baseline sample")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-mix", action="store_true", help="skip the C2 concurrent-mix sub-measurement")
    ap.add_argument("--profile-steps", type=int, default=0, help="ncu mode: run N untimed steps and exit")
    ap.add_argument("--mix", action="store_true",
                    help="only the C2 50/50 concurrent mix (paper E4 shape, P:428): prefill, then "
                         "insert(K)/deletemin(K) pairs on the persistent CTAs (bgpq_run_mixed)")
    ap.add_argument("--prefill-log2", type=int, default=23, help="mix prefill 2^p keys (-1: empty heap)")
    ap.add_argument("--mix-log2", type=int, default=None, help="mix keys inserted (default: --n-log2)")
    ap.add_argument("--grid", type=int, default=0, help="mix: persistent CTAs of the mixed call (0 = all co-resident)")
    ap.add_argument("--mode", default="default", choices=["default", "locks"],
                    help="execution: default (insert level pipeline + deletemin cluster engine and top-CTA tail, "
                         "walkers taking the paper's per-node locks below), or the paper-literal per-node-lock engine "
                         "for every call (BGPQ_FLAG_LOCKS)")
    args = ap.parse_args()
    if args.mix_log2 is None:
        args.mix_log2 = args.n_log2
    world, rank, local = _dist_setup()

    if args.impl == "reference":
        run_reference(args, world, rank)
        return
    if args.mix:
        run_mix_only(args, world, rank, local)
        return

    import torch
    import synth
    import paper_conf_icpp_chenhjz21_b200 as pkg

    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    n, K = 1 << args.n_log2, args.K
    w = 8 if args.values else 4
    keys = synth.keys(n, seed=synth.SEEDS["C2"] + rank, dist=args.dist)
    dk = torch.from_numpy(keys.view(np.int32)).cuda()
    dv = torch.arange(n, dtype=torch.int32, device="cuda") if args.values else None
    out_k = torch.empty(n, dtype=torch.int32, device="cuda")
    out_v = torch.empty(n, dtype=torch.int32, device="cuda") if args.values else None
    q = pkg.BGPQ(capacity=n, K=K, values=args.values, locks=(args.mode == "locks"))
    stream = torch.cuda.current_stream()

    def step(ev=None):
        if ev: ev[0].record(stream)
        q.insert(dk, dv, stream=stream)
        if ev: ev[1].record(stream)
        q.deletemin(n, out_k, out_v, stream=stream)
        if ev: ev[2].record(stream)

    if args.profile_steps:
        for _ in range(args.profile_steps):
            step()
        torch.cuda.synchronize()
        return

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    # parity spot check of the warm-up pass (full output vs sorted input, on device)
    mask = 0xFFFFFFFF
    ref_sorted = torch.sort(dk.to(torch.int64) & mask)[0]
    ok_parity = bool(torch.equal(out_k.to(torch.int64) & mask, ref_sorted))
    del ref_sorted

    st0 = q.stats()
    l0 = pkg.launch_count()
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    clk = ClockSampler(local)
    clk.start()
    if dist: dist.barrier()
    torch.cuda.synchronize()
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    t_start.record(stream)
    for i in range(args.steps):
        step(evs[i])
    t_end.record(stream)
    torch.cuda.synchronize()
    if dist: dist.barrier()
    clocks = clk.stop()
    launches = pkg.launch_count() - l0
    st1 = q.stats()
    total_ms = t_start.elapsed_time(t_end)
    ins_ms = [e[0].elapsed_time(e[1]) for e in evs]
    del_ms = [e[1].elapsed_time(e[2]) for e in evs]
    total_ms = max_over_ranks(total_ms, dist, device="cuda")
    ms_per_step = total_ms / args.steps
    value = job_throughput(n, args.steps, world, total_ms)

    dst = {k: (st1[k] - st0[k]) // args.steps for k in st1}
    bm = byte_model(dst, K, w)
    peak, peak_src = _peaks()
    del_s = float(np.mean(del_ms)) / 1e3
    ins_s = float(np.mean(ins_ms)) / 1e3
    achieved = bm["deletemin"] / del_s / 1e9
    traffic, traffic_src = None, None
    prof = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(prof):
        try:
            pj = json.load(open(prof))
            ent = pj.get(f"K{K}_w{w}_n{args.n_log2}", {})
            traffic, traffic_src = ent.get("deletemin_dram_bytes"), ent.get("source")
        except Exception:
            traffic = None
    n_ops = dst["del_ops"] or (n // K)
    floor_cyc = CHAIN_FLOOR_CYCLES.get(K)
    crit = None
    if floor_cyc and args.mode == "default":
        floor_s = n_ops * floor_cyc / (SM_MHZ * 1e6)
        crit = {"what": "serial DELETEMIN chain (Alg.3 l.10-15): one link per batch",
                "cycles_per_op_floor": floor_cyc, "cycles_per_op_measured": del_s / n_ops * SM_MHZ * 1e6,
                "ms_floor": floor_s * 1e3, "frac_of_roofline_at_floor": bm["deletemin"] / floor_s / 1e9 / peak,
                "measured_over_floor": del_s / floor_s}

    e2e = None
    if not args.no_e2e:
        # public API with HOST buffers: H2D of the inputs and D2H of the results in the region
        hk = torch.from_numpy(keys.view(np.int32)).pin_memory().numpy().view(np.uint32)
        hv = np.arange(n, dtype=np.uint32) if args.values else None
        if hv is not None:
            hv = torch.from_numpy(hv.view(np.int32)).pin_memory().numpy().view(np.uint32)
        ho = torch.empty(n, dtype=torch.int32).pin_memory().numpy().view(np.uint32)
        hov = torch.empty(n, dtype=torch.int32).pin_memory().numpy().view(np.uint32) if args.values else None
        q.insert_host(hk, hv)
        q.deletemin_host(n, ho, hov)  # warm the staging buffers
        e_steps = max(1, min(args.steps, 3))
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(e_steps):
            q.insert_host(hk, hv)
            cnt = q.deletemin_host(n, ho, hov)
        torch.cuda.synchronize()
        e_dt = (time.perf_counter() - t0) / e_steps
        e_dt = max_over_ranks(e_dt, dist, device="cuda")
        assert cnt == n
        e2e = {"value": world * n / e_dt, "unit": "keys/s", "h2d_bytes_per_step": n * w,
               "d2h_bytes_per_step": n * w + 8, "ms_per_step": e_dt * 1e3}
    q.close()

    mix = None
    if not args.no_mix and args.mode == "default":
        mix = measure_mix(args, world, rank, local, dist)

    if rank == 0:
        cpu = None if args.no_cpu_baseline else cpu_baseline(args)
        line = {
            "metric": METRIC, "value": value, "unit": "keys/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": _config(args),
            "parallelism": "replicas only (one linearizable heap per GPU)",
            "phases_ms": {"insert": float(np.mean(ins_ms)), "deletemin": float(np.mean(del_ms))},
            "roofline": {"bound": "hbm",
                         "kernel": ("bgpq_dsys_kernel (+ its bgpq_dtop_kernel tail, ~2% of the DELETEMIN call "
                                    "in the ncu launch list profiles/r2/launches_r2.csv)" if args.mode == "default"
                                    else "bgpq_locks_kernel (DELETEMIN launch)"),
                         "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": traffic, "traffic_source": traffic_src, "peak_source": peak_src,
                         "alg_bytes_per_launch": bm["deletemin"],
                         "alg_bytes_rule": "K*w out + 2K*w refill read/final write + 4K*w per heapify level (counters)",
                         "critical_path_bound": crit},
            "roofline_step": {"alg_bytes_per_step": bm["total"], "b_eff_per_step": bm["total_eff"],
                              "insert_noop_bytes_skipped": bm["insert_noop_skipped"],
                              "achieved_GBps": bm["total"] / (ms_per_step / 1e3) / 1e9,
                              "frac": bm["total"] / (ms_per_step / 1e3) / 1e9 / peak,
                              "b_eff_frac": bm["total_eff"] / (ms_per_step / 1e3) / 1e9 / peak,
                              "insert_GBps": bm["insert"] / ins_s / 1e9,
                              "insert_eff_GBps": bm["insert_eff"] / ins_s / 1e9,
                              "insert_kernel": "bgpq_ins_pipe2_kernel"},
            "counters_per_step": dst,
            "gpu_launches": launches,
            "clocks": clocks,
            "e2e": e2e,
            "cpu_baseline": cpu,
            "mix": mix,
            "parity_warmup_output_sorted": ok_parity,
        }
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
