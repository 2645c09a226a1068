"""Multi-process (world_size 2 and 3, gloo, CPU) tests of the applications' multi-GPU driver
(paper_conf_icpp_chenhjz21_b200/apps.py: run_search, rebalance_plan, TorchComm): incumbent
all-reduce, queue-size all-gather, donor -> receiver K-batch transfers and the termination
rule (every queue empty), with a CPU stand-in for the per-GPU search (a best-first knapsack
branch and bound on a Python heap; its expansion is test code, the driver is the product's).
The reached optimum must equal the oracle's DP (P:477-479 pinned by the textbook DP)."""
import heapq
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_icpp_chenhjz21_b200 import apps


class CpuKnapsack:
    """Stand-in for apps.KnapsackSearch with the same driver-facing surface."""
    maximize = True

    def __init__(self, w, p, C, K, seed_root):
        order = sorted(range(len(w)), key=lambda i: (-int(p[i]) / int(w[i]), i))
        self.w = [int(w[i]) for i in order]
        self.p = [int(p[i]) for i in order]
        self.C, self.K, self.n = int(C), K, len(w)
        self.heap = []
        self.inc = 0
        self.expanded = 0
        if seed_root:
            self._push_node(0, 0, 0)

    def _bound(self, l, W, P):
        room, ub, j = self.C - W, P, l
        while j < self.n and self.w[j] <= room:
            room -= self.w[j]; ub += self.p[j]; j += 1
        if j < self.n:
            ub += room * self.p[j] // self.w[j]
        return ub

    def _push_node(self, l, W, P):
        ub = self._bound(l, W, P)
        heapq.heappush(self.heap, (0xFFFFFFFF - ub, (l << 22) | W, P))

    def size(self):
        return len(self.heap)

    def incumbent(self):
        return self.inc

    def set_incumbent(self, v):
        self.inc = max(self.inc, v)

    def run(self, budget=1 << 30):
        for _ in range(budget):
            batch = [heapq.heappop(self.heap) for _ in range(min(self.K, len(self.heap)))]
            if not batch:
                return
            for key, v, P in batch:
                ub, l, W = 0xFFFFFFFF - key, v >> 22, v & ((1 << 22) - 1)
                if ub <= self.inc or l == self.n:
                    continue
                self.expanded += 1
                for W2, P2 in ((W + self.w[l], P + self.p[l]), (W, P)):
                    if W2 > self.C:
                        continue
                    self.inc = max(self.inc, P2)
                    if self._bound(l + 1, W2, P2) > self.inc:
                        self._push_node(l + 1, W2, P2)

    def pop(self, n):
        batch = [heapq.heappop(self.heap) for _ in range(n)]
        k = torch.tensor([b[0] for b in batch], dtype=torch.int64).to(torch.int32)
        v = torch.tensor([b[1] for b in batch], dtype=torch.int64).to(torch.int32)
        self._ptab = {(int(b[0]), int(b[1])): b[2] for b in batch}
        return k, v

    def push(self, keys, vals):
        # profit is recoverable from (key, value) as in the GPU encoding: P = ub - g(l, W)
        for key, v in zip(keys.tolist(), vals.tolist()):
            key &= 0xFFFFFFFF; v &= 0xFFFFFFFF
            l, W = v >> 22, v & ((1 << 22) - 1)
            g = self._bound(l, W, 0)
            heapq.heappush(self.heap, (key, v, (0xFFFFFFFF - key) - g))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out, n_items, K, budget):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    w, p, C = synth.knapsack_items(n_items, synth.SEEDS["C4"], "strong")
    solver = CpuKnapsack(w, p, C, K, seed_root=(rank == 0))
    comm = apps.TorchComm(dist, "cpu")
    inc, rounds, moved = apps.run_search(solver, comm, budget=budget)
    out.put((rank, inc, rounds, moved, solver.expanded, solver.size()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_knapsack_driver_reaches_dp_optimum(world):
    n_items, K, budget = 34, 4, 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, n_items, K, budget)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = sorted(q.get(timeout=300) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    w, p, C = synth.knapsack_items(n_items, synth.SEEDS["C4"], "strong")
    want = oracle.ks_dp(w, p, C)
    assert all(r[1] == want for r in res)           # the all-reduced incumbent is the optimum
    assert len({r[2] for r in res}) == 1            # every rank ran the same number of rounds
    assert all(r[5] == 0 for r in res)              # terminated with every queue empty
    assert sum(r[3] for r in res) > 0               # work was moved between ranks
    assert all(r[4] > 0 for r in res)               # every rank expanded nodes


def test_rebalance_plan_rules():
    K = 8
    assert apps.rebalance_plan([0, 0, 0], K) == []
    assert apps.rebalance_plan([100, 0], K) == [(0, 1, 48)]
    plan = apps.rebalance_plan([96, 0, 0, 32], K)
    assert all(n % K == 0 and n >= K for _, _, n in plan)
    moved = {r: 0 for r in range(4)}
    for s, d, n in plan:
        moved[s] -= n; moved[d] += n
    sizes = [96 + moved[0], moved[1], moved[2], 32 + moved[3]]
    assert max(sizes) - min(sizes) <= 2 * K and sum(sizes) == 128
    assert apps.rebalance_plan([10, 9], K) == []    # within a batch of the mean: no transfer
