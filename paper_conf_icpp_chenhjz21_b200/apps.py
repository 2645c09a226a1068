"""The paper's applications on BGPQ (§6.5): 0-1 knapsack branch and bound
and A* on a grid, one BGPQ per GPU, with a round-based multi-GPU driver.

Thin marshalling over include/bgpq_apps.h (the kernels are in csrc/bgpq_apps.cu: every
expansion, bound, prune and queue operation runs on the GPU).  The driver between rounds is
host logic over torch.distributed collectives (NCCL over NVLink on GPUs, gloo in the CPU
tests): all-reduce of the incumbent (max profit / min cost), all-gather of the queue sizes, and
donor -> receiver batches of K entries (send / recv) to rebalance.
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import BGPQ, _check, _ptr, _stream, lib

_vp, _u32, _u64 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64

ST_INC, ST_PENDING, ST_EXPANDED, ST_INSERTED, ST_POPS, ST_ERR, ST_PRUNED, ST_EMPTY = range(8)
STATE_NAMES = ("incumbent", "pending", "expanded", "inserted", "pops", "err", "pruned", "empty_pops")
UNBOUNDED = 1 << 31  # per-CTA DELETEMIN budget of a single-GPU run (effectively unbounded)


class _KsT(ctypes.Structure):
    _fields_ = [("n", _u32), ("C", _u64), ("w", _vp), ("p", _vp), ("Wp", _vp), ("Pp", _vp)]


class _AsT(ctypes.Structure):
    _fields_ = [("N", _u32), ("M", _u32), ("grid", _vp), ("g", _vp), ("tr", _u32), ("tc", _u32)]


def _bind():
    L = lib()
    if not getattr(L, "_apps_bound", False):
        L.bgpq_ks_prepare.argtypes = [_u32, _vp, _vp, _u64, ctypes.POINTER(_KsT), _vp]
        L.bgpq_ks_root.argtypes = [ctypes.POINTER(_KsT), _vp, _vp, _vp]
        L.bgpq_ks_run.argtypes = [_vp, ctypes.POINTER(_KsT), _vp, _u32, _vp]
        L.bgpq_astar_init.argtypes = [ctypes.POINTER(_AsT), _u32, _u32, _vp, _vp, _vp]
        L.bgpq_astar_run.argtypes = [_vp, ctypes.POINTER(_AsT), _vp, _u32, _vp]
        L._apps_bound = True
    return L


class _Search:
    """Common part: one heap (values on), the 8-word state, pop / push of raw entries."""
    maximize = True
    # CTAs of the application kernel when the caller does not choose (None); 0 = all
    # co-resident.  From the one-B200 sweeps in profiles/r2 (ks_ctas_*.json, astar_ctas_*.json):
    # fewer CTAs contend less for the root lock when the frontier is narrow.
    DEFAULT_CTAS = 0

    def __init__(self, K: int, capacity: int, ctas: int | None = None):
        import torch
        self.K = K
        self.q = BGPQ(capacity=capacity, K=K, values=True)
        ctas = self.DEFAULT_CTAS if ctas is None else ctas
        if ctas:
            self.q.set_grid(ctas)
        self.state = torch.zeros(8, dtype=torch.int64, device="cuda")
        self._one_k = torch.zeros(1, dtype=torch.int32, device="cuda")
        self._one_v = torch.zeros(1, dtype=torch.int32, device="cuda")

    def size(self) -> int:
        return self.q.size()

    def incumbent(self) -> int:
        return int(self.state[ST_INC].item())

    def set_incumbent(self, v: int):
        self.state[ST_INC] = int(v)

    def stats(self) -> dict:
        s = self.state.cpu().numpy()
        return {nm: int(s[i]) for i, nm in enumerate(STATE_NAMES)}

    def pop(self, n: int):
        """DELETEMIN n entries (the best ones) for a transfer to another GPU."""
        k, v = self.q.deletemin(n)
        return k, v

    def push(self, keys, vals):
        if keys.numel():
            self.q.insert(keys.cuda(), vals.cuda())

    def _prepare_run(self):
        self.state[ST_PENDING] = self.size()

    def close(self):
        self.q.close()


class KnapsackSearch(_Search):
    """0-1 knapsack branch and bound (R23) on the current GPU."""
    maximize = True
    # C4: 1.58-1.64 s in 6 of 6 solves at 16 CTAs; at 32 / 64 CTAs the relaxed best-first order
    # expands up to 10x more nodes in some solves (1.4-13 s / 1.8-16 s; one 64-CTA solve ran
    # > 2 min), a heavy tail from late incumbents (tools/ab_ks.py, one B200)
    DEFAULT_CTAS = 16

    def __init__(self, w: np.ndarray, p: np.ndarray, C: int, K: int = 1024, capacity: int = 1 << 27,
                 ctas: int | None = None):
        import torch
        super().__init__(K, capacity, ctas)
        n = len(w)
        self.n, self.C = n, int(C)
        dw = torch.from_numpy(np.ascontiguousarray(w, np.uint32).view(np.int32)).cuda()
        dp = torch.from_numpy(np.ascontiguousarray(p, np.uint32).view(np.int32)).cuda()
        self._w = torch.empty(n, dtype=torch.int32, device="cuda")
        self._p = torch.empty(n, dtype=torch.int32, device="cuda")
        self._Wp = torch.empty(n + 1, dtype=torch.int64, device="cuda")
        self._Pp = torch.empty(n + 1, dtype=torch.int64, device="cuda")
        self.ks = _KsT(n, self.C, self._w.data_ptr(), self._p.data_ptr(), self._Wp.data_ptr(), self._Pp.data_ptr())
        _check(_bind().bgpq_ks_prepare(n, _ptr(dw), _ptr(dp), self.C, ctypes.byref(self.ks), _stream(None)))
        torch.cuda.synchronize()

    def seed(self):
        """Insert the root of the search tree (level 0, nothing taken)."""
        _check(_bind().bgpq_ks_root(ctypes.byref(self.ks), _ptr(self._one_k), _ptr(self._one_v), _stream(None)))
        self.q.insert(self._one_k, self._one_v)

    def run(self, budget: int = UNBOUNDED):
        self._prepare_run()
        _check(_bind().bgpq_ks_run(self.q._h, ctypes.byref(self.ks), _ptr(self.state), int(budget), _stream(None)))


class AStarSearch(_Search):
    """A* on an N x M obstacle grid (R24) on the current GPU."""
    maximize = False
    INF = 0xFFFFFFFF
    DEFAULT_CTAS = 8  # C5 10 %: 2.06 s at 8 CTAs vs 3.64 s with all 148

    def __init__(self, grid: np.ndarray, start, target, K: int = 1024, capacity: int = 1 << 27, dgrid=None,
                 ctas: int | None = None):
        import torch
        super().__init__(K, capacity, ctas)
        N, M = grid.shape if dgrid is None else dgrid.shape
        self.N, self.M = int(N), int(M)
        self.start, self.target = tuple(start), tuple(target)
        self._grid = dgrid if dgrid is not None else torch.from_numpy(np.ascontiguousarray(grid, np.uint8)).cuda()
        self._g = torch.empty(self.N * self.M, dtype=torch.int32, device="cuda")
        self.asr = _AsT(self.N, self.M, self._grid.data_ptr(), self._g.data_ptr(), int(target[0]), int(target[1]))
        self.state[ST_INC] = self.INF

    def seed(self):
        _check(_bind().bgpq_astar_init(ctypes.byref(self.asr), int(self.start[0]), int(self.start[1]),
                                       _ptr(self._one_k), _ptr(self._one_v), _stream(None)))
        self.q.insert(self._one_k, self._one_v)

    def reset_g(self):
        """g := +inf everywhere (a rank that never seeds still needs an initialised g)."""
        self._g.fill_(-1)

    def run(self, budget: int = UNBOUNDED):
        self._prepare_run()
        _check(_bind().bgpq_astar_run(self.q._h, ctypes.byref(self.asr), _ptr(self.state), int(budget),
                                      _stream(None)))


# ------------------------------------------------------------------------------------------
# multi-GPU driver: rounds of local search + incumbent all-reduce + rebalance
# ------------------------------------------------------------------------------------------
def rebalance_plan(sizes, K: int):
    """Deterministic donor -> receiver transfers [(src, dst, n)] with n a multiple of K: ranks
    above the mean by >= K give whole K-batches to ranks below it by >= K, largest first."""
    G = len(sizes)
    total = int(sum(sizes))
    target = total // G
    sur = sorted(((s - target, r) for r, s in enumerate(sizes) if s - target >= K), key=lambda x: (-x[0], x[1]))
    dfc = sorted(((target - s, r) for r, s in enumerate(sizes) if target - s >= K), key=lambda x: (-x[0], x[1]))
    sur = [list(x) for x in sur]
    dfc = [list(x) for x in dfc]
    plan = []
    i = j = 0
    while i < len(sur) and j < len(dfc):
        amt = min(sur[i][0], dfc[j][0]) // K * K
        if amt >= K:
            plan.append((sur[i][1], dfc[j][1], amt))
            sur[i][0] -= amt
            dfc[j][0] -= amt
        if sur[i][0] < K:
            i += 1
        if j < len(dfc) and dfc[j][0] < K:
            j += 1
    return plan


class TorchComm:
    """Collectives of the driver on torch.distributed (NCCL on GPUs, gloo on CPU)."""

    def __init__(self, dist, device):
        self.dist, self.device = dist, device
        self.rank, self.world = dist.get_rank(), dist.get_world_size()

    def allreduce(self, v: int, op: str) -> int:
        import torch
        t = torch.tensor([v], dtype=torch.int64, device=self.device)
        self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX if op == "max" else self.dist.ReduceOp.MIN)
        return int(t.item())

    def allgather(self, v: int):
        import torch
        t = torch.tensor([v], dtype=torch.int64, device=self.device)
        out = [torch.zeros_like(t) for _ in range(self.world)]
        self.dist.all_gather(out, t)
        return [int(x.item()) for x in out]

    def send(self, t, dst):
        self.dist.send(t.to(self.device), dst)

    def recv(self, n, src):
        """n int32 entries (uint32 bit patterns) from rank src."""
        import torch
        t = torch.empty(n, dtype=torch.int32, device=self.device)
        self.dist.recv(t, src)
        return t


def run_search(solver, comm=None, budget: int = 64, max_rounds: int = 1 << 30):
    """Run a search to completion.  Single process (comm None): one unbounded kernel run.
    Several ranks: rounds of `budget` DELETEMINs per CTA, then incumbent all-reduce, size
    all-gather and rebalancing; ends when every queue is empty (reading R19 / R25).
    Returns (global incumbent, rounds, bytes moved between ranks)."""
    if comm is None or comm.world == 1:
        solver.run()
        return solver.incumbent(), 1, 0
    rounds, moved = 0, 0
    inc = solver.incumbent()
    while rounds < max_rounds:
        solver.run(budget)
        inc = comm.allreduce(solver.incumbent(), "max" if solver.maximize else "min")
        solver.set_incumbent(inc)
        sizes = comm.allgather(solver.size())
        rounds += 1
        if sum(sizes) == 0:
            break
        for src, dst, n in rebalance_plan(sizes, solver.K):
            if comm.rank == src:
                k, v = solver.pop(n)
                comm.send(k[:n], dst)
                comm.send(v[:n], dst)
            elif comm.rank == dst:
                k = comm.recv(n, src)
                v = comm.recv(n, src)
                solver.push(k, v)
            moved += 8 * n
    return inc, rounds, moved
