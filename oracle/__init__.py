"""CPU oracle for the BGPQ hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import this package.  The product package
(``paper_conf_icpp_chenhjz21_b200``) never imports it; the two share no code.

Everything here is a thin ctypes marshalling layer over ``bgpq_oracle.cpp`` (plain C++17,
see its header for what each function transcribes from PAPER.md), plus ``build()``.

Pins: see tests/test_oracle.py.  Parity status per function is in DESIGN.md §Oracle.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "bgpq_oracle.cpp")
_SRCS = [_SRC, os.path.join(_HERE, "apps_oracle.cpp")]
_LIB = os.path.join(_HERE, "liboracle.so")

AVAIL, EMPTY, TARGET, MARKED = 0, 1, 2, 3  # P:180 §4

_u32p = ctypes.POINTER(ctypes.c_uint32)
_u64p = ctypes.POINTER(ctypes.c_uint64)
_i64p = ctypes.POINTER(ctypes.c_longlong)


def build(force: bool = False) -> str:
    """Compile liboracle.so with g++ (-O2, C++17).  Building the checker is not using it."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(map(os.path.getmtime, _SRCS)):
        cmd = ["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", _LIB + ".tmp", *_SRCS]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        L.orc_sort_split.argtypes = [_u32p, _u32p, ctypes.c_uint32, _u32p, _u32p, ctypes.c_uint32,
                                     ctypes.c_uint32, _u32p, _u32p, _u32p, _u32p]
        L.orc_pq_new.restype = ctypes.c_void_p
        L.orc_pq_free.argtypes = [ctypes.c_void_p]
        L.orc_pq_size.argtypes = [ctypes.c_void_p]
        L.orc_pq_size.restype = ctypes.c_uint64
        L.orc_pq_insert.argtypes = [ctypes.c_void_p, _u32p, _u32p, ctypes.c_uint64]
        L.orc_pq_deletemin.argtypes = [ctypes.c_void_p, ctypes.c_uint64, _u32p, _u32p]
        L.orc_pq_deletemin.restype = ctypes.c_uint64
        L.orc_pq_phased.argtypes = [_u32p, ctypes.c_uint64, ctypes.c_uint32, _u32p]
        L.orc_pq_phased.restype = ctypes.c_uint64
        L.orc_seq_new.argtypes = [ctypes.c_uint32, ctypes.c_uint32]
        L.orc_seq_new.restype = ctypes.c_void_p
        L.orc_seq_free.argtypes = [ctypes.c_void_p]
        L.orc_seq_set_mutation.argtypes = [ctypes.c_void_p, ctypes.c_int]
        L.orc_seq_insert.argtypes = [ctypes.c_void_p, _u32p, _u32p, ctypes.c_uint32]
        L.orc_seq_insert.restype = ctypes.c_int
        L.orc_seq_deletemin.argtypes = [ctypes.c_void_p, ctypes.c_uint32, _u32p, _u32p]
        L.orc_seq_deletemin.restype = ctypes.c_longlong
        L.orc_seq_header.argtypes = [ctypes.c_void_p, _i64p]
        L.orc_seq_dump.argtypes = [ctypes.c_void_p, _u32p, _u32p, _u32p]
        L.orc_seq_counters.argtypes = [ctypes.c_void_p, _u64p]
        L.orc_check_invariants.argtypes = [ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                           ctypes.c_uint32, ctypes.c_uint32, _u32p, _u32p, _u64p]
        L.orc_check_invariants.restype = ctypes.c_int
        for nm in ("orc_binheap_phased", "orc_sort_phased"):
            getattr(L, nm).argtypes = [_u32p, ctypes.c_uint64, _u32p]
            getattr(L, nm).restype = ctypes.c_uint64
        for nm in ("orc_ks_dp", "orc_ks_brute"):
            getattr(L, nm).argtypes = [ctypes.c_uint32, _u32p, _u32p, ctypes.c_uint64]
            getattr(L, nm).restype = ctypes.c_longlong
        L.orc_ks_bnb.argtypes = [ctypes.c_uint32, _u32p, _u32p, ctypes.c_uint64, _u64p]
        for nm in ("orc_astar", "orc_dijkstra"):
            getattr(L, nm).argtypes = [ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p] + [ctypes.c_uint32] * 4 + [_u64p]
        _lib = L
    return _lib


def _p32(a):
    if a is None:
        return None
    assert a.dtype == np.uint32 and a.flags.c_contiguous
    return a.ctypes.data_as(_u32p)


def _u32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.uint32))


def sort_split(zk, zv, wk, wv, ma):
    """SORT_SPLIT: returns (xk, xv, yk, yv) = sorted(Z ∪ W) split at Ma."""
    zk, zv, wk, wv = _u32(zk), _u32(zv), _u32(wk), _u32(wv)
    na, nb = len(zk), len(wk)
    xk = np.empty(ma, np.uint32); xv = np.empty(ma, np.uint32)
    yk = np.empty(na + nb - ma, np.uint32); yv = np.empty(na + nb - ma, np.uint32)
    rc = lib().orc_sort_split(_p32(zk), _p32(zv), na, _p32(wk), _p32(wv), nb, ma,
                              _p32(xk), _p32(xv), _p32(yk), _p32(yv))
    if rc != 0:
        raise ValueError("Ma > Na + Nb")
    return xk, xv, yk, yv


class OraclePQ:
    """The ADT: std::multiset; deletemin(m) -> the m smallest, ascending."""

    def __init__(self):
        self._h = lib().orc_pq_new()

    def __del__(self):
        if getattr(self, "_h", None):
            lib().orc_pq_free(self._h)
            self._h = None

    def insert(self, keys, vals=None):
        keys = _u32(keys)
        vals = None if vals is None else _u32(vals)
        lib().orc_pq_insert(self._h, _p32(keys), _p32(vals), len(keys))

    def deletemin(self, m):
        ok = np.empty(m, np.uint32); ov = np.empty(m, np.uint32)
        c = lib().orc_pq_deletemin(self._h, m, _p32(ok), _p32(ov))
        return ok[:c], ov[:c]

    def size(self):
        return int(lib().orc_pq_size(self._h))


def pq_phased(keys, K):
    """Insert all keys in K-batches, then deletemin all in K-batches (OracleBPQ)."""
    keys = _u32(keys)
    out = np.empty_like(keys)
    c = lib().orc_pq_phased(_p32(keys), len(keys), K, _p32(out))
    return out[:c]


def binheap_phased(keys):
    """Baseline (not a pin): the phased workload through std::priority_queue, one key per op."""
    keys = _u32(keys)
    out = np.empty_like(keys)
    lib().orc_binheap_phased(_p32(keys), len(keys), _p32(out))
    return out


def sort_phased(keys):
    """Baseline (not a pin): the closed form of the phased workload, std::sort."""
    keys = _u32(keys)
    out = np.empty_like(keys)
    lib().orc_sort_phased(_p32(keys), len(keys), _p32(out))
    return out


class SeqBGPQ:
    """Literal sequential model of Alg.1-3 (see bgpq_oracle.cpp)."""

    COUNTER_NAMES = ("ins_ops", "ins_heapify_ops", "ins_levels", "ins_noop", "ins_swap",
                     "ins_merge", "del_ops", "del_refill_ops", "del_levels", "del_lr_merge",
                     "del_lr_skip")

    def __init__(self, K, cap_nodes, mutation=0):
        self.K, self.cap = int(K), int(cap_nodes)
        self._h = lib().orc_seq_new(self.K, self.cap)
        if not self._h:
            raise ValueError("K must be > 1 (P:146)")
        if mutation:
            lib().orc_seq_set_mutation(self._h, mutation)

    def __del__(self):
        if getattr(self, "_h", None):
            lib().orc_seq_free(self._h)
            self._h = None

    def insert(self, keys, vals=None):
        keys = _u32(keys)
        vals = None if vals is None else _u32(vals)
        rc = lib().orc_seq_insert(self._h, _p32(keys), _p32(vals), len(keys))
        if rc == -1:
            raise ValueError("insert size must be in 1..K (P:150)")
        return rc

    def deletemin(self, size):
        ok = np.empty(size, np.uint32); ov = np.empty(size, np.uint32)
        c = lib().orc_seq_deletemin(self._h, size, _p32(ok), _p32(ov))
        if c < 0:
            raise ValueError("deletemin size must be in 1..K (P:150)")
        return ok[:c], ov[:c]

    def header(self):
        h = (ctypes.c_longlong * 4)()
        lib().orc_seq_header(self._h, h)
        return {"heapSize": h[0], "rootSize": h[1], "pbSize": h[2], "err": h[3]}

    def dump(self):
        K, cap = self.K, self.cap
        keys = np.empty((cap + 1) * K, np.uint32)
        vals = np.empty((cap + 1) * K, np.uint32)
        states = np.empty(cap + 1, np.uint32)
        lib().orc_seq_dump(self._h, _p32(keys), _p32(vals), _p32(states))
        return keys.reshape(cap + 1, K), vals.reshape(cap + 1, K), states

    def counters(self):
        c = (ctypes.c_uint64 * len(self.COUNTER_NAMES))()
        lib().orc_seq_counters(self._h, c)
        return dict(zip(self.COUNTER_NAMES, list(c)))


def check_invariants(K, cap, heap_size, root_size, pb_size, node_keys, states):
    """P:146 / P:367 invariants on a node-major dump; returns (code, node)."""
    nk = np.ascontiguousarray(node_keys, dtype=np.uint32).reshape(-1)
    st = np.ascontiguousarray(states, dtype=np.uint32)
    assert len(nk) == (cap + 1) * K and len(st) == cap + 1
    where = ctypes.c_uint64(0)
    rc = lib().orc_check_invariants(K, cap, heap_size, root_size, pb_size, _p32(nk), _p32(st),
                                    ctypes.byref(where))
    return int(rc), int(where.value)


def replay(ops, q=None):
    """Replay a linearization log through OraclePQ.

    ``ops`` is an iterable of (kind, payload) in linearization (ticket) order:
    kind 0 = insert, payload = (keys, vals or None); kind 1 = deletemin, payload = size.
    Returns the list of (keys, vals) the oracle gives each deletemin (P:390-394:
    x_{k+1} = min_r(I_k - D_k), or all of I_k - D_k if fewer than r remain).  ``q``: an
    OraclePQ to replay into (its state after the log is then available to the caller)."""
    q = OraclePQ() if q is None else q
    res = []
    for kind, payload in ops:
        if kind == 0:
            q.insert(*payload)
        else:
            res.append(q.deletemin(int(payload)))
    return res


# ---------------------------------------------------------------------------------------
# applications (apps_oracle.cpp)
# ---------------------------------------------------------------------------------------
UNREACHABLE = (1 << 64) - 1


def ks_dp(w, p, C) -> int:
    """0-1 knapsack optimum by the textbook dynamic program (pin)."""
    w, p = _u32(w), _u32(p)
    r = lib().orc_ks_dp(len(w), _p32(w), _p32(p), int(C))
    if r < 0:
        raise ValueError("capacity too large for the DP")
    return int(r)


def ks_brute(w, p, C) -> int:
    """0-1 knapsack optimum by enumerating every subset, n <= 24 (pin)."""
    w, p = _u32(w), _u32(p)
    r = lib().orc_ks_brute(len(w), _p32(w), _p32(p), int(C))
    if r < 0:
        raise ValueError("n > 24")
    return int(r)


def ks_bnb(w, p, C) -> dict:
    """Sequential best-first branch and bound (readings R23): optimum, nodes
    expanded, nodes inserted into the priority queue."""
    w, p = _u32(w), _u32(p)
    out = (ctypes.c_uint64 * 3)()
    lib().orc_ks_bnb(len(w), _p32(w), _p32(p), int(C), out)
    return {"optimum": int(out[0]), "expanded": int(out[1]), "inserted": int(out[2])}


def _grid_call(fn, grid, src, dst):
    g = np.ascontiguousarray(grid, dtype=np.uint8)
    N, M = g.shape
    out = (ctypes.c_uint64 * 2)()
    fn(N, M, g.ctypes.data_as(ctypes.c_void_p), int(src[0]), int(src[1]), int(dst[0]), int(dst[1]), out)
    return int(out[0]), int(out[1])


def astar(grid, src, dst) -> dict:
    """Sequential A* (reading R24: 8 moves, orthogonal 1 / diagonal 2, Manhattan h):
    shortest path cost (UNREACHABLE if none) and nodes expanded."""
    c, e = _grid_call(lib().orc_astar, grid, src, dst)
    return {"cost": c, "expanded": e}


def dijkstra(grid, src, dst) -> int:
    """Dijkstra on the same graph (pin of the A* cost)."""
    return _grid_call(lib().orc_dijkstra, grid, src, dst)[0]
