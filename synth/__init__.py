"""Seeded synthetic input generators shared by tests, bench.py and the oracle harness.

This module holds NONE of the method's arithmetic (no sorting-into-batches, merging or
heap logic): only counter-based random numbers and the input shapes of the paper's
workloads.  Recipes are stated in DESIGN.md §Inputs.

- uniform:    key_i = high 32 bits of splitmix64(seed * 2**40 + i)        ("32-bit keys")
- ascending:  the uniform array sorted ascending   ("sorting the random keys")
- descending: its reverse
- gaussian:   Box-Muller in float64 from two splitmix streams, mu=2**31, sigma=2**29,
              round-half-even, clamped to [0, 2**32-1]   (§8(d) of SURVEY.md)
- bits30:     uniform >> 2 (the paper's 30-bit random keys, P:420 fn.3)
Values are the input index (val_i = i) so every output pair can be checked
(key == input_key[val]).

Applications (no method arithmetic — the instances only):
- knapsack: P:479 names generator [19] without its type.  Default (C4) "strong", the
            strongly correlated class: w_i = 1 + u_i mod 1000, p_i = w_i + 100,
            C = floor(sum w / 2) (R23: the weakly correlated and uncorrelated classes
            are solved by best-first B&B in < 2,000 nodes at n = 1000; the strongly correlated
            one needs ~9.2e7, the scale of the paper's 0.9-1.8 s GPU runs, Table 2);
            "weak": p_i = max(1, w_i - 100 + v_i mod 201); "uncorrelated": p_i = 1 + v_i mod 1000
- grid:     i.i.d. obstacles, cell = 1 iff u < rate * 2**32 ("r% of the nodes ... are
            obstacles ... randomly distributed"); start (0, 0) and target (N-1, M-1) forced free.
"""
from __future__ import annotations

import numpy as np

_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)

SEEDS = {"C1": 1, "C2": 2, "C2_mix": 22, "C3": 3, "C4": 4, "C5": 5}
DISTS = ("uniform", "ascending", "descending", "gaussian")


def splitmix64(counter: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser applied to (counter + golden); counter is uint64."""
    with np.errstate(over="ignore"):
        z = counter.astype(np.uint64) + _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        return z ^ (z >> np.uint64(31))


def _counters(seed: int, n: int, start: int = 0) -> np.ndarray:
    base = np.uint64((int(seed) << 40) & 0xFFFFFFFFFFFFFFFF)
    return base + np.arange(start, start + n, dtype=np.uint64)


def uniform_keys(n: int, seed: int, chunk: int = 1 << 24) -> np.ndarray:
    out = np.empty(n, np.uint32)
    for s in range(0, n, chunk):
        m = min(chunk, n - s)
        out[s:s + m] = (splitmix64(_counters(seed, m, s)) >> np.uint64(32)).astype(np.uint32)
    return out


def gaussian_keys(n: int, seed: int, mu: float = 2.0 ** 31, sigma: float = 2.0 ** 29) -> np.ndarray:
    u1 = (splitmix64(_counters(seed, n)) >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
    u2 = (splitmix64(_counters(seed + 1000003, n)) >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
    u1 = np.maximum(u1, 2.0 ** -60)
    z = np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u2)
    x = np.rint(mu + sigma * z)
    return np.clip(x, 0, 2.0 ** 32 - 1).astype(np.uint32)


def keys(n: int, seed: int, dist: str = "uniform") -> np.ndarray:
    if dist == "uniform":
        return uniform_keys(n, seed)
    if dist == "bits30":
        return uniform_keys(n, seed) >> np.uint32(2)
    if dist == "ascending":
        return np.sort(uniform_keys(n, seed))
    if dist == "descending":
        return np.sort(uniform_keys(n, seed))[::-1].copy()
    if dist == "gaussian":
        return gaussian_keys(n, seed)
    if dist == "dups":  # duplicate-heavy: keys in [0, 64)
        return (uniform_keys(n, seed) % np.uint32(64)).astype(np.uint32)
    raise ValueError(f"unknown distribution {dist!r}")


def values(n: int) -> np.ndarray:
    return np.arange(n, dtype=np.uint32)


def mixed_ops(n_pairs: int, K: int, seed: int, partial: bool = False):
    """Op stream of the utilisation workload: insert/deletemin pairs.

    Returns (op_types uint8 [0=insert, 1=deletemin], op_sizes uint32).  With
    ``partial`` the sizes are drawn uniformly from 1..K (1..k keys per op)."""
    types = np.tile(np.array([0, 1], np.uint8), n_pairs)
    if partial:
        r = uniform_keys(2 * n_pairs, seed)
        sizes = (r % np.uint32(K)).astype(np.uint32) + np.uint32(1)
    else:
        sizes = np.full(2 * n_pairs, K, np.uint32)
    return types, sizes


def random_ops(n_ops: int, K: int, seed: int, p_insert: float = 0.5):
    """Random op types and sizes 1..K (for concurrency stress tests)."""
    r = uniform_keys(2 * n_ops, seed)
    types = (r[:n_ops] >= np.uint32(int(p_insert * 2 ** 32))).astype(np.uint8)
    sizes = (r[n_ops:] % np.uint32(K)).astype(np.uint32) + np.uint32(1)
    return types, sizes


def knapsack_items(n: int, seed: int, kind: str = "strong"):
    """(w, p, C) of a synthetic 0-1 knapsack instance (C4: n = 1000).
    kind "weak": weakly correlated (p_i in [w_i - 100, w_i + 100]); "uncorrelated": p_i
    independent of w_i in [1, 1000]."""
    r = uniform_keys(2 * n, seed)
    w = (np.uint32(1) + r[:n] % np.uint32(1000)).astype(np.uint32)
    if kind == "weak":
        p = np.maximum(1, w.astype(np.int64) - 100 + (r[n:] % np.uint32(201)).astype(np.int64)).astype(np.uint32)
    elif kind == "uncorrelated":
        p = (np.uint32(1) + r[n:] % np.uint32(1000)).astype(np.uint32)
    elif kind == "strong":  # strongly correlated: p_i = w_i + 100
        p = (w + np.uint32(100)).astype(np.uint32)
    else:
        raise ValueError(kind)
    C = int(w.astype(np.uint64).sum() // 2)
    return w, p, C


def grid(N: int, M: int, rate: float, seed: int, chunk: int = 1 << 24) -> np.ndarray:
    """N x M uint8 obstacle grid (1 = obstacle) with i.i.d. obstacles at `rate` (C5: 20000^2 at
    10% / 20%); cells (0, 0) and (N-1, M-1) are forced free."""
    thr = np.uint32(int(rate * 2 ** 32))
    out = np.empty(N * M, np.uint8)
    for s in range(0, N * M, chunk):
        m = min(chunk, N * M - s)
        out[s:s + m] = (splitmix64(_counters(seed, m, s)) >> np.uint64(32)).astype(np.uint32) < thr
    out[0] = 0
    out[-1] = 0
    return out.reshape(N, M)
