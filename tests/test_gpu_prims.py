"""Primitive-level GPU parity: the exact device primitives of the hot path (through the
test-only C entry ``bgpq_test_prim``) against the oracle.  -m gpu.

* SORT_SPLIT: X = the Ma smallest of Z u W, Y = the rest, both sorted — compared
  bit-exactly (keys) with ``oracle.sort_split`` over a grid of (Na, Nb, Ma) shapes that
  includes 0 and K, all-equal keys, heavy duplicates, 0xFFFFFFFF keys, and the no-op / swap
  shapes of the heapify walks.  Values: the output (key, value) pairs are a permutation of
  the input pairs (reading R9: equal keys may carry their values in any order).
  variant 0 = the lock / pipeline executions' split (bitonic for full keys-only batches at
  K >= 512, register-window merge path otherwise); 1 = the top CTA's 256-thread group split
  (warp-cooperative merge path, bitonic for full keys-only K >= 512); 2 = the top CTA's
  register-window merge path.
* Sort(items) (Alg.1 l.2): ``cta_sort`` of 1..K entries vs np.sort.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_icpp_chenhjz21_b200 as pkg

VALID_K = (64, 128, 256, 512, 1024)


def _case_keys(rng, n, kind):
    if kind == "uniform":
        k = rng.integers(0, 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    elif kind == "dups":
        k = rng.integers(0, 4, n).astype(np.uint32)
    elif kind == "equal":
        k = np.full(n, 7, np.uint32)
    elif kind == "max":
        k = np.where(rng.random(n) < 0.5, 0xFFFFFFFF, rng.integers(0, 1 << 32, n, dtype=np.uint64)).astype(np.uint32)
    elif kind == "low":
        k = rng.integers(0, 1 << 20, n).astype(np.uint32)
    elif kind == "high":
        k = rng.integers((1 << 32) - (1 << 20), 1 << 32, n, dtype=np.uint64).astype(np.uint32)
    else:
        raise ValueError(kind)
    return np.sort(k)


def _grid(K, full_only=False):
    """(na, nb, ma, kind_z, kind_w) cases."""
    shapes = [(K, K, K)] if full_only else [
        (K, K, K), (0, K, 0), (K, 0, K), (0, K, K), (K, 0, 0), (1, K, 1), (K, 1, K), (K - 1, K, K),
        (K, K, K - 1), (K, K, 1), (K, K, 2 * K - 1), (K, K, 2 * K), (K, K, 0), (3, 5, 4),
        (K // 2 + 3, K - 7, K), (K, K // 3, K // 2), (1, 1, 1), (0, 0, 0)]
    kinds = [("uniform", "uniform"), ("dups", "dups"), ("equal", "equal"), ("max", "max"),
             ("low", "high"), ("high", "low"), ("uniform", "equal")]
    return [(na, nb, ma, kz, kw) for (na, nb, ma) in shapes for (kz, kw) in kinds]


def _run_split(variant, K, values, cases, seed):
    rng = np.random.default_rng(seed)
    n = len(cases)
    Z = np.zeros((n, K), np.uint32)
    W = np.zeros((n, K), np.uint32)
    ZV = np.zeros((n, K), np.uint32)
    WV = np.zeros((n, K), np.uint32)
    for c, (na, nb, ma, kz, kw) in enumerate(cases):
        Z[c, :na] = _case_keys(rng, na, kz)
        W[c, :nb] = _case_keys(rng, nb, kw)
        ZV[c, :na] = np.arange(na) + (c << 16)           # distinct value per input entry
        WV[c, :nb] = np.arange(nb) + (c << 16) + 0x8000
    t = lambda a: torch.from_numpy(a.view(np.int32)).cuda()
    na = torch.tensor([c[0] for c in cases], dtype=torch.int32, device="cuda")
    nb = torch.tensor([c[1] for c in cases], dtype=torch.int32, device="cuda")
    ma = torch.tensor([c[2] for c in cases], dtype=torch.int32, device="cuda")
    xk, xv, yk, yv = pkg.test_prim(variant, K, t(Z), t(W), na, nb, ma,
                                   t(ZV) if values else None, t(WV) if values else None)
    torch.cuda.synchronize()
    h = lambda a: None if a is None else a.cpu().numpy().view(np.uint32)
    xk, xv, yk, yv = h(xk), h(xv), h(yk), h(yv)
    for c, (na_, nb_, ma_, kz, kw) in enumerate(cases):
        wx, _, wy, _ = oracle.sort_split(Z[c, :na_], ZV[c, :na_], W[c, :nb_], WV[c, :nb_], ma_)
        gx, gy = xk[c, :ma_], yk[c, :na_ + nb_ - ma_]
        assert np.array_equal(gx, wx), (variant, K, values, na_, nb_, ma_, kz, kw, "X")
        assert np.array_equal(gy, wy), (variant, K, values, na_, nb_, ma_, kz, kw, "Y")
        if values:
            pin = sorted(zip(np.concatenate([Z[c, :na_], W[c, :nb_]]).tolist(),
                             np.concatenate([ZV[c, :na_], WV[c, :nb_]]).tolist()))
            pout = sorted(zip(np.concatenate([gx, gy]).tolist(),
                              np.concatenate([xv[c, :ma_], yv[c, :na_ + nb_ - ma_]]).tolist()))
            assert pin == pout, (variant, K, na_, nb_, ma_, kz, kw, "value pairing")


@pytest.mark.parametrize("values", [False, True])
@pytest.mark.parametrize("K", VALID_K)
@pytest.mark.parametrize("variant", [0, 1, 2])
def test_sort_split_grid(variant, K, values):
    _run_split(variant, K, values, _grid(K), seed=1000 + K + variant)


@pytest.mark.parametrize("K,values", [(2048, False), (2048, True), (4096, False)])
def test_sort_split_grid_large_k(K, values):
    """K beyond the paper's 1K (NEXT-3): the lock / pipeline executions' SORT_SPLIT."""
    _run_split(0, K, values, _grid(K), seed=3000 + K)


@pytest.mark.parametrize("K", [512, 1024])
@pytest.mark.parametrize("variant", [0, 1])
def test_bitonic_split_full_random(variant, K):
    """The search-free bitonic split runs only for full keys-only batches at K >= 512: many
    random full cases so every compare-exchange stage sees both outcomes."""
    cases = [(K, K, K, kz, kw) for kz, kw in [("uniform", "uniform"), ("dups", "uniform"), ("low", "high"),
                                             ("high", "low"), ("max", "dups")] for _ in range(40)]
    _run_split(variant, K, False, cases, seed=77 + K)


@pytest.mark.parametrize("K,values", [(k, v) for k in VALID_K for v in (False, True)] +
                         [(2048, False), (2048, True), (4096, False)])
def test_cta_sort(K, values):
    rng = np.random.default_rng(K)
    sizes = sorted(set([1, 2, 31, 32, 33, 63, 64, 65, K // 2, K - 1, K] + list(rng.integers(1, K + 1, 20))))
    sizes = [s for s in sizes if 1 <= s <= K]
    n = len(sizes)
    Z = np.zeros((n, K), np.uint32)
    ZV = np.zeros((n, K), np.uint32)
    for c, s in enumerate(sizes):
        kind = ["uniform", "dups", "max", "equal"][c % 4]
        Z[c, :s] = rng.permutation(_case_keys(rng, s, kind))
        ZV[c, :s] = np.arange(s)
    t = lambda a: torch.from_numpy(a.view(np.int32)).cuda()
    na = torch.tensor(sizes, dtype=torch.int32, device="cuda")
    zero = torch.zeros(n, dtype=torch.int32, device="cuda")
    xk, xv, _, _ = pkg.test_prim(3, K, t(Z), t(Z), na, zero, na, t(ZV) if values else None,
                                 t(ZV) if values else None)
    torch.cuda.synchronize()
    xk = xk.cpu().numpy().view(np.uint32)
    xv = xv.cpu().numpy().view(np.uint32) if values else None
    for c, s in enumerate(sizes):
        assert np.array_equal(xk[c, :s], np.sort(Z[c, :s])), (K, s)
        if values:
            assert np.array_equal(Z[c, xv[c, :s]], xk[c, :s]), (K, s, "pairing")
            assert np.array_equal(np.sort(xv[c, :s]), np.arange(s)), (K, s, "permutation")
