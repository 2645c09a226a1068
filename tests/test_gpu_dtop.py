"""GPU parity of the default DELETEMIN execution (top CTA + walkers, bgpq_dtop.cuh) against
the CPU oracle.  -m gpu.

The top CTA changes mode with the heap size (pipelined with the refill node taken one slot
ahead while heapSize >= 64, synchronous below), keeps the root / pBuffer / depths 1-2 on chip
for the whole call and writes them back at the end, and must handle |root| = 0 (a drained heap
keeps heapSize = 1, reading R4), partial batches, and calls that end mid-heap.  Every call is
compared bit-exactly (keys) with the multiset oracle (deletemin(m) returns the m
smallest, ascending); values by pairing (R9); quiescent heaps by the invariant checker.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_icpp_chenhjz21_b200 as pkg


def _dev(a: np.ndarray):
    return torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).cuda()


def _host(t):
    return t.cpu().numpy().view(np.uint32)


def _inv(q):
    nk, _, meta, h = q.dump()
    states = pkg.to_oracle_states(meta[:, 1])
    return oracle.check_invariants(q.K, q.slots() - 1, h["heapSize"], h["rootSize"], h["pbSize"], nk, states)


@pytest.mark.parametrize("K,values,dist", [(64, True, "uniform"), (128, False, "uniform"), (512, False, "uniform"),
                                           (512, True, "uniform"), (1024, True, "uniform"),
                                           (1024, False, "uniform"), (256, False, "gaussian"),
                                           (1024, False, "gaussian"), (512, True, "gaussian")])
def test_call_sequence_vs_oracle(K, values, dist):
    """Random insert / deletemin calls of ragged sizes on one heap, call by call vs the oracle:
    crosses the pipelined / synchronous boundary (heapSize 64) in both directions, drains to
    empty (|root| = 0 afterwards) and refills."""
    rng = np.random.default_rng(K + values)
    cap = 600 * K
    q = pkg.BGPQ(capacity=cap, K=K, values=values)
    ref = oracle.OraclePQ()
    base = 0
    allk = np.empty(0, np.uint32)
    plan = [("ins", 300 * K + 17), ("del", 7 * K + 3), ("del", 150 * K), ("ins", 2 * K - 5),
            ("del", 200 * K + 999), ("del", 10 * K), ("ins", 250 * K), ("del", 1), ("del", K - 1),
            ("del", 600 * K), ("ins", 90 * K + 33), ("del", 45 * K), ("del", 600 * K)]
    for kind, n in plan:
        if kind == "ins":
            keys = synth.keys(n, seed=int(rng.integers(1 << 30)), dist=dist)
            keys = (keys % np.uint32(1 << 20)).astype(np.uint32) if K == 128 else keys  # duplicates
            vals = np.arange(base, base + n, dtype=np.uint32)
            base += n
            q.insert(_dev(keys), _dev(vals) if values else None)
            ref.insert(keys, vals)
            allk = np.concatenate([allk, keys])
        else:
            want_k, _ = ref.deletemin(n)
            cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
            ok, ov = q.deletemin(n, d_count=cnt)
            c = int(cnt.item())
            assert c == len(want_k)
            got = _host(ok)[:c]
            assert np.array_equal(got, want_k), (kind, n)
            if values:
                assert np.array_equal(allk[_host(ov)[:c]], got)
        assert q.size() == ref.size()
        assert _inv(q) == (0, 0)
    q.close()


@pytest.mark.parametrize("K", [64, 1024])
def test_reused_heap_drain_cycles(K):
    """insert-all / deletemin-all three times on one handle: after the first drain the root
    stays empty (R4), the state the benchmark's timed steps run in."""
    n = 200 * K + 5
    q = pkg.BGPQ(capacity=n, K=K, values=True)
    for rep in range(3):
        keys = synth.keys(n, seed=40 + rep)
        vals = synth.values(n)
        q.insert(_dev(keys), _dev(vals))
        assert _inv(q) == (0, 0)
        ok, ov = q.deletemin(n)
        outk, outv = _host(ok), _host(ov)
        assert np.array_equal(outk, np.sort(keys))
        assert np.array_equal(keys[outv], outk)
        assert np.array_equal(np.sort(outv), np.arange(n, dtype=np.uint32))
        assert q.size() == 0
    q.close()


@pytest.mark.parametrize("dist", ["uniform", "ascending", "descending", "dups"])
def test_partial_drain_leaves_valid_heap(dist):
    """A call that stops mid-heap writes the on-chip part back: the dumped heap satisfies the
    structural invariants and the remainder drains to the rest of sorted(input)."""
    K = 256
    n = 500 * K + 77
    keys = synth.keys(n, seed=5, dist=dist)
    q = pkg.BGPQ(capacity=n, K=K, values=False)
    q.insert(_dev(keys))
    srt = np.sort(keys)
    done = 0
    for m in [3 * K, 61 * K + 9, 1, 100 * K, K - 1]:
        ok, _ = q.deletemin(m)
        assert np.array_equal(_host(ok), srt[done:done + m])
        done += m
        assert q.size() == n - done
        assert _inv(q) == (0, 0)
    ok, _ = q.deletemin(n)
    assert np.array_equal(_host(ok)[:n - done], srt[done:])
    q.close()


def test_stats_count_every_level():
    """The device counters feed bench.py's byte model: every DELETEMIN op is counted once and
    every heapify level once (top CTA + walkers)."""
    K, n = 1024, 1 << 20
    keys = synth.keys(n, seed=9)
    q = pkg.BGPQ(capacity=n, K=K, values=False)
    q.insert(_dev(keys))
    s0 = q.stats()
    q.deletemin(n)
    s1 = q.stats()
    d = {k: s1[k] - s0[k] for k in s1}
    assert d["del_ops"] == n // K
    assert d["keys_out"] == n
    # 1024 nodes: a walk has at most log2(1024) = 10 levels and almost every op goes deep
    assert 5 * (n // K) < d["del_levels"] <= 10 * (n // K)
    q.close()


def test_reused_heap_full_size_multiset():
    """C2 size, heap reused across drains (|root| = 0 state): after every INSERT call the keys
    stored in the heap (root, pBuffer, nodes 2..heapSize) are exactly the input multiset, and the
    drain returns sorted(input).  Guards the insert pipeline's write-back ordering, which the
    structural invariants alone cannot see (a lost key leaves a valid heap)."""
    n, K = 1 << 27, 1024
    keys = synth.keys(n, seed=synth.SEEDS["C2"])
    srt = np.sort(keys)
    q = pkg.BGPQ(capacity=n, K=K, values=False)
    dk = _dev(keys)
    for rep in range(2):
        q.insert(dk)
        nk, _, _, h = q.dump()
        hs, rs, ps = h["heapSize"], h["rootSize"], h["pbSize"]
        nk2 = nk.reshape(-1, K)
        parts = [nk2[1, :rs], nk2[0, :ps]] + ([nk2[2:hs + 1].ravel()] if hs >= 2 else [])
        assert np.array_equal(np.sort(np.concatenate(parts)), srt), rep
        ok, _ = q.deletemin(n)
        assert np.array_equal(_host(ok), srt), rep
    q.close()
