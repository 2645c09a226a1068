"""GPU parity of the cluster DELETEMIN engine (csrc/bgpq_dsys.cuh: 5-CTA systolic cluster for
the steady state of deletemin calls, heapSize >= 1026, |root| = K, empty pBuffer; the top-CTA
kernel finishes each call).  -m gpu.

Every call is compared bit-exactly with the closed form / the multiset oracle;
values by pairing (R9); quiescent heaps by the invariant checker.  The distributions drive the
engine's rare paths: all-equal keys stop every walk at the root (Alg.3 l.4: message ASTOP
down the cluster), duplicate-heavy keys make the (cur, y) SORT_SPLIT (l.12) merge instead of
swap, ascending / descending inputs give no-op l/r splits (l.10)."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_icpp_chenhjz21_b200 as pkg


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).cuda()


def _host(t):
    return t.cpu().numpy().view(np.uint32)


def _inv(q):
    nk, _, meta, h = q.dump()
    states = pkg.to_oracle_states(meta[:, 1])
    return oracle.check_invariants(q.K, q.slots() - 1, h["heapSize"], h["rootSize"], h["pbSize"], nk, states)


def _keys(n, dist, seed):
    if dist == "equal":
        return np.full(n, 123456789, np.uint32)
    if dist == "two":
        return (synth.keys(n, seed) & np.uint32(1)).astype(np.uint32)
    return synth.keys(n, seed=seed, dist=dist)


@pytest.mark.parametrize("values", [False, True])
@pytest.mark.parametrize("dist", ["uniform", "ascending", "descending", "gaussian", "dups", "equal", "two"])
@pytest.mark.parametrize("K", [256, 1024])
def test_cluster_engine_phased_and_partial(K, dist, values):
    n = 1400 * K + 77
    keys = _keys(n, dist, seed=900 + K)
    q = pkg.BGPQ(capacity=n, K=K, values=values)
    q.insert(_dev(keys), _dev(synth.values(n)) if values else None)
    srt = np.sort(keys)
    done = 0
    for m in [150 * K, 7, 90 * K + 3, n]:          # the first call runs on the cluster engine
        l0 = pkg.launch_count()
        ok, ov = q.deletemin(m)
        launched = pkg.launch_count() - l0
        take = min(m, n - done)
        got = _host(ok)[:take]
        assert np.array_equal(got, srt[done:done + take]), (dist, K, m)
        if values:
            assert np.array_equal(keys[_host(ov)[:take]], got)
        done += take
        assert q.size() == n - done
        assert _inv(q) == (0, 0)
        if m == 150 * K:
            assert launched == 2  # cluster engine + top CTA
    q.close()


@pytest.mark.parametrize("K,values", [(512, False), (512, True), (256, True)])
def test_cluster_engine_call_sequence_vs_oracle(K, values):
    """Insert / deletemin calls of ragged sizes across the engine's boundary (heapSize 1026
    both ways, |root| < K after partial batches, non-empty pBuffer), call by call vs the oracle."""
    rng = np.random.default_rng(K)
    q = pkg.BGPQ(capacity=4000 * K, K=K, values=values)
    ref = oracle.OraclePQ()
    base = 0
    allk = np.empty(0, np.uint32)
    plan = [("ins", 2000 * K), ("del", 600 * K), ("del", 3), ("del", 300 * K), ("ins", 1500 * K + 9),
            ("del", 1000 * K), ("ins", 5), ("del", 2200 * K), ("del", 4000 * K)]
    for kind, n in plan:
        if kind == "ins":
            keys = synth.keys(n, seed=int(rng.integers(1 << 30)))
            vals = np.arange(base, base + n, dtype=np.uint32)
            base += n
            q.insert(_dev(keys), _dev(vals) if values else None)
            ref.insert(keys, vals)
            allk = np.concatenate([allk, keys])
        else:
            want, _ = ref.deletemin(n)
            cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
            ok, ov = q.deletemin(n, d_count=cnt)
            c = int(cnt.item())
            assert c == len(want)
            got = _host(ok)[:c]
            assert np.array_equal(got, want), (kind, n)
            if values:
                assert np.array_equal(allk[_host(ov)[:c]], got)
        assert q.size() == ref.size()
        assert _inv(q) == (0, 0)
    q.close()


def test_cluster_engine_disabled_switch_same_output():
    """bgpq_set_debug bit 256 routes deletemin calls to the top CTA alone: same output."""
    K, n = 1024, 1 << 22
    keys = synth.keys(n, seed=17)
    outs = []
    for bits in (0, 256):
        pkg.set_debug(bits)
        try:
            q = pkg.BGPQ(capacity=n, K=K, values=False)
            q.insert(_dev(keys))
            ok, _ = q.deletemin(n)
            outs.append(_host(ok))
            q.close()
        finally:
            pkg.set_debug(0)
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], np.sort(keys))


@pytest.mark.parametrize("K,values", [(1024, False), (256, True)])
def test_cluster_engine_reused_heap_root_empty(K, values):
    """After a full drain the heap keeps heapSize = 1 with an empty root (R4); the next insert
    call leaves |root| = 0 and every DELETEMIN then refills the root and extracts all K keys
    after the heapify (Alg.2 l.4-14, Alg.3 l.5-6 / l.13).  The engine runs in that regime too."""
    n = 1500 * K + 3
    q = pkg.BGPQ(capacity=n, K=K, values=values)
    for rep in range(3):
        keys = synth.keys(n, seed=70 + rep, dist="uniform" if rep != 1 else "dups")
        q.insert(_dev(keys), _dev(synth.values(n)) if values else None)
        if rep:
            assert q.dump()[3]["rootSize"] == 0
        l0 = pkg.launch_count()
        ok, ov = q.deletemin(n)
        assert pkg.launch_count() - l0 == 2
        out = _host(ok)
        assert np.array_equal(out, np.sort(keys)), rep
        if values:
            assert np.array_equal(keys[_host(ov)], out)
        assert q.size() == 0
    q.close()
