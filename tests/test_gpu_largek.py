"""GPU parity at node capacities beyond the paper's 1K ("Due to the
limits in shared memory size per thread block, the maximum batch size we used is 1K"): K = 2048
(keys and values) and K = 4096 (keys only) on B200's 227 KB of shared memory per CTA.  The INSERT
level pipeline runs with 12 or 24 node slots per stage, DELETEMIN calls on the cluster engine
(K = 2048 keys only) and the per-node-lock engine for the rest.  -m gpu."""
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


@pytest.mark.parametrize("K,values", [(2048, False), (2048, True), (4096, False)])
@pytest.mark.parametrize("dist", ["uniform", "ascending", "descending", "gaussian", "dups"])
@pytest.mark.parametrize("nodes", [40, 1300])
def test_large_k_phased_sorted(K, values, dist, nodes):
    n = nodes * K + 37
    keys = synth.keys(n, seed=synth.SEEDS["C3"] + K, dist=dist)
    q = pkg.BGPQ(capacity=n, K=K, values=values)
    for rep in range(2):  # fresh heap, then the drained-root state
        q.insert(_dev(keys), _dev(synth.values(n)) if values else None)
        assert q.size() == n
        assert _inv(q) == (0, 0)
        ok, ov = q.deletemin(n)
        outk = _host(ok)
        assert np.array_equal(outk, np.sort(keys)), rep
        if values:
            assert np.array_equal(keys[_host(ov)], outk)
        assert q.size() == 0
    q.close()


@pytest.mark.parametrize("K,values", [(2048, True), (4096, False)])
def test_large_k_call_sequence_vs_oracle(K, values):
    rng = np.random.default_rng(K)
    q = pkg.BGPQ(capacity=1600 * K, K=K, values=values)
    ref = oracle.OraclePQ()
    base = 0
    allk = np.empty(0, np.uint32)
    for kind, n in [("ins", 1300 * K + 11), ("del", 200 * K + 5), ("del", 3), ("ins", 77), ("del", 900 * K),
                    ("ins", 250 * K), ("del", 1600 * K)]:
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
            assert np.array_equal(_host(ok)[:c], want), (kind, n)
            if values:
                assert np.array_equal(allk[_host(ov)[:c]], want)
        assert q.size() == ref.size()
        assert _inv(q) == (0, 0)
    q.close()


def test_k4096_values_rejected():
    with pytest.raises(ValueError):
        pkg.BGPQ(capacity=1 << 20, K=4096, values=True)
    assert pkg.lib().bgpq_create_ex(1 << 20, 4096, pkg.FLAG_VALUES) is None
    assert pkg.lib().bgpq_last_error() == pkg.BGPQ_EINVAL
