"""GPU parity of mixed calls on the cluster engine (bgpq_dsys.cuh: bgpq_msort_kernel +
ds_r0_mixed, reading R26): op streams that start with (INSERT(K), DELETEMIN(K)) pairs — the
utilisation workload — run those pairs on the 5-CTA cluster, the rest of the call on
the per-node-lock engine.  Every DELETEMIN is compared bit-exactly with the oracle replayed
in linearization-ticket order; values by pairing; heap invariants and the remaining
multiset after the call.  -m gpu."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_icpp_chenhjz21_b200 as pkg

from test_gpu_parity import _dev, _host, _gpu_inv, _mixed_inputs, _run_mixed, _replay_check


def _prefilled(K, values, n_pre, regime, seed=100):
    """A heap holding n_pre keys with |root| = K ("full": built on a fresh heap) or |root| = 0
    ("drained": built after a drain, R4)."""
    pre = synth.keys(n_pre, seed=seed)
    q = pkg.BGPQ(capacity=2 * n_pre + 4096 * K, K=K, values=values)
    pv = _dev(synth.values(n_pre)) if values else None
    if regime == "drained":
        q.insert(_dev(pre), pv)
        q.deletemin(n_pre)
    q.insert(_dev(pre), pv)
    torch.cuda.synchronize()
    h = q.dump()[3]
    assert h["rootSize"] == (0 if regime == "drained" else K) and h["pbSize"] == 0
    return q, pre


def _check_rest(q, ref):
    assert _gpu_inv(q) == (0, 0)
    assert q.size() == ref.size()
    rest, _ = q.deletemin(q.size() + 1)
    rk, _ = ref.deletemin(ref.size())
    assert np.array_equal(_host(rest)[:len(rk)], rk)


@pytest.mark.parametrize("K,values", [(256, False), (512, True), (1024, False), (1024, True), (2048, False)])
@pytest.mark.parametrize("regime", ["full", "drained"])
def test_mixed_pairs_cluster_replay(K, values, regime):
    n_pairs = 700
    q, pre = _prefilled(K, values, 200 * K, regime)
    types, sizes = synth.mixed_ops(n_pairs, K, seed=101)
    keys, in_off = _mixed_inputs(types, sizes, K, seed=102)
    st0, l0 = q.stats(), pkg.launch_count()
    outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
    st1 = q.stats()
    assert pkg.launch_count() - l0 == 3  # sort kernel, cluster engine, lock engine (empty rest)
    assert st1["marked"] - st0["marked"] == n_pairs  # every pair ran on the cluster engine
    assert np.array_equal(lin - lin.min(), np.arange(len(types)))  # linearization = call order
    ref = _replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin - lin.min(), prefill=pre)
    if values:  # inserted batches carry their input index, the prefill its own index
        for j in np.nonzero(types == 1)[0]:
            v, k = outv[j, :cnt[j]].astype(np.int64), outk[j, :cnt[j]]
            ins = (v < len(keys)) & (keys[np.minimum(v, len(keys) - 1)] == k)
            pref = (v < len(pre)) & (pre[np.minimum(v, len(pre) - 1)] == k)
            assert (ins | pref).all(), f"op {j}: value pairing"
    _check_rest(q, ref)


@pytest.mark.parametrize("K", [256, 1024])
def test_mixed_pairs_then_random_ops(K):
    """The engine runs the leading pairs; the per-node-lock engine continues with arbitrary ops
    (random types, sizes 1..K) at the op the engine stopped at."""
    q, pre = _prefilled(K, True, 150 * K, "full", seed=110)
    t1, s1 = synth.mixed_ops(300, K, seed=111)
    t2, s2 = synth.random_ops(400, K, seed=112, p_insert=0.5)
    types, sizes = np.concatenate([t1, t2]), np.concatenate([s1, s2])
    keys, in_off = _mixed_inputs(types, sizes, K, seed=113)
    st0 = q.stats()
    outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
    assert q.stats()["marked"] - st0["marked"] >= 300
    assert np.array_equal(lin[:600] - lin.min(), np.arange(600))
    ref = _replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin - lin.min(), prefill=pre)
    _check_rest(q, ref)


@pytest.mark.parametrize("K", [512])
def test_mixed_pair_stream_broken_in_the_middle(K):
    """A partial INSERT in the middle of the pair stream ends the engine's part there."""
    q, pre = _prefilled(K, False, 120 * K, "drained", seed=120)
    types, sizes = synth.mixed_ops(500, K, seed=121)
    sizes = sizes.copy()
    sizes[2 * 173] = K - 5
    keys, in_off = _mixed_inputs(types, sizes, K, seed=122)
    st0 = q.stats()
    outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
    assert q.stats()["marked"] - st0["marked"] >= 173
    ref = _replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin - lin.min(), prefill=pre)
    _check_rest(q, ref)


@pytest.mark.parametrize("dist", ["ascending", "descending", "dups"])
def test_mixed_pairs_key_distributions(dist):
    """Sorted and duplicate-heavy inserted batches: the INSERT's root / depth-1 splits become
    swaps or all-equal merges, the carried items are rewritten on chip (dirty) before they
    sink by reference."""
    K = 1024
    q, pre = _prefilled(K, False, 100 * K, "full", seed=130)
    types, sizes = synth.mixed_ops(400, K, seed=131)
    keys, in_off = _mixed_inputs(types, sizes, K, seed=132, dist=dist)
    outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
    ref = _replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin - lin.min(), prefill=pre)
    _check_rest(q, ref)


def test_mixed_small_heap_uses_lock_engine():
    """heapSize below the engine's floor: the whole call runs on the per-node-lock engine."""
    K = 256
    q, pre = _prefilled(K, False, 20 * K, "full", seed=140)
    types, sizes = synth.mixed_ops(200, K, seed=141)
    keys, in_off = _mixed_inputs(types, sizes, K, seed=142)
    outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
    ref = _replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin - lin.min(), prefill=pre)
    _check_rest(q, ref)
