"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.  -m gpu.

Bit-exact for keys (integer work).  Values: several assignments are correct for equal
keys (R9), so values are checked by pairing (key == input_key[val]) and conservation.
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


def _gpu_inv(q):
    nk, _, meta, h = q.dump()
    states = pkg.to_oracle_states(meta[:, 1])
    return oracle.check_invariants(q.K, q.slots() - 1, h["heapSize"], h["rootSize"], h["pbSize"], nk, states)


# --------------------------------------------------------------------------------------
# phased insert-all then deletemin-all: output == sorted(input) (closed form, §8(c))
# --------------------------------------------------------------------------------------
MODES = ["default", "locks"]


def _mode(mode):
    """default: INSERT calls as the level pipeline + top-CTA DELETEMIN with walkers; locks: paper-literal
    per-node locks for every call."""
    return {"locks": mode == "locks"}


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("K", [64, 128, 256, 512, 1024])
@pytest.mark.parametrize("dist", ["uniform", "ascending", "descending", "gaussian", "dups"])
def test_phased_sorted(K, dist, mode):
    n = 40 * K + 37  # several tiles and a ragged tail
    keys = synth.keys(n, seed=synth.SEEDS["C3"], dist=dist)
    vals = synth.values(n)
    q = pkg.BGPQ(capacity=n, K=K, values=True, **_mode(mode))
    q.insert(_dev(keys), _dev(vals))
    assert q.size() == n
    assert _gpu_inv(q) == (0, 0)
    ok, ov = q.deletemin(n)
    outk, outv = _host(ok), _host(ov)
    assert np.array_equal(outk, oracle.pq_phased(keys, K))
    assert np.array_equal(keys[outv], outk)
    assert np.array_equal(np.sort(outv), np.arange(n, dtype=np.uint32))
    assert q.size() == 0
    q.close()


@pytest.mark.parametrize("values", [False, True])
@pytest.mark.parametrize("K", [64, 128, 256, 512, 1024])
@pytest.mark.parametrize("dist", ["uniform", "ascending", "descending", "gaussian", "dups"])
def test_phased_sorted_pipelined(K, dist, values):
    """heapSize >= 64 (300 nodes): the top CTA runs its pipelined mode (refill taken one slot
    ahead, depths 0-2 on chip, walkers below) for most of the drain; keys-only at K >= 512 takes
    the bitonic SORT_SPLIT in the insert pipeline, the top CTA's groups and the walkers."""
    n = 300 * K + 17
    keys = synth.keys(n, seed=synth.SEEDS["C3"] + K, dist=dist)
    q = pkg.BGPQ(capacity=n, K=K, values=values)
    q.insert(_dev(keys), _dev(synth.values(n)) if values else None)
    assert q.size() == n
    ok, ov = q.deletemin(n)
    outk = _host(ok)
    assert np.array_equal(outk, np.sort(keys))
    if values:
        outv = _host(ov)
        assert np.array_equal(keys[outv], outk)
        assert np.array_equal(np.sort(outv), np.arange(n, dtype=np.uint32))
    assert q.size() == 0
    q.close()


@pytest.mark.parametrize("dist", ["uniform", "ascending", "descending", "gaussian"])
def test_c3_matrix_full_size(dist):
    """Config C3 in full (BASELINE configs[2]): 2^26 keys of each distribution at K in
    {128, 256, 512, 1024}, keys only, phased insert-all / deletemin-all on one handle per K;
    the concatenated output must equal sorted(input) (closed form, §8(c))."""
    n = 1 << 26
    keys = synth.keys(n, seed=synth.SEEDS["C3"], dist=dist)
    srt = np.sort(keys)
    dk = _dev(keys)
    for K in (128, 256, 512, 1024):
        q = pkg.BGPQ(capacity=n, K=K, values=False)
        q.insert(dk)
        assert q.size() == n
        ok, _ = q.deletemin(n)
        assert np.array_equal(_host(ok), srt), (dist, K)
        assert q.size() == 0
        q.close()
        del ok


def test_phased_c1_keys_only():
    """Config C1: 2^16 uniform keys, K = 64, keys only (w = 4)."""
    n, K = 1 << 16, 64
    keys = synth.keys(n, seed=synth.SEEDS["C1"])
    q = pkg.BGPQ(capacity=n, K=K, values=False)
    q.insert(_dev(keys))
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    ok, _ = q.deletemin(n, d_count=cnt)
    assert int(cnt.item()) == n
    assert np.array_equal(_host(ok), oracle.pq_phased(keys, K))
    st = q.stats()
    assert st["ins_heapify_ops"] == n // K - 1 and st["del_refill_ops"] == n // K - 1


# --------------------------------------------------------------------------------------
# serialized mode (1 CTA): node layout bit-exact against the sequential Alg.1-3 model
# --------------------------------------------------------------------------------------
def _compare_layout(q, seq):
    nk, _, meta, h = q.dump()
    sk, _, sst = seq.dump()
    sh = seq.header()
    assert (h["heapSize"], h["rootSize"], h["pbSize"]) == (sh["heapSize"], sh["rootSize"], sh["pbSize"])
    gst = pkg.to_oracle_states(meta[:, 1])
    assert np.array_equal(gst[2:], sst[2:])
    assert np.array_equal(nk[1, :h["rootSize"]], sk[1, :sh["rootSize"]])
    assert np.array_equal(nk[0, :h["pbSize"]], sk[0, :sh["pbSize"]])
    live = np.nonzero(sst[2:] == oracle.AVAIL)[0] + 2
    assert np.array_equal(nk[live], sk[live])


def _compare_counters(q, seq, before=None):
    """Device counters (bench.py's byte model) equal the sequential model's counters."""
    g = q.stats()
    if before is not None:
        g = {k: g[k] - before[k] for k in g}
    g["del_lr_merge"] += g["del_lr_nomove"]  # the GPU splits l/r SORT_SPLITs into moving / no-move
    for k, v in seq.counters().items():
        assert g[k] == v, (k, g[k], v)


@pytest.mark.parametrize("K", [64, 256])
def test_serialized_layout_bitexact_phased(K):
    n = 96 * K + 5
    keys = synth.keys(n, seed=5)
    q = pkg.BGPQ(capacity=n, K=K, values=False, serial=True)
    seq = oracle.SeqBGPQ(K, q.slots() - 1)
    q.insert(_dev(keys))
    for off in range(0, n, K):
        seq.insert(keys[off:off + K])
    _compare_layout(q, seq)
    m = 37 * K
    ok, _ = q.deletemin(m)
    want = np.concatenate([seq.deletemin(K)[0] for _ in range(37)])
    assert np.array_equal(_host(ok), want)
    _compare_layout(q, seq)
    _compare_counters(q, seq)


@pytest.mark.parametrize("K", [64, 512, 1024])
@pytest.mark.parametrize("values", [False, True])
def test_pipelined_insert_layout_bitexact(K, values):
    """INSERT calls run as a level pipeline that applies the batches at every node in call
    order: the heap after the call equals the sequential Alg.1 model node for node, including
    a second call on a non-empty heap with a partial batch and a non-empty pBuffer."""
    n1, n2 = 37 * K + 5, 50 * K + 11
    keys = synth.keys(n1 + n2, seed=9, dist="dups")
    q = pkg.BGPQ(capacity=n1 + n2, K=K, values=values)
    seq = oracle.SeqBGPQ(K, q.slots() - 1)
    for a, b in ((0, n1), (n1, n1 + n2)):
        q.insert(_dev(keys[a:b]), _dev(synth.values(b - a)) if values else None)
        for off in range(a, b, K):
            seq.insert(keys[off:min(off + K, b)])
        _compare_layout(q, seq)
    ok, _ = q.deletemin(n1 + n2)
    assert np.array_equal(_host(ok), np.sort(keys))


def _mixed_inputs(types, sizes, K, seed, dist="uniform"):
    n_in = int(sizes[types == 0].sum())
    keys = synth.keys(max(n_in, 1), seed=seed, dist=dist)
    in_off = np.zeros(len(types), np.uint64)
    off = 0
    for j in range(len(types)):
        if types[j] == 0:
            in_off[j] = off
            off += int(sizes[j])
    return keys, in_off


def _run_mixed(q, types, sizes, keys, in_off):
    K = q.K
    n_ops = len(types)
    vals = synth.values(len(keys))
    out_k = torch.zeros(n_ops * K, dtype=torch.int32, device="cuda")
    out_v = torch.zeros(n_ops * K, dtype=torch.int32, device="cuda")
    cnt = torch.zeros(n_ops, dtype=torch.int32, device="cuda")
    lin = torch.zeros(n_ops, dtype=torch.int64, device="cuda")
    q.run_mixed(torch.from_numpy(types).cuda(), torch.from_numpy(sizes.view(np.int32)).cuda(),
                torch.from_numpy(in_off.view(np.int64)).cuda(), _dev(keys), _dev(vals),
                out_k, out_v, cnt, lin)
    torch.cuda.synchronize()
    return (_host(out_k).reshape(n_ops, K), _host(out_v).reshape(n_ops, K),
            cnt.cpu().numpy(), lin.cpu().numpy())


def test_serialized_mixed_partial_sizes_bitexact():
    K = 64
    types, sizes = synth.random_ops(3000, K, seed=31, p_insert=0.6)
    keys, in_off = _mixed_inputs(types, sizes, K, seed=32, dist="dups")
    q = pkg.BGPQ(capacity=len(keys) + K, K=K, values=True, serial=True)
    seq = oracle.SeqBGPQ(K, q.slots() - 1)
    outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
    assert np.array_equal(np.sort(lin), np.arange(len(types)))  # one CTA: ticket order = op order
    for j in range(len(types)):
        if types[j] == 0:
            seq.insert(keys[in_off[j]:in_off[j] + sizes[j]])
        else:
            want, _ = seq.deletemin(int(sizes[j]))
            assert cnt[j] == len(want)
            assert np.array_equal(outk[j, :cnt[j]], want), f"op {j}"
            assert np.array_equal(keys[outv[j, :cnt[j]]], want)
    _compare_layout(q, seq)


# --------------------------------------------------------------------------------------
# concurrent mixes: replay the linearization log (ticket order) through the oracle
# --------------------------------------------------------------------------------------
def _replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin, prefill=None):
    """Ticket-order replay (the linearization point is in the root section) through
    oracle.replay: every deletemin's keys bit-exact.  Returns the oracle queue after the log."""
    order = np.argsort(lin, kind="stable")
    assert np.array_equal(lin[order], np.arange(len(lin)) + (lin.min() if len(lin) else 0))
    log = [] if prefill is None else [(0, (prefill, None))]
    for j in order:
        if types[j] == 0:
            log.append((0, (keys[in_off[j]:in_off[j] + sizes[j]], None)))
        else:
            log.append((1, int(sizes[j])))
    q = oracle.OraclePQ()
    res = oracle.replay(log, q=q)
    dels = [j for j in order if types[j] == 1]
    assert len(res) == len(dels)
    for j, (want, _) in zip(dels, res):
        got = outk[j, :cnt[j]]
        assert cnt[j] == len(want), f"op {j}: count {cnt[j]} != {len(want)}"
        assert np.array_equal(got, want), f"op {j} (ticket {lin[j]}) differs from replay"
    return q


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("K,p_ins,partial", [(64, 0.5, True), (64, 0.5, False), (128, 0.55, True),
                                             (1024, 0.5, False)])
def test_concurrent_mixed_replay(K, p_ins, partial, mode):
    n_ops = 4000 if K <= 128 else 1200
    if partial:
        types, sizes = synth.random_ops(n_ops, K, seed=41 + K, p_insert=p_ins)
    else:
        types, _ = synth.random_ops(n_ops, K, seed=41 + K, p_insert=p_ins)
        sizes = np.full(n_ops, K, np.uint32)
    keys, in_off = _mixed_inputs(types, sizes, K, seed=43)
    q = pkg.BGPQ(capacity=len(keys) + K, K=K, values=True, **_mode(mode))
    outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
    ref = _replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin)
    for j in np.nonzero(types == 1)[0]:
        assert np.array_equal(keys[outv[j, :cnt[j]]], outk[j, :cnt[j]])  # value pairing
    assert _gpu_inv(q) == (0, 0)
    assert q.size() == ref.size()
    rest, _ = q.deletemin(q.size() + 1)
    rk, _ = ref.deletemin(ref.size())
    assert np.array_equal(_host(rest)[:len(rk)], rk)


@pytest.mark.parametrize("mode", MODES)
def test_concurrent_pairs_with_prefill_replay(mode):
    """Utilisation shape: prefill, then insert/deletemin pairs on all CTAs."""
    K = 64
    pre = synth.keys(1 << 17, seed=50)
    q = pkg.BGPQ(capacity=(1 << 18) + 4096 * K, K=K, values=True, **_mode(mode))
    q.insert(_dev(pre), _dev(synth.values(len(pre))))
    types, sizes = synth.mixed_ops(3000, K, seed=51, partial=True)
    keys, in_off = _mixed_inputs(types, sizes, K, seed=52)
    outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
    _replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin - lin.min(), prefill=pre)
    assert _gpu_inv(q) == (0, 0)


@pytest.mark.parametrize("mode", MODES)
def test_marked_handoff_replay(mode):
    """Small heap, many concurrent full-batch inserts/deletemins: drives the TARGET/MARKED
    collaboration — the replay must stay exact whether or not it fires."""
    K = 64
    total_marked = 0
    for seed in range(4):
        types, _ = synth.random_ops(3000, K, seed=60 + seed, p_insert=0.5)
        sizes = np.full(len(types), K, np.uint32)
        keys, in_off = _mixed_inputs(types, sizes, K, seed=70 + seed)
        q = pkg.BGPQ(capacity=len(keys) + K, K=K, values=True, **_mode(mode))
        outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
        _replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin)
        assert _gpu_inv(q) == (0, 0)
        total_marked += q.stats()["marked"]
    print("MARKED hand-offs observed:", total_marked)
    if mode == "locks":  # every call on the per-node-lock engine: the collaboration must fire
        assert total_marked > 0


def test_forced_collaboration_replay():
    """Schedule forcing (bgpq_set_debug 32768): inserts hold their target node TARGET for 20 us
    before the placement, so concurrent deletemins must steal from in-flight inserts
    (TARGET -> MARKED, Alg.2 l.7-9; the insert then fills the root, Alg.1 l.11-13) and
    walk past a TARGET child (exactly one AVAIL child, R5).  Both paths are asserted to fire
    and the ticket-order replay stays bit-exact."""
    K = 64
    marked = skip = 0
    pkg.set_debug(32768)
    try:
        for seed in range(2):
            types, _ = synth.random_ops(2000, K, seed=80 + seed, p_insert=0.5)
            sizes = np.full(len(types), K, np.uint32)
            keys, in_off = _mixed_inputs(types, sizes, K, seed=90 + seed)
            q = pkg.BGPQ(capacity=len(keys) + K, K=K, values=True, locks=True)
            outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
            _replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin)
            for j in np.nonzero(types == 1)[0]:
                assert np.array_equal(keys[outv[j, :cnt[j]]], outk[j, :cnt[j]])
            assert _gpu_inv(q) == (0, 0)
            st = q.stats()
            marked += st["marked"]
            skip += st["del_lr_skip"]
            q.close()
    finally:
        pkg.set_debug(0)
    print("forced: MARKED", marked, "one-AVAIL-child levels", skip)
    assert marked > 0 and skip > 0


# --------------------------------------------------------------------------------------
# edge cases
# --------------------------------------------------------------------------------------
def test_edge_cases():
    K = 64
    q = pkg.BGPQ(capacity=1000, K=K, values=True)
    cnt = torch.zeros(1, dtype=torch.int64, device="cuda")
    q.deletemin(5, d_count=cnt)                       # empty heap -> nothing (Alg.2 l.16)
    assert int(cnt.item()) == 0 and q.size() == 0
    q.insert(_dev(np.array([7], np.uint32)), _dev(np.array([0], np.uint32)))
    ok, ov = q.deletemin(3, d_count=cnt)              # fewer than asked -> all
    assert int(cnt.item()) == 1 and _host(ok)[0] == 7
    keys = np.array([0xFFFFFFFF, 0, 0xFFFFFFFF, 1, 0xFFFFFFFF], np.uint32)  # extreme keys
    q.insert(_dev(keys), _dev(np.arange(5, dtype=np.uint32)))
    ok, ov = q.deletemin(5)
    assert np.array_equal(_host(ok), np.sort(keys))
    assert np.array_equal(keys[_host(ov)], np.sort(keys))
    q.close()


def test_capacity_overflow_sticky():
    K = 64
    q = pkg.BGPQ(capacity=4 * K, K=K, values=False)
    q.insert(_dev(synth.keys(20 * K, seed=3)))
    with pytest.raises(pkg.BGPQError):
        q.size()


def test_host_api_roundtrip():
    n, K = 10000, 128
    keys = synth.keys(n, seed=8)
    vals = synth.values(n)
    q = pkg.BGPQ(capacity=n, K=K, values=True)
    q.insert_host(keys, vals)
    ok = np.empty(n, np.uint32)
    ov = np.empty(n, np.uint32)
    assert q.deletemin_host(n, ok, ov) == n
    assert np.array_equal(ok, np.sort(keys)) and np.array_equal(keys[ov], ok)


# --------------------------------------------------------------------------------------
# full size: config C2 (2^27 keys, K = 1024) in the launch configuration bench.py times
# --------------------------------------------------------------------------------------
@pytest.mark.parametrize("mode", MODES)
def test_full_size_c2_properties(mode):
    n, K = 1 << 27, 1024
    keys = synth.keys(n, seed=synth.SEEDS["C2"])
    dk = _dev(keys)
    q = pkg.BGPQ(capacity=n, K=K, values=False, **_mode(mode))
    q.insert(dk)
    assert q.size() == n
    ok, _ = q.deletemin(n)
    torch.cuda.synchronize()
    # sampled outputs the oracle computes one by one: batch t holds ranks [tK, (t+1)K)
    srt = np.sort(keys)
    out = _host(ok)
    for t in [0, 1, 2, 1000, 65535, 131070, 131071]:
        assert np.array_equal(out[t * K:(t + 1) * K], srt[t * K:(t + 1) * K])
    # properties at full size: ascending and a permutation of the input
    assert np.all(out[1:] >= out[:-1])
    assert np.array_equal(out, srt)
    assert q.size() == 0


@pytest.mark.parametrize("K", [64, 256, 1024, 4096])
def test_pipelined_insert_reused_small_heap_layout(K):
    """Regression: on a small heap refilled after drains, the level stages revisit the leftmost
    path node of their depth each time tar enters a new depth; the stage's prefetch helper must
    not load it before the compute's write-back of that node retired (keys were lost at K =
    4096).  The layout after every insert call equals the sequential Alg.1 model's."""
    n = 40 * K + 37
    keys = synth.keys(n, seed=synth.SEEDS["C3"] + K)
    q = pkg.BGPQ(capacity=n, K=K, values=False)
    seq = oracle.SeqBGPQ(K, q.slots() - 1)
    for rep in range(5):
        q.insert(_dev(keys))
        for off in range(0, n, K):
            seq.insert(keys[off:min(off + K, n)])
        _compare_layout(q, seq)
        ok, _ = q.deletemin(n)
        want = np.concatenate([seq.deletemin(K)[0] for _ in range((n + K - 1) // K)])
        assert np.array_equal(_host(ok), want), rep
    q.close()
