"""Pins for the CPU oracle (oracle/), run with -m "not gpu".

Each test pins an oracle function to something other than itself: the paper's own
definitions and invariants, hand-traced golden sequences
(tests/golden/, derived by hand from Alg.1-3), brute force on tiny inputs (a Python
list), the textbook binary heap (heapq) for single-key operations, and the closed form
"phased output == sorted(input)".  Mutation tests show the checks catch plausible bugs.
"""
import collections
import heapq
import os

import numpy as np
import pytest

import oracle
import synth
from conftest import parse_trace

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _state_of(q: oracle.SeqBGPQ):
    keys, _, states = q.dump()
    h = q.header()
    st = {"hs": h["heapSize"], "root": list(keys[1][:h["rootSize"]]),
          "pb": list(keys[0][:h["pbSize"]])}
    for i in range(2, q.cap + 1):
        if states[i] == oracle.AVAIL:
            st[f"n{i}"] = list(keys[i])
    return st


def _check_inv(q: oracle.SeqBGPQ):
    keys, _, states = q.dump()
    h = q.header()
    return oracle.check_invariants(q.K, q.cap, h["heapSize"], h["rootSize"], h["pbSize"], keys, states)


# --------------------------------------------------------------------------------------
# Golden hand traces (stand-in for the lost Fig.2-4 example)
# --------------------------------------------------------------------------------------
@pytest.mark.parametrize("name", ["k4_trace.txt", "k2_trace.txt"])
def test_seq_model_matches_hand_trace(name):
    K, cap, steps = parse_trace(os.path.join(GOLDEN, name))
    q = oracle.SeqBGPQ(K, cap)
    adt = oracle.OraclePQ()
    vid = 0
    for step in steps:
        kind, arg, out, state = step
        if kind == "I":
            vals = np.arange(vid, vid + len(arg), dtype=np.uint32)
            vid += len(arg)
            assert q.insert(arg, vals) == 0
            adt.insert(arg, vals)
        else:
            k, _ = q.deletemin(arg)
            assert list(k) == out, f"deletemin({arg}) output"
            ak, _ = adt.deletemin(arg)
            assert list(ak) == out, "ADT oracle disagrees with the hand trace"
        got = _state_of(q)
        assert got == state, f"state after {kind} {arg}: {got} != {state}"
        assert _check_inv(q) == (0, 0)


def test_tie_rule_is_load_bearing_in_golden():
    """Reversing x/y (mutation 1) must diverge from the k2 hand trace (pins R6)."""
    K, cap, steps = parse_trace(os.path.join(GOLDEN, "k2_trace.txt"))
    q = oracle.SeqBGPQ(K, cap, mutation=1)
    diverged = False
    for kind, arg, out, state in steps:
        if kind == "I":
            q.insert(arg)
        else:
            q.deletemin(arg)
        if _state_of(q) != state:
            diverged = True
            break
    assert diverged


# --------------------------------------------------------------------------------------
# SORT_SPLIT: postconditions of P:196-198
# --------------------------------------------------------------------------------------
def _ss_post(zk, zv, wk, wv, ma, xk, xv, yk, yv):
    assert len(xk) == ma and len(yk) == len(zk) + len(wk) - ma           # Ma + Mb = Na + Nb
    assert np.all(np.diff(xk.astype(np.int64)) >= 0)                     # X sorted
    assert np.all(np.diff(yk.astype(np.int64)) >= 0)                     # Y sorted
    if len(xk) and len(yk):
        assert xk.max() <= yk.min()                                      # max X <= min Y
    inp = collections.Counter(zip(list(zk) + list(wk), list(zv) + list(wv)))
    outp = collections.Counter(zip(list(xk) + list(yk), list(xv) + list(yv)))
    assert inp == outp                                                   # (X, Y) = sorted(Z, W)


def test_sort_split_exhaustive_small():
    rng = np.random.default_rng(0)
    for na in range(0, 5):
        for nb in range(0, 5):
            for ma in range(0, na + nb + 1):
                for _ in range(4):
                    zk = np.sort(rng.integers(0, 4, na)).astype(np.uint32)
                    wk = np.sort(rng.integers(0, 4, nb)).astype(np.uint32)
                    zv = np.arange(na, dtype=np.uint32)
                    wv = np.arange(100, 100 + nb, dtype=np.uint32)
                    xk, xv, yk, yv = oracle.sort_split(zk, zv, wk, wv, ma)
                    _ss_post(zk, zv, wk, wv, ma, xk, xv, yk, yv)


def test_sort_split_random_large():
    rng = np.random.default_rng(1)
    for _ in range(200):
        na, nb = rng.integers(0, 1025, 2)
        ma = int(rng.integers(0, na + nb + 1))
        hi = int(rng.choice([3, 1000, 2 ** 32]))
        zk = np.sort(rng.integers(0, hi, na, dtype=np.uint64)).astype(np.uint32)
        wk = np.sort(rng.integers(0, hi, nb, dtype=np.uint64)).astype(np.uint32)
        zv = rng.integers(0, 2 ** 32, na, dtype=np.uint64).astype(np.uint32)
        wv = rng.integers(0, 2 ** 32, nb, dtype=np.uint64).astype(np.uint32)
        xk, xv, yk, yv = oracle.sort_split(zk, zv, wk, wv, ma)
        _ss_post(zk, zv, wk, wv, ma, xk, xv, yk, yv)


def test_sort_split_rejects_bad_ma():
    with pytest.raises(ValueError):
        oracle.sort_split([1], [0], [2], [0], 3)


# --------------------------------------------------------------------------------------
# OracleBPQ: brute force, heapq, closed form
# --------------------------------------------------------------------------------------
def test_oracle_pq_vs_bruteforce():
    rng = np.random.default_rng(2)
    for trial in range(50):
        q = oracle.OraclePQ()
        brute = []  # plain Python list, re-sorted after each op
        for _ in range(60):
            if rng.random() < 0.55:
                ks = rng.integers(0, 20, int(rng.integers(1, 6))).astype(np.uint32)
                q.insert(ks)
                brute = sorted(brute + [int(k) for k in ks])
            else:
                m = int(rng.integers(1, 6))
                got, _ = q.deletemin(m)
                want, brute = brute[:m], brute[m:]
                assert list(got) == want
            assert q.size() == len(brute)


def test_oracle_pq_single_key_matches_heapq():
    rng = np.random.default_rng(3)
    q = oracle.OraclePQ()
    h = []
    for _ in range(3000):
        if rng.random() < 0.6:
            k = int(rng.integers(0, 2 ** 32))
            q.insert([k])
            heapq.heappush(h, k)
        elif h:
            got, _ = q.deletemin(1)
            assert int(got[0]) == heapq.heappop(h)


def test_oracle_pq_phased_closed_form():
    keys = synth.keys(1 << 16, seed=1)
    out = oracle.pq_phased(keys, 64)
    assert np.array_equal(out, np.sort(keys))


def test_oracle_pq_value_pairing():
    keys = synth.keys(5000, seed=7, dist="dups")
    vals = synth.values(5000)
    q = oracle.OraclePQ()
    q.insert(keys, vals)
    k, v = q.deletemin(5000)
    assert np.array_equal(k, np.sort(keys))
    assert np.array_equal(keys[v], k)
    assert sorted(v.tolist()) == list(range(5000))


# --------------------------------------------------------------------------------------
# SeqBGPQ (Alg.1-3) vs the ADT, with invariants after every op
# --------------------------------------------------------------------------------------
def _random_run(K, n_ops, seed, key_hi, cap=None, mutation=0, check_every=1):
    rng = np.random.default_rng(seed)
    cap = cap or (n_ops + 4)
    q = oracle.SeqBGPQ(K, cap, mutation=mutation)
    ref = oracle.OraclePQ()
    vid = 0
    bad_out = bad_inv = 0
    for i in range(n_ops):
        if rng.random() < 0.55:
            s = int(rng.integers(1, K + 1))
            ks = rng.integers(0, key_hi, s, dtype=np.uint64).astype(np.uint32)
            vs = np.arange(vid, vid + s, dtype=np.uint32)
            vid += s
            q.insert(ks, vs)
            ref.insert(ks, vs)
        else:
            s = int(rng.integers(1, K + 1))
            k, v = q.deletemin(s)
            rk, _ = ref.deletemin(s)
            if not np.array_equal(k, rk):
                bad_out += 1
        if i % check_every == 0 and _check_inv(q)[0] != 0:
            bad_inv += 1
    return q, ref, bad_out, bad_inv


@pytest.mark.parametrize("K", [2, 3, 4, 8])
def test_seq_model_vs_oracle_random(K):
    for seed in range(60):
        q, ref, bad_out, bad_inv = _random_run(K, 200, seed, key_hi=int([50, 2 ** 32][seed % 2]))
        assert bad_out == 0 and bad_inv == 0, (seed, bad_out, bad_inv)
        # drain: multiset conservation + value pairing via the ADT
        rest_k, rest_v = [], []
        while True:
            k, v = q.deletemin(K)
            if len(k) == 0:
                break
            rest_k += list(k); rest_v += list(v)
        rk, _ = ref.deletemin(10 ** 6)
        assert rest_k == list(rk)


def test_seq_model_phased_c1_closed_form():
    """Config C1 (2^16 uniform keys, K=64): the concatenated output equals sorted(input)."""
    n, K = 1 << 16, 64
    keys = synth.keys(n, seed=synth.SEEDS["C1"])
    vals = synth.values(n)
    q = oracle.SeqBGPQ(K, n // K + 2)
    for off in range(0, n, K):
        q.insert(keys[off:off + K], vals[off:off + K])
    assert _check_inv(q) == (0, 0)
    h = q.header()
    assert h["heapSize"] == n // K and h["rootSize"] == K and h["pbSize"] == 0
    outk, outv = [], []
    for _ in range(n // K):
        k, v = q.deletemin(K)
        assert len(k) == K
        outk.append(k); outv.append(v)
    outk = np.concatenate(outk); outv = np.concatenate(outv)
    assert np.array_equal(outk, np.sort(keys))
    assert np.array_equal(keys[outv], outk)
    c = q.counters()
    assert c["ins_heapify_ops"] == n // K - 1
    assert c["del_refill_ops"] == n // K - 1


def test_seq_model_ragged_and_edge_cases():
    K = 8
    q = oracle.SeqBGPQ(K, 256)
    assert list(q.deletemin(3)[0]) == []          # empty heap (Alg.2 l.16-17)
    with pytest.raises(ValueError):
        q.insert(np.arange(K + 1))                # at most k keys per op
    with pytest.raises(ValueError):
        q.deletemin(0)
    q.insert([5])
    assert list(q.deletemin(K)[0]) == [5]         # fewer than requested -> all
    keys = synth.keys(1000, seed=9)
    for off in range(0, 1000, 7):
        q.insert(keys[off:off + 7])
    got = np.concatenate([q.deletemin(5)[0] for _ in range(201)])
    assert np.array_equal(got, np.sort(keys))


def test_seq_model_capacity_overflow_is_sticky():
    K = 4
    q = oracle.SeqBGPQ(K, 3)  # root + nodes 2, 3
    for i in range(3):
        assert q.insert(np.arange(4 * i, 4 * i + 4)) == 0
    assert q.insert(np.arange(100, 104)) == -3   # R15: sticky EFULL, op dropped
    assert q.header()["err"] == -3


# --------------------------------------------------------------------------------------
# Mutation tests: the checks must catch plausible mistakes
# --------------------------------------------------------------------------------------
@pytest.mark.parametrize("mutation", [1, 2, 3])
def test_mutations_are_caught(mutation):
    caught = 0
    for seed in range(40):
        _, _, bad_out, bad_inv = _random_run(4, 200, seed, key_hi=50, mutation=mutation)
        caught += (bad_out + bad_inv) > 0
    assert caught >= 30, f"mutation {mutation} caught only in {caught}/40 runs"


def test_invariant_checker_catches_corruption():
    K = 4
    q = oracle.SeqBGPQ(K, 32)
    keys = synth.keys(4 * 20, seed=11)
    for off in range(0, 80, 4):
        q.insert(keys[off:off + 4])
    h = q.header()
    nk, _, st = q.dump()
    args = (K, q.cap, h["heapSize"], h["rootSize"], h["pbSize"])
    assert oracle.check_invariants(*args, nk, st) == (0, 0)
    bad = nk.copy(); bad[5] = bad[5][::-1]                          # unsorted node
    assert oracle.check_invariants(*args, bad, st)[0] == -2
    bad = nk.copy(); bad[5][0], bad[2][3] = bad[2][3], bad[5][0]    # parent/child order
    bad[2].sort(); bad[5].sort()
    assert oracle.check_invariants(*args, bad, st)[0] in (-4,)
    bad_st = st.copy(); bad_st[h["heapSize"] + 1] = oracle.AVAIL    # AVAIL beyond heapSize
    assert oracle.check_invariants(*args, nk, bad_st)[0] == -3
    assert oracle.check_invariants(K, q.cap, h["heapSize"], K + 1, 0, nk, st)[0] == -1


@pytest.mark.parametrize("K", [4, 64])
def test_seq_model_sorted_input_special_cases(K):
    """Special cases fixed by Alg.1 and SORT_SPLIT's definition.

    Ascending full-K batches: every new batch is >= every stored key, so the root section
    and each INSERT_HEAPIFY level keep their node (no-op split) and batch j lands whole at
    node tar = j+1 (heapSize++ per op, Alg.1 l.16-18): the node array is the input in BFS
    order.  Descending batches: every batch is <= every stored key, so every split along
    the path is a pure swap and the root always holds the last batch.
    """
    nb = 37                                     # ragged last level of the tree
    base = np.sort(synth.keys(nb * K, seed=5))
    q = oracle.SeqBGPQ(K, nb + 2)
    for j in range(nb):
        q.insert(base[j * K:(j + 1) * K])
    nk, _, st = q.dump()
    for j in range(nb):
        assert np.array_equal(nk[j + 1], base[j * K:(j + 1) * K]), j
        assert st[j + 1] == oracle.AVAIL
    c = q.counters()
    assert c["ins_swap"] == 0 and c["ins_merge"] == 0
    assert c["ins_noop"] == c["ins_levels"]
    assert _check_inv(q) == (0, 0)

    desc = base[::-1].copy()
    q = oracle.SeqBGPQ(K, nb + 2)
    for j in range(nb):
        q.insert(desc[j * K:(j + 1) * K])
    nk, _, _ = q.dump()
    assert np.array_equal(nk[1], np.sort(desc[(nb - 1) * K:]))
    c = q.counters()
    assert c["ins_noop"] == 0 and c["ins_merge"] == 0
    assert c["ins_swap"] == c["ins_levels"]
    assert _check_inv(q) == (0, 0)
    out = np.concatenate([q.deletemin(K)[0] for _ in range(nb)])
    assert np.array_equal(out, base)


def test_replay_matches_bruteforce_log():
    """oracle.replay (used by the GPU ticket-order replays) against a brute-force sorted list
    on random logs with partial sizes and over-asking deletemins (fewer than asked ->
    everything left; x_{k+1} = min_r(I_k - D_k))."""
    rng = np.random.default_rng(5)
    for trial in range(30):
        log, brute, want = [], [], []
        for _ in range(60):
            if rng.random() < 0.55:
                k = rng.integers(0, 40, rng.integers(1, 9)).astype(np.uint32)
                log.append((0, (k, None)))
                brute.extend(int(x) for x in k)
            else:
                m = int(rng.integers(1, 12))
                log.append((1, m))
                brute.sort()
                want.append(brute[:m])
                del brute[:m]
        got = oracle.replay(log)
        assert len(got) == len(want)
        for (gk, _), w in zip(got, want):
            assert gk.tolist() == w
    q = oracle.OraclePQ()
    oracle.replay([(0, (np.array([3, 1, 2], np.uint32), None)), (1, 2)], q=q)
    assert q.size() == 1 and q.deletemin(5)[0].tolist() == [3]


def test_invariant_checker_root_and_buffer_codes():
    """Codes -5 (pBuffer entry below the root's max: P:146 keeps every buffered key >= the
    root's keys) and -6 (non-empty heap whose root is not AVAIL)."""
    K = 4
    q = oracle.SeqBGPQ(K, 32)
    keys = synth.keys(4 * 6 + 2, seed=12)
    for off in range(0, 24, 4):
        q.insert(keys[off:off + 4])
    q.insert(keys[24:26])                      # partial batch -> pBuffer non-empty
    h = q.header()
    assert h["pbSize"] > 0 and h["rootSize"] == K
    nk, _, st = q.dump()
    args = (K, q.cap, h["heapSize"], h["rootSize"], h["pbSize"])
    assert oracle.check_invariants(*args, nk, st) == (0, 0)
    bad = nk.copy(); bad[0][0] = 0; bad[1][:] = np.sort(bad[1]); bad[0][:h["pbSize"]].sort()
    bad[1][K - 1] = 0xFFFFFFFF                 # root max above the buffer's min
    assert oracle.check_invariants(*args, bad, st)[0] == -5
    bad_st = st.copy(); bad_st[1] = oracle.EMPTY
    assert oracle.check_invariants(*args, nk, bad_st)[0] == -6


def test_seq_model_del_levels_closed_forms():
    """DELETEMIN_HEAPIFY level counter (the byte model's del_levels, Alg.3 l.4): with all keys
    equal, l.4's stop test max(cur) <= min(l, r) holds at the root, so no level is traversed and
    every full-K deletemin but the last refills (Alg.2 l.5-14); with two batches the single
    refill walks at most one level (root -> node 2 has no children)."""
    K, nb = 8, 50
    q = oracle.SeqBGPQ(K, nb + 2)
    for _ in range(nb):
        q.insert(np.full(K, 9, np.uint32))
    for _ in range(nb):
        assert q.deletemin(K)[0].tolist() == [9] * K
    c = q.counters()
    assert c["del_levels"] == 0 and c["del_ops"] == nb and c["del_refill_ops"] == nb - 1
    q = oracle.SeqBGPQ(K, 8)
    q.insert(np.arange(8, 16, dtype=np.uint32))
    q.insert(np.arange(0, 8, dtype=np.uint32))
    q.insert(np.arange(16, 24, dtype=np.uint32))  # heapSize 3: root [0..7], node 2 [8..15], node 3 [16..23]
    assert q.deletemin(K)[0].tolist() == list(range(8))
    c = q.counters()
    # refill takes node 3 into the root; one level: l = 2 AVAIL, r = 3 now EMPTY (R5) -> y = 2
    assert c["del_refill_ops"] == 1 and c["del_levels"] == 1 and c["del_lr_skip"] == 1
