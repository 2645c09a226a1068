"""CPU pin of bench.byte_model (the algorithmic bytes behind roofline.achieved).

INSERT op to target j moves K*w (input) + (floor(log2 j) - 1) * 2K*w (read + write of each
intermediate path node, Alg.1 l.7-14 P:208-215) + K*w (write at tar, l.30-34).  The level
count comes from the sequential model of Alg.1 (oracle.SeqBGPQ counters) and is checked
here against the closed-form path length, so a wrong depth or factor in either fails."""
import numpy as np

import bench
import oracle
import synth


def test_insert_levels_and_bytes_closed_form():
    K, nb, w = 64, 300, 4
    keys = synth.keys(nb * K, seed=7)
    q = oracle.SeqBGPQ(K, nb + 2)
    for j in range(nb):
        q.insert(keys[j * K:(j + 1) * K])
    c = q.counters()
    # op 0 fills the root; op j >= 1 heapifies to tar = j + 1
    want_levels = sum(int(np.floor(np.log2(t))) - 1 for t in range(2, nb + 1))
    assert c["ins_levels"] == want_levels
    assert c["ins_heapify_ops"] == nb - 1
    st = dict.fromkeys(["del_refill_ops", "del_levels", "keys_out", "ins_noop"], 0)
    st.update(ins_ops=c["ins_ops"], ins_levels=c["ins_levels"], ins_heapify_ops=c["ins_heapify_ops"])
    bm = bench.byte_model(st, K, w)
    want = nb * K * w + sum((int(np.floor(np.log2(t))) - 1) * 2 * K * w + K * w for t in range(2, nb + 1))
    assert bm["insert"] == want
    assert bm["deletemin"] == 0 and bm["total"] == want


def test_deletemin_bytes_formula():
    """DELETEMIN: K*w output + K*w refill read + 4K*w per heapify level (read l, r; write
    x, cur; Alg.3 l.2-13 P:316-328) + K*w final write."""
    K, w = 1024, 8
    st = {"ins_ops": 0, "ins_levels": 0, "ins_heapify_ops": 0, "ins_noop": 0,
          "keys_out": 10 * K, "del_refill_ops": 10, "del_levels": 37}
    bm = bench.byte_model(st, K, w)
    assert bm["deletemin"] == 10 * K * w + 10 * K * w + 37 * 4 * K * w + 10 * K * w
