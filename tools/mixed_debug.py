"""Debug aid: one mixed call on a prefilled heap (argv: K regime break_at debug)."""
import sys, numpy as np, torch
sys.path.insert(0, "."); sys.path.insert(0, "tests")
import synth, paper_conf_icpp_chenhjz21_b200 as pkg
from test_gpu_mixed import _prefilled
from test_gpu_parity import _mixed_inputs, _run_mixed, _replay_check
K, regime, brk, dbg = int(sys.argv[1]), sys.argv[2], int(sys.argv[3]), int(sys.argv[4])
pkg.set_debug(dbg)
q, pre = _prefilled(K, False, 120 * K, regime, seed=120)
types, sizes = synth.mixed_ops(500, K, seed=121)
sizes = sizes.copy()
if brk >= 0: sizes[2 * brk] = K - 5
keys, in_off = _mixed_inputs(types, sizes, K, seed=122)
outk, outv, cnt, lin = _run_mixed(q, types, sizes, keys, in_off)
print("stats", q.stats())
_replay_check(types, sizes, keys, in_off, outk, outv, cnt, lin - lin.min(), prefill=pre)
print("OK", sys.argv[1:])
