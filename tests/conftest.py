import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a B200 (run with -m gpu)")
    config.addinivalue_line("markers", "slow: long-running CPU test")


def parse_trace(path):
    """Parse a hand-traced golden file (tests/golden/*_trace.txt)."""
    K = cap = None
    steps = []
    with open(path) as f:
        for raw in f:
            line = raw.strip()
            if not line or line.startswith("#"):
                continue
            tok = line.split()
            if tok[0] == "K":
                K = int(tok[1])
            elif tok[0] == "CAP":
                cap = int(tok[1])
            elif tok[0] == "I":
                steps.append(["I", [int(t) for t in tok[1:]], None])
            elif tok[0] == "D":
                m = int(tok[1])
                assert tok[2] == "=>"
                out = [] if tok[3] == "-" else [int(t) for t in tok[3:]]
                steps.append(["D", m, out])
            elif tok[0] == "S":
                st = {}
                for kv in tok[1:]:
                    k, v = kv.split("=")
                    st[k] = int(v) if k == "hs" else ([] if v == "-" else [int(x) for x in v.split(",")])
                steps[-1].append(st)
    return K, cap, steps
