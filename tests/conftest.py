import os
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

GOLDEN = os.path.join(ROOT, "tests", "golden")


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running test")


def load_g1():
    """Parse tests/golden/fig1_g1.txt (Fig. 1 reconstruction, PAPER.md P:69, P:115,
    P:212-214).  Returns 0-based adjacency [12, 8], points [12, 4], query [4] and the
    expected traces."""
    adj = {}
    order = None
    ex2_its, ex2 = [], {}
    ex1 = {}
    with open(os.path.join(GOLDEN, "fig1_g1.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            tok = line.split()
            if tok[0] == "adj":
                adj[int(tok[1][1:]) - 1] = [int(t) - 1 for t in tok[2:]]
            elif tok[0] == "order":
                order = [int(t) - 1 for t in tok[1:]]
            elif tok[0] == "ex2" and tok[1] == "it":
                ti = tok.index("tsorted")
                ni = tok.index("N")
                ex2_its.append(dict(
                    explore=int(tok[4]) - 1,
                    tsorted=[int(t) - 1 for t in tok[ti + 1:ni]],
                    N=[int(t.rstrip("*")) - 1 for t in tok[ni + 1:]],
                    flags=[int(t.endswith("*")) for t in tok[ni + 1:]]))
            elif tok[0] == "ex2" and tok[1] == "stats":
                ex2["stats"] = [int(tok[3]), int(tok[5]), int(tok[7])]
            elif tok[0] == "ex2":
                ex2[tok[1]] = [float(t) if tok[1] == "dists" else int(t) - 1 for t in tok[2:]]
            elif tok[0] == "ex1":
                vals = [int(t) for t in tok[2:]]
                ex1[tok[1]] = vals if tok[1] == "dist_comps" else [v - 1 for v in vals]
    n = len(adj)
    nbr = np.full((n, 8), -1, np.int32)
    for v, row in adj.items():
        nbr[v, :len(row)] = row
    X = np.zeros((n, 4), np.float32)
    for rank, v in enumerate(order, start=1):
        X[v, 0] = rank
    q = np.zeros(4, np.float32)
    ex2["its"] = ex2_its
    return dict(nbr=nbr, X=X, q=q, ex2=ex2, ex1=ex1, order=order)


@pytest.fixture(scope="session")
def g1():
    return load_g1()
