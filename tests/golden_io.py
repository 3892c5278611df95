"""Parser for the cited text fixtures under tests/golden/."""
import os

import numpy as np

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load(name):
    """Return {section: list of token rows}; '*' kept as None."""
    out, cur = {}, None
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            if line.startswith("["):
                cur = line[1:line.index("]")]
                out[cur] = []
                continue
            out[cur].append([None if t == "*" else float(t) for t in line.split()])
    return out


def matrix(sec, dtype=np.float64):
    return np.array(sec, dtype=dtype)


def fig1():
    """The paper's Figure 1: (u, v, r) observed ratings, P (5x2), Q (n x k = 4x2), Rp printed."""
    g = load("fig1.txt")
    R = g["R"]
    u, v, r = [], [], []
    for i, row in enumerate(R):
        for j, x in enumerate(row):
            if x is not None:
                u.append(i), v.append(j), r.append(x)
    P = matrix(g["P"])
    Q = matrix(g["Q"]).T.copy()  # stored n x k
    Rp = matrix(g["Rp"])
    return (np.array(u, np.int32), np.array(v, np.int32), np.array(r, np.float32)), P, Q, Rp
