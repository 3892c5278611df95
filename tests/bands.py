"""The Hogwild accuracy bar (R15, R29), shared by every band test.

Hogwild is nondeterministic, so it is held to the oracle's test-RMSE curve in the same
schedule, not to its factors:
  * final: gpu[E] <= oracle[E] + 0.005 ("reach test RMSE within 0.005 of the
    oracle's", at the epoch E where the oracle's curve has flattened, R15), and not below
    oracle[E] - 4 x 0.005 (a sanity floor: R33 -- Hogwild's interleaved users are a better-mixed
    SGD order than the oracle's row-sorted serial sweep and may end lower, e.g. C4 at lambda 1);
  * every epoch e >= 2, one-sided: gpu[e] <= oracle[e] + max(0.005, 0.5 (oracle[e-1] -
    oracle[e])) -- never worse than the oracle by more than 0.005, or, in the steep phase,
    than half an epoch of the oracle's own progress (R29: concurrent rating groups read q_v
    up to one L2 round trip stale, which delays the descent by a fraction of an epoch;
    measured worst cases 0.24 epoch for C2 at G = 1 and 0.32 for the C2 replica all-reduce,
    profiles/r02_band_gaps.md).  Epoch 1 (the jump from the random init) is reported, not
    asserted (R20: the heavy-first task order).
Every checked curve and its per-epoch gaps are appended to $HCCMF_BAND_REPORT (JSON lines)
when that variable is set, so runs leave the evidence behind.
"""
import json
import os

import numpy as np


def check(gpu, ora, tag, final_epoch=None, scale=1.0):
    """scale: the band is 0.005 per 4 rating units (the 1..5-star range of C2/C3);
    C4's 0..100 range gives scale 25 (band 0.125), R29."""
    gpu, ora = np.asarray(gpu, float), np.asarray(ora, float)
    band = 0.005 * scale
    E = len(ora) - 1 if final_epoch is None else final_epoch
    assert len(gpu) >= E + 1, (tag, len(gpu), E)
    gap = gpu[:E + 1] - ora[:E + 1]
    allow = np.full(E + 1, np.inf)
    for e in range(2, E + 1):
        allow[e] = max(band, 0.5 * (ora[e - 1] - ora[e]))
    rec = {"tag": tag, "epochs": E, "gap": [round(float(x), 5) for x in gap],
           "allow": [None if not np.isfinite(a) else round(float(a), 5) for a in allow],
           "oracle": [round(float(x), 5) for x in ora[:E + 1]], "gpu": [round(float(x), 5) for x in gpu[:E + 1]],
           "band": band, "final_ok": bool(-4 * band <= gap[E] <= band), "one_sided_ok": bool(np.all(gap[2:] <= allow[2:]))}
    path = os.environ.get("HCCMF_BAND_REPORT")
    if path:
        with open(path, "a") as f:
            f.write(json.dumps(rec) + "\n")
    assert rec["final_ok"], rec
    assert rec["one_sided_ok"], rec
    return gap
