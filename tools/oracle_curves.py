#!/usr/bin/env python
"""Write the oracle's reference test-RMSE curves (tests/golden/oracle_curve_<cfg>.json).

Calls only oracle/ and synth/ (the stored values are the oracle's, never the CUDA
path's).  bench.py reads these files to report epochs-to-RMSE (the
first epoch whose GPU test RMSE <= oracle RMSE@E + 0.005).  Settings mirror bench.py:
one shard, grid (1, 1), shuffle seed = config seed, init seed 1, serial order.

    python tools/oracle_curves.py c1 c2 c3      # C3: ~4 min on one core
"""
import hashlib
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import synth  # noqa: E402

EPOCHS = {"c1": 5, "c2": 20, "c3": 10}


def partition_digest(prob):
    """SHA-256 over the oracle's partition outputs (perm_row, perm_col, bounds, block
    offsets, sorted records) -- compared bit-exactly with the GPU blocker's."""
    h = hashlib.sha256()
    for a in (prob.perm_row, prob.perm_col, prob.b, prob.off, prob.ru, prob.rv, prob.rr):
        h.update(a.tobytes())
    return h.hexdigest()


def det_digest(name, B):
    cfg = synth.CONFIGS[name]
    (u, v, r), _ = synth.make(cfg)
    prob = oracle.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=cfg.seed)
    path = os.path.join(ROOT, "tests", "golden", f"oracle_curve_{name}.json")
    with open(path) as f:
        out = json.load(f)
    out[f"partition_sha256_grid_{B}x{B}"] = partition_digest(prob)
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(name, B, out[f"partition_sha256_grid_{B}x{B}"], flush=True)


def main(names):
    for name in names:
        if ":" in name:  # e.g. c3:2048 -> digest of the B x B DET partition only
            n_, B = name.split(":")
            det_digest(n_, int(B))
            continue
        cfg = synth.CONFIGS[name]
        (u, v, r), (tu, tv, tr) = synth.make(cfg)
        t0 = time.time()
        prob = oracle.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=1, Br=1, Bc=1, seed=cfg.seed)
        prob.init(1)
        digest = partition_digest(prob)
        curve = [prob.rmse(tu, tv, tr)]
        for _ in range(EPOCHS[name]):
            prob.epoch("serial", "none")
            curve.append(prob.rmse(tu, tv, tr))
        out = {"config": name, "workload": cfg.name, "epochs": EPOCHS[name], "test_rmse": curve,
               "partition_sha256_grid_1x1": digest,
               "note": "curve[0] = before training; curve[e] = after e serial oracle epochs (fp64), "
                       "shuffle seed = config seed, init seed 1, grid (1,1)",
               "oracle_seconds": time.time() - t0}
        path = os.path.join(ROOT, "tests", "golden", f"oracle_curve_{name}.json")
        with open(path, "w") as f:
            json.dump(out, f, indent=1)
        print(name, [round(x, 5) for x in curve], f"{out['oracle_seconds']:.0f}s", flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or ["c1", "c2", "c3"])
