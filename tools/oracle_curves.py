#!/usr/bin/env python
"""Write the oracle's reference test-RMSE curves (tests/golden/oracle_curve_<cfg>.json).

Calls only oracle/ and synth/ (the stored values are the oracle's, never the CUDA
path's).  bench.py reads these files to report epochs-to-RMSE (the
first epoch whose GPU test RMSE <= oracle RMSE@E + 0.005).  Settings mirror bench.py:
one shard, grid (1, 1), shuffle seed = config seed, init seed 1, serial order.

    python tools/oracle_curves.py c1 c2 c3      # C3: ~4 min on one core
    python tools/oracle_curves.py c3:2048        # digest of the 2048 x 2048 DET partition
    python tools/oracle_curves.py det:c3:2048    # sampled P, Q rows after one DET epoch
    python tools/oracle_curves.py ring:c3:8:8    # Hogwild-ring reference curve, G = 8, Bc = 8
    python tools/oracle_curves.py det:c3:2048:bal  # the same DET sample with degree-balanced columns (R30)
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


def det_digest(name, B, bal=0):
    cfg = synth.CONFIGS[name]
    (u, v, r), _ = synth.make(cfg)
    prob = oracle.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=cfg.seed,
                          col_balance=bal)
    path = os.path.join(ROOT, "tests", "golden", f"oracle_curve_{name}.json")
    with open(path) as f:
        out = json.load(f)
    key = f"partition_sha256_grid_{B}x{B}" + ("_bal" if bal else "")
    out[key] = partition_digest(prob)
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(name, B, out[key], flush=True)


def det_epoch_sample(name, B, rows=128, bal=0):
    """One DET epoch (B x B grid, the bench's DET configuration: shuffle seed = config
    seed, init seed 1) by the oracle; stores `rows` sampled rows of P and of Q (the
    heaviest users / items first, then uniform draws) as float32 in
    tests/golden/oracle_det_<name>_B<B>.npz, for the full-size DET parity test."""
    import numpy as np
    cfg = synth.CONFIGS[name]
    (u, v, r), _ = synth.make(cfg)
    t0 = time.time()
    prob = oracle.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=1, Br=B, Bc=B, seed=cfg.seed,
                          col_balance=bal)
    prob.init(1)
    prob.epoch("det", "none")
    P, Q = prob.factors()
    rng = np.random.default_rng(7)
    cu, cv = np.bincount(u, minlength=cfg.m), np.bincount(v, minlength=cfg.n)

    def pick(cnt, n):
        top = np.argsort(-cnt, kind="stable")[: rows // 4]
        rest = rng.choice(np.setdiff1d(np.arange(n), top), rows - len(top), replace=False)
        return np.sort(np.concatenate([top, rest])).astype(np.int64)

    iu, iv = pick(cu, cfg.m), pick(cv, cfg.n)
    path = os.path.join(ROOT, "tests", "golden", f"oracle_det_{name}_B{B}{'_bal' if bal else ''}.npz")
    np.savez_compressed(path, users=iu, items=iv, P=P[iu].astype(np.float32), Q=Q[iv].astype(np.float32),
                        digest=np.array(partition_digest(prob)),
                        note=np.array("oracle DET epoch 1 from init(1), shuffle seed = config seed, "
                                      f"grid {B}x{B}{', degree-balanced columns (R30)' if bal else ''}; rows of P "
                                      "(users) and Q (items) in original ids; digest = the partition's SHA-256"))
    print(name, B, "det sample", path, f"{time.time() - t0:.0f}s", flush=True)


def ring_curve(name, G, Bc):
    """The oracle's serialisation of the G-shard Hogwild ring (R19: stage t, shard s,
    its column blocks of group (s+t) mod G in order), grid (1, Bc), init seed 1: the reference
    curve of the multi-rank band tests (tests/golden/oracle_curve_<name>_ring_G<G>_Bc<Bc>.json)."""
    cfg = synth.CONFIGS[name]
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    t0 = time.time()
    prob = oracle.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=G, Br=1, Bc=Bc, seed=cfg.seed)
    prob.init(1)
    digest = partition_digest(prob)
    curve = [prob.rmse(tu, tv, tr)]
    for _ in range(EPOCHS[name]):
        prob.epoch("serial", "ring")
        curve.append(prob.rmse(tu, tv, tr))
    out = {"config": name, "workload": cfg.name, "epochs": EPOCHS[name], "G": G, "Bc": Bc, "test_rmse": curve,
           f"partition_sha256_G{G}_grid_1x{Bc}": digest,
           "note": "curve[0] = before training; curve[e] = after e oracle epochs in the ring serialisation "
                   "(R19), shuffle seed = config seed, init seed 1",
           "oracle_seconds": time.time() - t0}
    path = os.path.join(ROOT, "tests", "golden", f"oracle_curve_{name}_ring_G{G}_Bc{Bc}.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(name, "ring", G, Bc, [round(x, 5) for x in curve], f"{out['oracle_seconds']:.0f}s", flush=True)


def main(names):
    for name in names:
        if name.startswith("ring:"):  # e.g. ring:c3:8:8
            _, n_, G, Bc = name.split(":")
            ring_curve(n_, int(G), int(Bc))
            continue
        if name.startswith("det:"):  # e.g. det:c3:2048[:bal] -> sampled rows after one DET epoch
            parts = name.split(":")
            det_epoch_sample(parts[1], int(parts[2]), bal=int(len(parts) > 3 and parts[3] == "bal"))
            continue
        if ":" in name:  # e.g. c3:2048[:bal] -> digest of the B x B DET partition only
            parts = name.split(":")
            det_digest(parts[0], int(parts[1]), bal=int(len(parts) > 2 and parts[2] == "bal"))
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
