#!/usr/bin/env python
"""Per-epoch test-RMSE gap of the Hogwild pipelined ring vs the oracle's ring order, on the
loopback data plane (G ranks on one GPU, each launching its own column blocks: one rank's
real race geometry).  GPU only.  One JSON line per setting, also appended to
gpurun_out/ring_band_sweep.jsonl.

    python tools/ring_band_sweep.py --config c2 --G 2 --Bc 2 --epochs 20 \
        --opt prefetch_depth=1 --opt conflict_ratio=3 [--frac 1.0] [--single]
"""
import argparse
import json
import os
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c2")
    ap.add_argument("--frac", type=float, default=1.0)
    ap.add_argument("--G", type=int, default=2)
    ap.add_argument("--Bc", type=int, default=0)
    ap.add_argument("--epochs", type=int, default=20)
    ap.add_argument("--opt", action="append", default=[])
    ap.add_argument("--storage", default="fp32")
    ap.add_argument("--single", action="store_true", help="G = 1, sync none (reference geometry)")
    ap.add_argument("--oracle-cache", default=None)
    ap.add_argument("--repeats", type=int, default=1)
    a = ap.parse_args()
    import oracle
    import paper_conf_icpp_huangylhbl21_b200 as pkg
    cfg = synth.CONFIGS[a.config]
    if a.frac != 1.0:
        cfg = synth.scaled(cfg, a.frac)
    G = 1 if a.single else a.G
    Bc = a.Bc or G
    sync = "none" if a.single else "ring"
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    cache = a.oracle_cache or os.path.join(ROOT, "gpurun_out", f"oracle_ring_{a.config}_{a.frac}_{G}_{Bc}_{a.epochs}.json")
    golden = os.path.join(ROOT, "tests", "golden", f"oracle_curve_{a.config}.json" if a.single else
                          f"oracle_curve_{a.config}_ring_G{G}_Bc{Bc}.json")
    if a.frac == 1.0 and os.path.exists(golden) and json.load(open(golden))["epochs"] == a.epochs:
        want = json.load(open(golden))["test_rmse"]
    elif os.path.exists(cache):
        want = json.load(open(cache))
    else:
        t0 = time.time()
        prob = oracle.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u, v, r, G=G, Br=1, Bc=Bc, seed=cfg.seed)
        prob.init(1)
        want = [prob.rmse(tu, tv, tr)]
        for _ in range(a.epochs):
            prob.epoch("serial", sync)
            want.append(prob.rmse(tu, tv, tr))
        os.makedirs(os.path.dirname(cache), exist_ok=True)
        json.dump(want, open(cache, "w"))
        print(f"oracle {time.time() - t0:.0f} s", file=sys.stderr)
    opts = [(kv.split("=")[0], int(kv.split("=")[1])) for kv in a.opt]
    for rep in range(a.repeats):
        if a.single:
            mdl = pkg.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam)
            for k_, v_ in opts:
                mdl.set_option(k_, v_)
            mdl.load(u, v, r)
            mdl.partition(1, (1, Bc), seed=cfg.seed, storage=a.storage)
            mdl.init(1)
            curve = [mdl.rmse(tu, tv, tr)]
            for _ in range(a.epochs):
                mdl.train_epoch("hogwild", "none")
                curve.append(mdl.rmse(tu, tv, tr))
            mdl.close()
        else:
            hub = pkg.Hub(G)
            out = [None] * G
            edges = np.linspace(0, len(u), G + 1).astype(np.int64)

            def work(rank):
                mdl = pkg.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, hub=hub, rank=rank)
                for k_, v_ in opts:
                    mdl.set_option(k_, v_)
                mdl.load_slice(u[edges[rank]:edges[rank + 1]], v[edges[rank]:edges[rank + 1]],
                               r[edges[rank]:edges[rank + 1]])
                mdl.partition(G, (1, Bc), seed=cfg.seed, storage=a.storage)
                mdl.init(1)
                c = [mdl.rmse(tu, tv, tr)]
                for _ in range(a.epochs):
                    mdl.train_epoch("hogwild", "ring")
                    c.append(mdl.rmse(tu, tv, tr))
                out[rank] = c
                mdl.close()

            ts = [threading.Thread(target=work, args=(q,)) for q in range(G)]
            [t.start() for t in ts]
            [t.join() for t in ts]
            hub.close()
            curve = out[0]
        gap = [g - w for g, w in zip(curve, want)]
        rec = {"config": a.config, "frac": a.frac, "G": G, "Bc": Bc, "opts": dict(opts), "storage": a.storage,
               "rep": rep, "max_gap_e2plus": max(gap[2:]), "final_gap": gap[-1],
               "gap": [round(x, 5) for x in gap], "oracle": [round(x, 5) for x in want],
               "gpu": [round(x, 5) for x in curve]}
        print(json.dumps(rec), flush=True)
        with open(os.path.join(ROOT, "gpurun_out", "ring_band_sweep.jsonl"), "a") as f:
            f.write(json.dumps(rec) + "\n")


if __name__ == "__main__":
    main()
