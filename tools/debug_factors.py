#!/usr/bin/env python
"""Per-epoch factor health (max |P|, max |Q|, non-finite counts, test RMSE) for Hogwild variants."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import synth  # noqa: E402
import paper_conf_icpp_huangylhbl21_b200 as hc  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="c3")
ap.add_argument("--epochs", type=int, default=3)
ap.add_argument("--warps", type=int, default=148)
ap.add_argument("--atomic", type=int, default=1)
ap.add_argument("--heavy", type=int, default=-1)
args = ap.parse_args()
cfg = synth.CONFIGS[args.config]
(u, v, r), (tu, tv, tr) = synth.make(cfg)
mdl = hc.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam)
mdl.set_option("heavy_first", args.heavy)
mdl.load(u, v, r)
mdl.partition(1, (1, 1), seed=cfg.seed)
mdl.set_option("hogwild_atomic", args.atomic)
mdl.set_option("hogwild_warps", args.warps)
mdl.init(1)
for e in range(args.epochs):
    mdl.train_epoch("hogwild", "none")
    P, Q = mdl.factors()
    bp, bq = ~np.isfinite(P), ~np.isfinite(Q)
    print(f"epoch {e}: rmse {mdl.rmse(tu, tv, tr):.5f} max|P| {np.nanmax(np.abs(P)):.3g} max|Q| "
          f"{np.nanmax(np.abs(Q)):.3g} nonfinite P rows {bp.any(1).sum()} Q rows {bq.any(1).sum()}", flush=True)
    if bq.any():
        deg = np.bincount(v, minlength=cfg.n)
        bad = np.where(bq.any(1))[0][:10]
        print("  bad items", bad.tolist(), "degrees", deg[bad].tolist(), "max deg", deg.max())
