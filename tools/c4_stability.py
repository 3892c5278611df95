#!/usr/bin/env python
"""How often does Hogwild on C4's rating scale (0..100, lambda 1) diverge? (GPU only)
C4 at a reduced size, grid (1, Bc), 5 epochs from init seed 1, `reps` runs per setting; prints the
final test RMSEs (nan = diverged) and the warps per launch.  Settings: staleness kappa x 1e4
(library option `staleness`, default 80) and heavy_first (R20).

    python tools/c4_stability.py --frac 0.05 --reps 10 --staleness 80 60 40 --heavy 1 0
"""
import argparse
import json
import math
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--frac", type=float, default=0.05)
    ap.add_argument("--Bc", type=int, default=1)
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--epochs", type=int, default=5)
    ap.add_argument("--staleness", type=int, nargs="+", default=[80])
    ap.add_argument("--heavy", type=int, nargs="+", default=[1024], help="heavy_first: 1024 default, -1 off")
    a = ap.parse_args()
    import paper_conf_icpp_huangylhbl21_b200 as pkg
    cfg = synth.scaled(synth.CONFIGS["c4"], a.frac)
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
    out = []
    for st in a.staleness:
        for hv in a.heavy:
            finals, curves = [], []
            for rep in range(a.reps):
                mdl = pkg.Model(cfg.m, cfg.n, 128, cfg.gamma, cfg.lam)
                mdl.set_option("staleness", st)
                mdl.set_option("heavy_first", hv)
                mdl.load(u, v, r)
                mdl.partition(1, (1, a.Bc), seed=cfg.seed)
                mdl.init(1)
                c = []
                for _ in range(a.epochs):
                    mdl.train_epoch("hogwild", "none")
                    c.append(round(mdl.rmse(tu, tv, tr), 4))
                mdl.close()
                finals.append(c[-1])
                curves.append(c)
            nan = sum(1 for x in finals if not math.isfinite(x))
            rec = {"staleness": st, "heavy_first": hv, "reps": a.reps, "diverged": nan,
                   "finals": finals, "epoch1": [x[0] for x in curves]}
            print(json.dumps(rec), flush=True)
            out.append(rec)


if __name__ == "__main__":
    main()
