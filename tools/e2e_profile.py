#!/usr/bin/env python
"""Wall time of each public call of one e2e job (pinned host buffers), GPU only.
HCCMF_PROFILE=1 adds the library's per-phase partition times on stderr."""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_huangylhbl21_b200 as hc  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="c3")
ap.add_argument("--epochs", type=int, default=5)
args = ap.parse_args()
cfg = synth.CONFIGS[args.config]
if cfg.nnz > 1_000_000_000:
    (u, v, r), (tu, tv, tr) = synth.make_device(cfg)
    u, v, r, tu, tv, tr = (x.cpu().numpy() for x in (u, v, r, tu, tv, tr))
    torch.cuda.empty_cache()
else:
    (u, v, r), (tu, tv, tr) = synth.make(cfg)
pin = [torch.from_numpy(x).pin_memory() for x in (u, v, r, tu, tv, tr)]
Ph = torch.empty((cfg.m, cfg.k), dtype=torch.float32).pin_memory()
Qh = torch.empty((cfg.n, cfg.k), dtype=torch.float32).pin_memory()
for rep in range(2):
    t = {}
    t0 = time.perf_counter()

    def mark(name):
        global t0
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        t[name] = t.get(name, 0.0) + (t1 - t0) * 1e3
        t0 = t1

    m = hc.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam)
    mark("create")
    m.load(pin[0], pin[1], pin[2])
    mark("load (H2D + validate)")
    m.partition(1, (1, 1), seed=cfg.seed)
    mark("partition")
    m.init(1)
    mark("init")
    for _ in range(args.epochs):
        m.train_epoch("hogwild", "none")
        mark("epochs")
        m.rmse(pin[3], pin[4], pin[5])
        mark("rmse")
    m.factors(Ph, Qh)
    mark("export (D2H)")
    m.close()
    mark("destroy")
    print(f"rep {rep}: total {sum(t.values()):.1f} ms", {k: round(v_, 1) for k, v_ in t.items()}, flush=True)
