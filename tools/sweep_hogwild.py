#!/usr/bin/env python
"""Measure Hogwild epoch time and test RMSE vs concurrency (warps) and atomic q updates.

GPU only (does not touch oracle/); compare the printed RMSEs with the oracle's serial
curve stored in tests/golden/oracle_curve_<cfg>.json (tools/oracle_curves.py; the band
tests are tests/test_gpu_full_size.py and tests/test_gpu_parity.py).  Usage:
    python tools/sweep_hogwild.py --config c3 --epochs 5 --warps 148,592,2368,4736 --atomic 0,1
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_icpp_huangylhbl21_b200 as hc  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="c3")
ap.add_argument("--frac", type=float, default=1.0)
ap.add_argument("--epochs", type=int, default=5)
ap.add_argument("--warps", default="148,592,1184,2368,4736")
ap.add_argument("--atomic", default="0,1")
ap.add_argument("--task", type=int, default=256)
ap.add_argument("--grid", default="1,1")
ap.add_argument("--vec", default="0")
ap.add_argument("--repeat", type=int, default=1)
ap.add_argument("--heavy", type=int, default=-1)
ap.add_argument("--sched", default="hogwild")
ap.add_argument("--persist", type=int, default=0)
ap.add_argument("--depth", default="1")
ap.add_argument("--storage", default="fp32")

ap.add_argument("--every", action="store_true", help="test RMSE after every epoch")
args = ap.parse_args()
cfg = synth.CONFIGS[args.config]
if args.frac != 1.0:
    cfg = synth.scaled(cfg, args.frac)
(u, v, r), (tu, tv, tr) = synth.make(cfg)
Br, Bc = (int(x) for x in args.grid.split(","))
st = torch.cuda.Stream()
mdl = hc.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam)
mdl.set_stream(st)
mdl.set_option("task_ratings", args.task)
mdl.set_option("heavy_first", args.heavy)
mdl.set_option("l2_persist", args.persist)

mdl.load(u, v, r)
mdl.partition(1, (Br, Bc), seed=cfg.seed, storage=args.storage)
dtu, dtv, dtr = (torch.from_numpy(x).cuda() for x in (tu, tv, tr))
for at, vec, w, dp in [(a_, v_, w_, d_) for a_ in (int(x) for x in args.atomic.split(","))
                       for v_ in (int(x) for x in args.vec.split(",")) for w_ in (int(x) for x in args.warps.split(","))
                       for d_ in (int(x) for x in args.depth.split(",")) for _ in range(args.repeat)]:
    if True:
        mdl.set_option("prefetch_depth", dp)
        mdl.set_option("vec", vec)
        mdl.set_option("hogwild_atomic", at)
        mdl.set_option("hogwild_warps", w)
        mdl.init(1)
        ts, rms = [], []
        for e in range(args.epochs):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(st)
            mdl.train_epoch(args.sched, "none")
            b.record(st)
            b.synchronize()
            ts.append(a.elapsed_time(b))
            if args.every or e == args.epochs - 1:
                rms.append(round(mdl.rmse(dtu, dtv, dtr), 5))
        rm = rms[-1]
        tmin = min(ts[1:] if len(ts) > 1 else ts)
        print(json.dumps({"config": cfg.name, "storage": args.storage, "depth": dp, "atomic": at, "vec": vec, "warps": w, "epoch_ms": tmin,
                          "gupd_s": cfg.nnz / tmin / 1e6, "test_rmse": rm, "per_epoch": rms}), flush=True)
