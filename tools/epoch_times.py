#!/usr/bin/env python
"""Per-epoch SGD time from a fresh init (CUDA events on the handle's stream), GPU only:
does an epoch's cost depend on where training is?  python tools/epoch_times.py --config c5"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5")
    ap.add_argument("--epochs", type=int, default=6)
    ap.add_argument("--opt", action="append", default=[], help="name=value library option")
    a = ap.parse_args()
    import torch

    import paper_conf_icpp_huangylhbl21_b200 as pkg
    cfg = synth.CONFIGS[a.config]
    (u, v, r), (tu, tv, tr) = synth.make_device(cfg, device="cuda:0")
    mdl = pkg.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam)
    for kv in a.opt:
        mdl.set_option(kv.split("=")[0], int(kv.split("=")[1]))
    s = torch.cuda.Stream()
    mdl.set_stream(s)
    mdl.load(u, v, r)
    del u, v, r
    torch.cuda.empty_cache()
    mdl.partition(1, (1, 1), seed=cfg.seed)
    out = []
    for rep in range(2):
        mdl.init(1)
        ts = []
        for e in range(a.epochs):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            mdl.train_epoch("hogwild", "none")
            e1.record(s)
            e1.synchronize()
            ts.append(round(e0.elapsed_time(e1), 2))
            mdl.rmse(tu, tv, tr)
        out.append(ts)
    print(json.dumps({"config": a.config, "epoch_ms_from_init": out, "info": {k: v for k, v in mdl.info().items()
                                                                           if k in ("hogwild_warps", "det_path")}}))


if __name__ == "__main__":
    main()
