#!/usr/bin/env python
"""Per-GPU throughput at one rank's real ring geometry (verdict item 2):
the ratings of every G-th user (one row shard's worth, users are randomly relabelled by the
generator) on ONE GPU, grid (1, G): each launch races on one column group of n/G items with the
per-launch concurrency cap n/(3G) -- exactly what rank s runs at ring stage t.  Reports the
epoch rate (CUDA events, warm-up excluded).  GPU only.

    python tools/rank_rate.py --config c5 --G 1 2 4 8
"""
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
    ap.add_argument("--G", type=int, nargs="+", default=[1, 2, 4, 8])
    ap.add_argument("--epochs", type=int, default=3)
    ap.add_argument("--storage", default="fp32")
    ap.add_argument("--opt", action="append", default=[], help="name=value library option (e.g. conflict_ratio=2)")
    a = ap.parse_args()
    opts = [(kv.split("=")[0], int(kv.split("=")[1])) for kv in a.opt]
    import torch

    import paper_conf_icpp_huangylhbl21_b200 as pkg
    cfg = synth.CONFIGS[a.config]
    res = []
    for G in a.G:
        # every G-th user's ratings, drawn part by part (bounded device memory at C5 scale)
        P = 16
        us, vs, rs = [], [], []
        for part in range(P):
            (du, dv, dr), _ = synth.make_device(cfg, n_test=1, device="cuda:0", part=(part, P))
            keep = (du % G) == 0
            us.append(du[keep])
            vs.append(dv[keep])
            rs.append(dr[keep])
            del du, dv, dr, keep
        u, v, r = torch.cat(us), torch.cat(vs), torch.cat(rs)
        del us, vs, rs
        torch.cuda.synchronize()
        mdl = pkg.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam)
        for k_, v_ in opts:
            mdl.set_option(k_, v_)
        mdl.load(u, v, r)
        nnz = int(u.numel())
        del u, v, r
        torch.cuda.empty_cache()
        mdl.partition(1, (1, G), seed=cfg.seed, storage=a.storage)
        mdl.init(1)
        mdl.train_epoch("hogwild", "none")
        s = torch.cuda.Stream()
        mdl.set_stream(s)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        for _ in range(a.epochs):
            mdl.train_epoch("hogwild", "none")
        e1.record(s)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.epochs
        rec = {"config": a.config, "G": G, "storage": a.storage, "opts": dict(opts), "ratings": nnz, "epoch_ms": ms,
               "updates_per_s": nnz / (ms / 1e3), "launches_per_epoch": G,
               "items_per_launch": -(-cfg.n // G), "note": "one rank's shard and launch geometry on one GPU"}
        res.append(rec)
        print(json.dumps(rec), flush=True)
        mdl.close()
        torch.cuda.empty_cache()
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    tag = "_".join(f"{k_}{v_}" for k_, v_ in opts)
    with open(os.path.join(ROOT, "gpurun_out", f"rank_rate_{a.config}_{a.storage}{'_' + tag if tag else ''}.json"), "w") as f:
        json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
