#!/usr/bin/env python
"""Latency of the DET slab wavefront's per-rating chain with no contention (GPU only): n = 2
items, a 2 x 2 grid, so each of the two warps walks one column block that holds ONE item -- every
rating of a block reads the q_v the previous one wrote (the heavy-item chain of the C3 critical
path), one warp per SM.  Reports ns per rating (CUDA events over the DET epoch).

    python tools/det_chain_latency.py [--ratings 2000000] [--k 128]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ratings", type=int, default=2_000_000)
    ap.add_argument("--k", type=int, default=128)
    ap.add_argument("--per-user", type=int, default=1, help="ratings per user (1: a new p_u every rating)")
    a = ap.parse_args()
    import numpy as np
    import torch

    import paper_conf_icpp_huangylhbl21_b200 as pkg
    rng = np.random.default_rng(1)
    m = a.ratings // a.per_user
    u = np.repeat(np.arange(m, dtype=np.int32), a.per_user)
    v = rng.integers(0, 2, len(u)).astype(np.int32)
    r = rng.uniform(1, 5, len(u)).astype(np.float32)
    mdl = pkg.Model(m, 2, a.k, 0.005, 0.01)
    mdl.load(u, v, r)
    mdl.partition(1, (2, 2), seed=3)
    mdl.init(1)
    s = torch.cuda.Stream()
    mdl.set_stream(s)
    out = []
    for _ in range(4):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        mdl.train_epoch("det", "none")
        e1.record(s)
        e1.synchronize()
        out.append(e0.elapsed_time(e1))
    info = mdl.info()
    ms = float(np.median(out[1:]))
    # two warps in parallel, each over about half the ratings (its two blocks, one per stratum)
    print(json.dumps({"ratings": len(u), "k": a.k, "per_user": a.per_user, "epoch_ms": round(ms, 3),
                      "ns_per_rating_per_warp": round(ms * 1e6 / (len(u) / 2), 1), "det_path": info["det_path"]}))


if __name__ == "__main__":
    main()
