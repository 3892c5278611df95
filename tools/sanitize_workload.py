#!/usr/bin/env python
"""A small workload that drives every synchronisation-heavy kernel once, for compute-sanitizer
(memcheck / racecheck / synccheck, PAPER.md L564-L570 write-after-write races):
the blocker (a1-a4), the DET slab wavefront (shared-memory Q slabs, inter-CTA progress flags),
the register wavefront, the per-stratum DET kernel, the Hogwild kernels (fp32, binary16 RN/SR,
narrow k = 32), logical-shard ring/all-reduce, RMSE and export.  Duplicate ratings make
consecutive same-item updates (the q forwarding paths).  Exit 0 when every call succeeded.

    compute-sanitizer --tool racecheck python tools/sanitize_workload.py
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_icpp_huangylhbl21_b200 as pkg  # noqa: E402


def problem(m, n, nnz, seed, dup):
    rng = np.random.default_rng(seed)
    u = rng.integers(0, m, nnz).astype(np.int32)
    v = (rng.zipf(1.6, nnz) % n).astype(np.int32)  # skewed items: hot column blocks
    r = rng.uniform(1, 5, nnz).astype(np.float32)
    if dup:
        u, v, r = (np.concatenate([x, x[: nnz // 3]]) for x in (u, v, r))
    return u, v, r


def main():
    quick = "--quick" in sys.argv
    runs = 0
    for (m, n, nnz, k, B, dup) in [(300, 120, 6000, 128, 8, False), (200, 90, 5000, 128, 37, True),
                                   (150, 400, 5000, 256, 12, True)][: 2 if quick else 3]:
        u, v, r = problem(m, n, nnz, B, dup)
        for wave in (1, 2, 0):
            mdl = pkg.Model(m, n, k, 0.02, 0.01)
            mdl.set_option("det_wave", wave)
            mdl.load(u, v, r)
            mdl.partition(1, (B, B), seed=3)
            mdl.init(1)
            mdl.train_epoch("det", "none")
            mdl.rmse(u[:100], v[:100], r[:100])
            mdl.factors()
            mdl.close()
            runs += 1
        for storage in ("fp32", "fp16", "fp16sr"):
            mdl = pkg.Model(m, n, k, 0.02, 0.01)
            mdl.set_option("task_ratings", 64)
            mdl.load(u, v, r)
            mdl.partition(1, (1, 2), seed=3, storage=storage)
            mdl.init(1)
            mdl.train_epoch("hogwild", "none")
            mdl.factors()
            mdl.close()
            runs += 1
    # narrow Hogwild (k = 32) and logical shards (ring + all-reduce, binary16 wire)
    u, v, r = problem(400, 160, 8000, 5, True)
    for k, G, Br, Bc, sched, sync, wire in [(32, 1, 1, 1, "hogwild", "none", 0), (16, 2, 3, 6, "det", "ring", 1),
                                            (128, 2, 2, 2, "det", "allreduce", 1),
                                            (128, 2, 1, 4, "hogwild", "ring", 0)]:
        mdl = pkg.Model(400, 160, k, 0.02, 0.01)
        mdl.load(u, v, r)
        mdl.partition(G, (Br, Bc), seed=4)
        mdl.set_option("wire_fp16", wire)
        mdl.init(2)
        mdl.train_epoch(sched, sync)
        mdl.rmse(u[:50], v[:50], r[:50])
        mdl.factors()
        mdl.close()
        runs += 1
    print(f"sanitize workload: {runs} jobs ok", flush=True)


if __name__ == "__main__":
    main()
