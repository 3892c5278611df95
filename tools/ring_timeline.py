#!/usr/bin/env python
"""Hidden synchronisation, measured (verdict item 8): the
pipelined Hogwild ring on the loopback data plane (G ranks on one GPU), with the library's
CUDA-event timeline (HCCMF_OPT_TIMELINE) around every SGD launch (compute stream) and every
column-block transfer (comm stream) of one epoch.  Reports, for rank 0: the epoch span, the
compute time, the transfer time, and how much of the transfer time overlaps compute.  GPU only;
writes gpurun_out/ring_timeline_<cfg>_G<G>_Bc<Bc>.json.

    python tools/ring_timeline.py [--config c3] [--G 4] [--Bc 8] [--wire16]
"""
import argparse
import json
import os
import sys
import threading

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402


def union(iv):
    iv = sorted(iv)
    out = []
    for a, b in iv:
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


def overlap(a, b, U):
    return sum(max(0.0, min(b, y) - max(a, x)) for x, y in U)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c3")
    ap.add_argument("--G", type=int, default=4)
    ap.add_argument("--Bc", type=int, default=0)
    ap.add_argument("--wire16", action="store_true")
    a = ap.parse_args()
    import paper_conf_icpp_huangylhbl21_b200 as pkg
    cfg = synth.CONFIGS[a.config]
    G, Bc = a.G, a.Bc or 2 * a.G
    hub = pkg.Hub(G)
    out = [None] * G
    errs = []
    device_gen = cfg.nnz >= 1_000_000_000
    if not device_gen:
        (u, v, r), _ = synth.make(cfg, n_test=1)
        edges = np.linspace(0, len(u), G + 1).astype(np.int64)

    def work(rank):
        try:
            mdl = pkg.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, hub=hub, rank=rank)
            if device_gen:
                import torch
                (du, dv, dr), _ = synth.make_device(cfg, n_test=1, device="cuda:0", part=(rank, G))
                torch.cuda.synchronize()
                mdl.load_slice(du, dv, dr)
                del du, dv, dr
            else:
                lo, hi = edges[rank], edges[rank + 1]
                mdl.load_slice(u[lo:hi], v[lo:hi], r[lo:hi])
            mdl.partition(G, (1, Bc), seed=cfg.seed)
            mdl.set_option("wire_fp16", int(a.wire16))
            mdl.init(1)
            mdl.train_epoch("hogwild", "ring")  # warm-up (plans, buffers)
            mdl.set_option("timeline", 1)
            mdl.train_epoch("hogwild", "ring")
            out[rank] = (mdl.timeline(), mdl.info())
            mdl.close()
        except Exception as e:  # noqa: BLE001
            errs.append(e)

    ts = [threading.Thread(target=work, args=(q,)) for q in range(G)]
    [t.start() for t in ts]
    [t.join() for t in ts]
    hub.close()
    if errs:
        raise errs[0]
    rep = {"config": a.config, "workload": cfg.name, "G": G, "Bc": Bc, "wire16": a.wire16,
           "backend": "loopback (G ranks on one GPU; transfers are device-to-device copies)", "ranks": []}
    for rank, (tl, info) in enumerate(out):
        comp = [(x[3], x[4]) for x in tl if x[0] == 0]
        xfer = [(x[3], x[4]) for x in tl if x[0] == 1]
        U = union(comp)
        span = max(x[4] for x in tl) - min(x[3] for x in tl)
        t_x = sum(b - a_ for a_, b in xfer)
        hidden = sum(overlap(a_, b, U) for a_, b in xfer)
        last_comp = max(b for _, b in comp)
        tail = max(0.0, max(b for _, b in xfer) - last_comp)
        rep["ranks"].append({"rank": rank, "local_nnz": info["local_nnz"], "epoch_span_ms": span,
                             "compute_ms": sum(b - a_ for a_, b in U), "launches": len(comp),
                             "transfers": len(xfer), "transfer_ms": t_x, "transfer_overlapped_ms": hidden,
                             "overlap_frac": hidden / t_x if t_x else None, "exposed_tail_ms": tail,
                             "rows": [[round(float(y), 4) for y in x] for x in tl]})
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    path = os.path.join(ROOT, "gpurun_out", f"ring_timeline_{a.config}_G{G}_Bc{Bc}{'_w16' if a.wire16 else ''}.json")
    with open(path, "w") as f:
        json.dump(rep, f, indent=1)
    print(json.dumps({k: v for k, v in rep.items() if k != "ranks"} |
                     {"rank0": {k: v for k, v in rep["ranks"][0].items() if k != "rows"}}))


if __name__ == "__main__":
    main()
