#!/usr/bin/env python
"""The Hogwild q_v round-trip ceilings of hccmf_probe_roundtrip on one config (GPU only):
LSU vector reductions (mode 0), LSU load + reduction (2), and the TMA bulk-engine variants
(5: bulk reductions only, 6/8/9: bulk load 3/7/1 ratings ahead + dependent bulk reduction,
7: LSU load + bulk reduction).  Same records and warps as the epoch; prints one JSON line.

    python tools/probe_modes.py --config c5
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
    ap.add_argument("--config", default="c3")
    ap.add_argument("--modes", nargs="+", default=["red_f32", "ldred_f32", "bulkred_f32", "bulkldred_f32",
                                                     "ldbulkred_f32", "bulkldred8_f32", "bulkldred2_f32"])
    a = ap.parse_args()
    import torch

    import paper_conf_icpp_huangylhbl21_b200 as pkg
    cfg = synth.CONFIGS[a.config]
    (u, v, r), _ = synth.make_device(cfg, n_test=1, device="cuda:0")
    mdl = pkg.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam)
    mdl.load(u, v, r)
    del u, v, r
    torch.cuda.empty_cache()
    mdl.partition(1, (1, 1), seed=cfg.seed)
    mdl.init(1)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    mdl.train_epoch("hogwild", "none")
    torch.cuda.synchronize()
    out = {"config": a.config, "nnz": cfg.nnz}
    for mode in a.modes:
        ms = mdl.probe_roundtrip(mode, reps=3)
        out[mode] = {"ms": round(ms, 3), "G_upd_per_s": round(cfg.nnz / ms / 1e6, 3)}
    print(json.dumps(out))
    os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
    with open(os.path.join(ROOT, "gpurun_out", f"probe_modes_{a.config}.json"), "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
