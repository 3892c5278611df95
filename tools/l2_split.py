#!/usr/bin/env python
"""Workload for the ncu capture of the SGD kernel and of the L2 hit-rate split (verdict item 8):
bench.py's configuration of a workload, one warm epoch, one epoch, then the Q-stream and
P-stream replays (hccmf_probe_roundtrip modes 3 and 4) and the reductions-only ceiling probe,
each as its own launch.  Run it under

    ncu --set full --clock-control none -k regex:"sgd_warp_kernel|stream_kernel|roundtrip_kernel" \\
        -o gpurun_out/l2split_c5 python tools/l2_split.py --config c5

and read lts__t_sector_hit_rate.pct per launch (tools/ncu_summary.py).
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c5")
    ap.add_argument("--storage", default="fp32")
    a = ap.parse_args()
    import torch

    import paper_conf_icpp_huangylhbl21_b200 as pkg
    cfg = synth.CONFIGS[a.config]
    (du, dv, dr), _ = synth.make_device(cfg, n_test=1, device="cuda:0")
    torch.cuda.synchronize()
    mdl = pkg.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam)
    mdl.load(du, dv, dr)
    del du, dv, dr
    torch.cuda.empty_cache()
    Bc = max(1, round(cfg.n * cfg.k * 4 / 80e6))
    mdl.partition(1, (1, Bc), seed=cfg.seed, storage=a.storage)
    mdl.init(1)
    mdl.train_epoch("hogwild", "none")
    mdl.train_epoch("hogwild", "none")
    for mode in ("q_stream", "p_stream", "red_f32"):
        mdl.probe_roundtrip(mode, reps=1)
    print("ok", flush=True)


if __name__ == "__main__":
    main()
