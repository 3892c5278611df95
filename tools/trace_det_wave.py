#!/usr/bin/env python
"""Where the DET wavefront's time goes (GPU only, diagnostic build).

Builds libhccmf with -DHCCMF_DIAG_TRACE into /tmp (the product library is untouched),
runs DET epochs of a config on a B x B grid with the shared-memory-slab wavefront, and
reads the per-(warp, stratum) %globaltimer stamps the kernel wrote: wait begin, wait
satisfied, block released.  Prints a JSON summary: a least-squares fit of block time =
o + c * ratings, the critical path traced back from the last release (blocks, ratings,
time spent in blocks vs in hand-offs), and writes gpurun_out/det_trace.json.

    python tools/trace_det_wave.py [--config c3] [--B 2048]
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c3")
    ap.add_argument("--B", type=int, default=2048)
    ap.add_argument("--wave", type=int, default=1, help="1 slab wavefront, 3 chain-parallel wavefront")
    ap.add_argument("--nobuild", action="store_true", help="use $HCCMF_LIB as built (a -DHCCMF_DIAG_TRACE build)")
    ap.add_argument("--bal", action="store_true", help="degree-balanced column blocks (R30)")
    args = ap.parse_args()
    if not args.nobuild:
        lib = "/tmp/libhccmf_trace.so"
        subprocess.check_call([sys.executable, os.path.join(ROOT, "paper_conf_icpp_huangylhbl21_b200", "_build.py"),
                               "-DHCCMF_DIAG_TRACE", f"--out={lib}"])
        os.environ["HCCMF_LIB"] = lib
    trace = "/tmp/det_trace.bin"
    import numpy as np
    import synth
    from paper_conf_icpp_huangylhbl21_b200 import Model

    cfg = synth.CONFIGS[args.config]
    B = args.B
    (u, v, r), _ = synth.make(cfg)
    with Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam) as mdl:
        mdl.load(u, v, r)
        mdl.set_option("det_wave", args.wave)
        mdl.partition(1, (B, B), "DP0", seed=cfg.seed, col_balance=args.bal)
        mdl.init(1)
        mdl.train_epoch("det", "none")  # warm
        os.environ["HCCMF_TRACE_OUT"] = trace
        mdl.train_epoch("det", "none")
        del os.environ["HCCMF_TRACE_OUT"]
        _, off, _, _ = mdl.get_partition()
    W = 4 if args.wave == 3 else 3
    T = np.fromfile(trace, dtype=np.uint32).reshape(B, B, W).astype(np.int64)
    steps = polls = segs = None
    if W == 4:  # chain wavefront word 3: steps (12 bits) | dependency polls (16) | segments (4), warp 0
        w3 = T[..., 3].copy()
        steps, polls, segs = w3 & 0xFFF, (w3 >> 12) & 0xFFFF, (w3 >> 28) & 0xF
    T = T[..., :3]
    T -= T[:, 0, 0].min()
    begin, got, end = T[..., 0], T[..., 1], T[..., 2]
    cnt = np.diff(off).reshape(B, B)
    ii = np.arange(B)[:, None]
    tt = np.arange(B)[None, :]
    n = cnt[ii, (ii + tt) % B]  # ratings of block (i, (i+t) mod B)
    dur = end - got
    nz = n > 0
    A = np.stack([np.ones(nz.sum()), n[nz]], 1)
    (o, c), *_ = np.linalg.lstsq(A, dur[nz].astype(float), rcond=None)
    # critical path: from the last release back to stratum 0
    i = int(np.argmax(end[:, B - 1]))
    t = B - 1
    path_blocks = path_ratings = path_dur = path_handoff = path_own = path_steps = path_polls = path_segs = 0
    while t >= 0:
        path_blocks += 1
        path_ratings += int(n[i, t])
        if steps is not None:
            path_steps += int(steps[i, t])
            path_polls += int(polls[i, t])
            path_segs += int(segs[i, t])
        path_dur += int(dur[i, t])
        if t == 0:
            break
        pred = (i + 1) % B
        if end[pred, t - 1] >= end[i, t - 1]:  # waited on the column block's previous owner
            path_handoff += int(got[i, t] - end[pred, t - 1])
            i = pred
        else:
            path_own += int(got[i, t] - end[i, t - 1])
        t -= 1
    out = {"config": args.config, "B": B, "wave": args.wave, "col_balance": bool(args.bal),
           "epoch_ms": float(end.max() / 1e6),
           "fit_block_ns": {"o": float(o), "c_per_rating": float(c)},
           "empty_block_ns_mean": float(dur[~nz].mean()) if (~nz).any() else None,
           "mean_wait_ns": float((got - begin)[:, 1:].mean()),
           "busy_fraction": float(dur.sum() / (B * end.max())),
           "critical_path": {"blocks": path_blocks, "ratings": path_ratings, "in_blocks_ms": path_dur / 1e6,
                             "handoff_ms": path_handoff / 1e6, "own_gap_ms": path_own / 1e6,
                             "steps": path_steps, "polls": path_polls, "segments": path_segs},
           "row_max_ratings": int(cnt.sum(1).max()), "col_max_ratings": int(cnt.sum(0).max())}
    if steps is not None:
        A2 = np.stack([np.ones(nz.sum()), steps[nz]], 1)
        (o2, c2), *_ = np.linalg.lstsq(A2, dur[nz].astype(float), rcond=None)
        out["fit_block_ns_steps"] = {"o": float(o2), "c_per_step": float(c2)}
        out["steps_per_rating"] = float(steps[nz].sum() / n[nz].sum())
    os.makedirs("gpurun_out", exist_ok=True)
    with open(f"gpurun_out/det_trace_w{args.wave}_B{B}{'_bal' if args.bal else ''}.json", "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
