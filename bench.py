#!/usr/bin/env python
"""bench.py -- rating updates/s of the HCC-MF hot path on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c3] [--sched hogwild]
    torchrun --nproc-per-node N bench.py --gpus N ...         (one rank per GPU, NCCL)
    python bench.py --impl reference ...                       (the oracle arm, host cores)

A "step" is one training epoch over every rating of the workload, the per-epoch
hot path of the paper's workflow (L549-L557): the SGD kernel over all nnz
(a5/a6), the Q synchronisation across GPUs (a7, G > 1) and the RMSE evaluation
of the held-out test set (a8, Fig. 7).  Preprocessing (a1-a4) happens once
before training, as in the paper (steps 1-3, L543-L548); the `e2e` object times
the WHOLE job through the public API from host buffers (ingest + shuffle +
partition + sort + init + epochs + RMSE + export), H2D/D2H inside the timed
region.  value = nnz * steps / device time (Eq. 8 "computing power", L1709-L1715),
max over ranks.  Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402

METRIC = "rating updates/sec (whole box)"
STORAGE = {"fp32": 0, "fp16": 1, "fp16sr": 2}
# what ncu says actually binds the SGD kernel (profiles/r01_ncu_c3_ring.md, C3): the
# formula roofline above counts p_u / q_v bytes that stay in registers / L2
BINDING = {
    "fp32": {"unit": "L2 atomic units (q_v vector reductions, 512 B/update; 48.7 % avg, 75.7 % hottest slice; "
                     "L1TEX->XBAR request port 71 %)", "ncu_pct_of_peak": 75.7,
             "dram_bytes_per_update": 17.1, "source": "profiles/r01_ncu_c3_final.md"},
    "fp16": {"unit": "instruction issue (stochastic-rounding hash and conversions, 66.7 instructions/update)",
             "ncu_pct_of_peak": 74.8, "dram_bytes_per_update": 17.0, "source": "profiles/r01_ncu_c3_final.md"},
}
PROBE = os.path.join(os.path.dirname(os.path.abspath(__file__)), "profiles", "r01_probe_l2_roundtrip_c3.json")


def binding_unit(storage, args, kernel_rate):
    """The unit that bounds the SGD kernel (ncu) and, for the C3 Hogwild kernel, the
    measured ceiling of its q_v round trip on this B200 (tools/probe_l2_roundtrip.py:
    same record stream and warp count, no SGD arithmetic): the reductions alone for fp32
    rows, load + reduction for binary16 rows."""
    b = dict(BINDING.get("fp32" if storage == "fp32" else "fp16"))
    if args.config == "c3" and args.sched == "hogwild" and os.path.exists(PROBE):
        with open(PROBE) as f:
            pr = json.load(f)
        key = "red only fp32" if storage == "fp32" else "ld+red binary16 (256+256 B)"
        ceil = pr[key]["G_upd_per_s"] * 1e9
        b["ceiling"] = {"probe": key, "updates_per_s": ceil, "kernel_updates_per_s": kernel_rate,
                        "frac": kernel_rate / ceil, "source": os.path.relpath(PROBE, os.path.dirname(PROBE) + "/..")}
    return b


UNIT = "updates/s"
FALLBACK_HBM_GBS = 6650.0
DEVICE_GEN_NNZ = 1_000_000_000


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c3", choices=sorted(synth.CONFIGS))
    ap.add_argument("--sched", default="hogwild", choices=["hogwild", "det"])
    ap.add_argument("--sync", default=None, choices=["none", "ring", "allreduce"])
    ap.add_argument("--grid", default=None, help="Br,Bc (default: hogwild 1,4G (ring) or 1,ceil(|Q|/80MB); det 64,64G)")
    ap.add_argument("--warps", type=int, default=0)
    ap.add_argument("--task", type=int, default=0)
    ap.add_argument("--vec", type=int, default=0, help="float4 slots per lane (0 = library auto)")
    ap.add_argument("--depth", type=int, default=0, help="Hogwild q_v prefetch distance (0 = library auto)")
    ap.add_argument("--no-det-leg", dest="det_leg", action="store_false",
                    help="skip the DET-schedule leg (C3 only) reported beside the Hogwild headline")
    ap.add_argument("--det-wave", type=int, default=1, choices=[0, 1, 2],
                    help="DET: 1 wavefront with Q slabs in shared memory, 2 wavefront, 0 per-stratum launches")
    ap.add_argument("--impl", default="hccmf", choices=["hccmf", "reference"])
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--storage", default="fp32", choices=["fp32", "fp16", "fp16sr"],
                    help="Q storage of the headline number (fp16 = binary16 Q, fp32 math, R26; "
                         "fp16sr = with stochastic rounding, R27)")
    ap.add_argument("--fp16-leg", default="fp16sr", choices=["fp16", "fp16sr", "none"],
                    help="secondary binary16-Q measurement added to the JSON line")
    return ap.parse_args()


# ------------------------------------------------------------------ helpers
class Clocks:
    """nvidia-smi sampler for the timed region (B200_PROFILING.md clocks line)."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index, self.rows, self.proc = index, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        self.proc.wait(timeout=5)
        self.t.join(timeout=2)
        sm = [float(r[0]) for r in self.rows if len(r) >= 8 and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) >= 8 and r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows if len(r) >= 8 for i in range(4) if r[4 + i] == "Active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(sm)}


def hbm_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def ncu_traffic(cfg_name, sched):
    """DRAM bytes per launch of the SGD kernel from the committed ncu --set full summary, if any."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            return json.load(f).get(f"{cfg_name}/{sched}")
    except Exception:
        return None


def epochs_to_rmse(name, curve):
    """first epoch whose test RMSE <= oracle RMSE@E + 0.005, against the
    oracle's stored reference curve (tests/golden/oracle_curve_<cfg>.json, written by
    tools/oracle_curves.py from oracle/ alone)."""
    out = {"test_per_epoch": [round(x, 6) for x in curve], "epochs": len(curve) - 1}
    try:
        with open(os.path.join(ROOT, "tests", "golden", f"oracle_curve_{name}.json")) as f:
            ref = json.load(f)
    except OSError:
        return out
    E = ref["epochs"]
    target = ref["test_rmse"][E] + 0.005
    first = lambda c: next((e for e in range(1, len(c)) if c[e] <= target), None)  # noqa: E731
    out.update({"oracle_E": E, "oracle_at_E": ref["test_rmse"][E], "target": target,
                "epochs_to_rmse": first(curve), "oracle_epochs_to_rmse": first(ref["test_rmse"]),
                "band_at_E": (abs(curve[E] - ref["test_rmse"][E]) if len(curve) > E else None)})
    return out


def host_mem_available():
    try:
        with open("/proc/meminfo") as f:
            for line in f:
                if line.startswith("MemAvailable:"):
                    return int(line.split()[1]) * 1024
    except OSError:
        pass
    return 0


def host_cpu():
    model = "unknown"
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return model, os.cpu_count()


def oracle_sample(cfg, u, v, r, seconds):
    """The oracle, as it stands, on a bounded prefix sample of the same workload (1 host core)."""
    import oracle
    S = int(min(len(u), 2_000_000 if cfg.k >= 64 else 8_000_000))
    prob = oracle.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u[:S], v[:S], r[:S], G=1, Br=1, Bc=1,
                          seed=cfg.seed)
    prob.init(1)
    # one host core: pin this thread while the serial oracle runs
    saved = os.sched_getaffinity(0) if hasattr(os, "sched_getaffinity") else None
    core = max(saved) if saved else -1
    if saved:
        os.sched_setaffinity(0, {core})
    try:
        t0 = time.perf_counter()
        epochs = 0
        while True:
            prob.epoch("serial", "none")
            epochs += 1
            if time.perf_counter() - t0 >= seconds:
                break
        dt = time.perf_counter() - t0
    finally:
        if saved:
            os.sched_setaffinity(0, saved)
    return S * epochs / dt, S, epochs, dt, core


# ------------------------------------------------------------ reference arm
def run_reference(args, cfg, rank, world):
    if rank != 0:
        return
    import oracle
    S = int(min(cfg.nnz, 1_000_000 if cfg.k >= 64 else 4_000_000))
    if cfg.kind == "planted":
        (u, v, r), _ = synth.make(cfg, n_test=1)
    else:  # a bounded sample drawn from the workload's distribution (never the full 37 GB of C5)
        (u, v, r), _ = synth.powerlaw(cfg.m, cfg.n, S, cfg.seed, cfg.alpha, cfg.scale, n_test=0)
    prob = oracle.Problem(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, u[:S], v[:S], r[:S], seed=cfg.seed)
    prob.init(1)
    for _ in range(args.warmup):
        prob.epoch("serial", "none")
    t0 = time.perf_counter()
    for _ in range(args.steps):
        prob.epoch("serial", "none")
    dt = time.perf_counter() - t0
    val = S * args.steps / dt
    model, ncpu = host_cpu()
    sample = (f"one serial fp64 oracle epoch over {S} ratings drawn from the {cfg.name} distribution "
              f"(k={cfg.k}) per step; 1 of {ncpu} host cores ({model})")
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{cfg.name} ({args.config})", "m": cfg.m, "n": cfg.n, "nnz": cfg.nnz, "k": cfg.k,
                   "gamma": cfg.gamma, "lambda": cfg.lam, "sample_ratings_per_step": S},
        "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample},
        "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


# --------------------------------------------------------------- main arm
def main():
    args = parse()
    cfg = synth.CONFIGS[args.config]
    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    if args.impl == "reference":
        run_reference(args, cfg, rank, world)
        return

    import torch
    import torch.distributed as dist

    import paper_conf_icpp_huangylhbl21_b200 as hc

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    G = world
    sync = args.sync or ("none" if G == 1 else "ring")
    if args.grid:
        Br, Bc = (int(x) for x in args.grid.split(","))
    elif args.sched == "hogwild":
        # ring: 4 column blocks per group so each block's transfer overlaps the next
        # block's compute (hidden synchronisation); one GPU: column-block-major phases
        # whenever Q exceeds ~80 MB of L2 (C4: 320 MB -> 4 phases)
        qmb = cfg.n * cfg.k * 4 / 80e6
        Br, Bc = 1, (4 * G if sync == "ring" else max(1, round(qmb)))
    else:
        Br, Bc = 64, 64 * (G if sync == "ring" else 1)

    t_gen = time.perf_counter()
    on_device = cfg.nnz > DEVICE_GEN_NNZ  # C5: 37 GB of COO, drawn on the GPU (synth.make_device)
    if on_device:
        (du, dv, dr), (dtu, dtv, dtr) = synth.make_device(cfg, device=f"cuda:{local}")
        u = v = r = tu = tv = tr = None
        S = 2_000_000
        sample = (du[:S].cpu().numpy(), dv[:S].cpu().numpy(), dr[:S].cpu().numpy())
    else:
        (u, v, r), (tu, tv, tr) = synth.make(cfg)
        sample = (u, v, r)
    torch.cuda.synchronize()
    t_gen = time.perf_counter() - t_gen

    stream = torch.cuda.Stream()
    mdl = hc.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, dist=world > 1, device=local)
    mdl.set_stream(stream)
    if args.warps:
        mdl.set_option("hogwild_warps", args.warps)
    if args.task:
        mdl.set_option("task_ratings", args.task)
    if args.vec:
        mdl.set_option("vec", args.vec)
    if args.depth:
        mdl.set_option("prefetch_depth", args.depth)
    if args.det_wave != 1:
        mdl.set_option("det_wave", args.det_wave)
    if not on_device:
        du, dv, dr = (torch.from_numpy(x).cuda() for x in (u, v, r))
        dtu, dtv, dtr = (torch.from_numpy(x).cuda() for x in (tu, tv, tr))
    nnz, nt = int(du.numel()), int(dtu.numel())
    torch.cuda.synchronize()
    t_prep = time.perf_counter()
    mdl.load(du, dv, dr)
    if on_device:  # keep a host-free copy only where it fits; free the generator's 37 GB first
        del du, dv, dr
        torch.cuda.empty_cache()
    mdl.partition(G, (Br, Bc), "DP0", seed=cfg.seed, storage=args.storage)
    mdl.init(1)
    t_prep = time.perf_counter() - t_prep
    info = mdl.info()
    if not on_device:
        del du, dv, dr
    peak, peak_src = hbm_peak()
    local_nnz = info["local_nnz"]

    def measure(storage, sched=None, steps=None):
        """W warm-up + K timed steps (epoch + Q sync + test RMSE) from a fresh init(1)."""
        sched = sched or args.sched
        steps = steps or args.steps
        rm0 = mdl.rmse(dtu, dtv, dtr)
        mdl.set_option("sync_stream", 0)

        def step(ev=None):
            if ev is not None:
                ev[0].record(stream)
            mdl.train_epoch(sched, sync)
            if ev is not None:
                ev[1].record(stream)
            return mdl.rmse(dtu, dtv, dtr)

        curve = [rm0] + [step() for _ in range(args.warmup)]
        kev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
               for _ in range(steps)]
        t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        clocks = Clocks(local)
        clocks.start()
        time.sleep(0.3)
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        l0 = hc.kernel_launches()
        t_start.record(stream)
        rms = [step(kev[i]) for i in range(steps)]
        t_end.record(stream)
        launches = hc.kernel_launches() - l0  # counted by the library at its launch sites
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        clk = clocks.stop()
        mdl.set_option("sync_stream", 1)
        ms = t_start.elapsed_time(t_end)
        k_ms = [a.elapsed_time(b) for a, b in kev]
        if world > 1:
            t = torch.tensor([ms, float(np.mean(k_ms))], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms, kmean = t.tolist()
        else:
            kmean = float(np.mean(k_ms))
        # roofline of the dominant kernel (the SGD epoch): north_star bytes/update = record
        # (12 B) + read and write of p_u and q_v: 12 + 16k (fp32), 12 + 12k (binary16 Q)
        b_upd = 12 + (16 if storage == "fp32" else 12) * cfg.k
        achieved = local_nnz * b_upd / (kmean / 1e3) / 1e9
        roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": ncu_traffic(args.config + ("" if storage == "fp32" else "-" + storage), sched),
                "kernel": "sgd_warp_kernel (a5/a6 epoch incl. Q sync%s)"
                          % ("" if storage == "fp32" else ", binary16 round-in/write-back of Q"),
                "bytes_per_update": b_upd, "updates_per_launch": local_nnz, "kernel_ms": kmean,
                "kernel_share_of_step": kmean / (ms / steps), "peak_source": peak_src,
                "binding_unit": binding_unit(storage, args, local_nnz / (kmean / 1e3)) if sched == "hogwild"
                else None}
        roof["kernel_launches_timed"] = launches
        return nnz * steps / (ms / 1e3), ms, roof, clk, curve + rms

    value, ms, roof, clk, curve = measure(args.storage)

    out = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
           "config": {"workload": f"{cfg.name} ({args.config})", "m": cfg.m, "n": cfg.n, "nnz": nnz, "k": cfg.k,
                      "test_ratings": nt, "gamma": cfg.gamma, "lambda": cfg.lam, "sched": args.sched,
                      "sync": sync, "grid": [Br, Bc], "parallelism": f"dp{world} (row shards, Q {sync})",
                      "step": "1 SGD epoch over all nnz + Q sync + test RMSE",
                      "l2": "inputs larger than L2 (records %.2f GB > 126 MB); Q is L2-resident by design"
                            % (12 * nnz / 1e9),
                      "hogwild_tasks": info["n_tasks"], "key_bits": info["key_bits"]},
           "roofline": roof, "clocks": clk,
           "gpu_launches": roof.pop("kernel_launches_timed"),
           "rmse": epochs_to_rmse(args.config, curve),
           "prep_s": t_prep, "gen_s": t_gen,
           "paper_context": {"netflix_hcc_updates_per_s": 2228476993,
                             "hardware": "2x Xeon Gold 6242 + RTX 2080 + RTX 2080S (Table 4, L2001)"}}
    out["config"]["storage"] = args.storage
    # secondary leg: the same workload with Q stored in binary16 (R26),
    # fp32 arithmetic; same steps, same clocks rule; reported beside the fp32 headline
    if args.storage == "fp32" and cfg.k % 128 == 0 and args.fp16_leg != "none":
        mdl.set_option("storage", STORAGE[args.fp16_leg])
        mdl.init(1)
        v16, ms16, roof16, clk16, curve16 = measure(args.fp16_leg)
        out["storage_fp16"] = {"storage": args.fp16_leg, "value": v16, "unit": UNIT,
                               "ms_per_step": ms16 / args.steps,
                               "gpu_launches": roof16.pop("kernel_launches_timed"), "roofline": roof16,
                               "clocks": clk16, "rmse": epochs_to_rmse(args.config, curve16),
                               "note": "Q held as IEEE binary16 during epochs (fp32 math, P fp32)%s; "
                                       "same band vs the fp64 oracle"
                                       % (", stochastic rounding of every q write" if args.fp16_leg == "fp16sr"
                                          else "")}

    # secondary leg: the deterministic schedule (a5) on the same data, the bench's DET
    # configuration (one shard, 2048 x 2048 grid, the shared-memory-slab wavefront: one
    # launch per epoch), fp32; parity with the oracle is the full-size GPU test's
    if (args.det_leg and args.sched == "hogwild" and world == 1 and args.config == "c3" and not on_device):
        mdl.close()  # the handle released its input COO after partition: a fresh one for DET
        mdl = hc.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, device=local)
        mdl.set_stream(stream)
        mdl.load(u, v, r)
        mdl.partition(1, (2048, 2048), "DP0", seed=cfg.seed)
        mdl.init(1)
        kd = min(args.steps, 3)
        vd, msd, roofd, clkd, curved = measure("fp32", sched="det", steps=kd)
        roofd["kernel"] = "sgd_wave_slab_kernel (a5 DET epoch, one launch)"
        out["det"] = {"sched": "det", "grid": [2048, 2048], "value": vd, "unit": UNIT, "steps": kd,
                      "warmup": args.warmup, "ms_per_step": msd / kd,
                      "gpu_launches": roofd.pop("kernel_launches_timed"), "roofline": roofd, "clocks": clkd,
                      "test_rmse": curved[-1],
                      "note": "serial-equivalent FPSGD strata (R19); bound by the hottest column block's "
                              "serial chain (profiles/r01_det_wavefront.md)"}

    mdl.close()  # free HBM before the e2e jobs build their own handles
    # ---- e2e: the whole job through the public API from pinned host buffers
    e2e_skip = None
    if on_device and not args.no_e2e:
        need = 12 * (nnz + nt) * 2 + 4 * (cfg.m + cfg.n) * cfg.k
        if host_mem_available() < need:
            e2e_skip = f"host memory {host_mem_available() / 1e9:.0f} GB < {need / 1e9:.0f} GB for pinned COO + P, Q"
        else:
            (u, v, r), (tu, tv, tr) = synth.make_device(cfg, device=f"cuda:{local}")
            u, v, r, tu, tv, tr = (x.cpu().numpy() for x in (u, v, r, tu, tv, tr))
            torch.cuda.empty_cache()
    if e2e_skip:
        out["e2e"] = {"value": None, "unit": UNIT, "skipped": e2e_skip}
    elif not args.no_e2e:
        pin = [torch.from_numpy(x).pin_memory() for x in (u, v, r, tu, tv, tr)]
        Ph = torch.empty((cfg.m, cfg.k), dtype=torch.float32).pin_memory()
        Qh = torch.empty((cfg.n, cfg.k), dtype=torch.float32).pin_memory()
        E = cfg.epochs

        def job():
            m2 = hc.Model(cfg.m, cfg.n, cfg.k, cfg.gamma, cfg.lam, dist=world > 1, device=local)
            m2.set_stream(stream)
            if args.warps:
                m2.set_option("hogwild_warps", args.warps)
            if args.vec:
                m2.set_option("vec", args.vec)
            m2.load(pin[0], pin[1], pin[2])
            m2.partition(G, (Br, Bc), "DP0", seed=cfg.seed, storage=args.storage)
            m2.init(1)
            for _ in range(E):
                m2.train_epoch(args.sched, sync)
                m2.rmse(pin[3], pin[4], pin[5])
            m2.factors(Ph, Qh)
            m2.close()

        job()
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()
        reps = 2
        t0 = time.perf_counter()
        for _ in range(reps):
            job()
        torch.cuda.synchronize()
        e2e_s = (time.perf_counter() - t0) / reps
        if world > 1:
            t = torch.tensor([e2e_s], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e2e_s = t.item()
        out["e2e"] = {"value": nnz * E / e2e_s, "unit": UNIT, "h2d_bytes_per_step": 12 * (nnz + nt),
                      "d2h_bytes_per_step": 4 * (cfg.m + cfg.n) * cfg.k + 8 * (E + 0),
                      "step": f"job: load+partition+init+{E} epochs (each with test RMSE)+export P,Q; "
                              "host pinned buffers", "s_per_step": e2e_s}

    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        val, S, ep, dt, core = oracle_sample(cfg, *sample, args.cpu_seconds)
        model, ncpu = host_cpu()
        out["cpu_baseline"] = {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle",
                               "sample": f"{ep} serial fp64 oracle epoch(s) over the first {S} ratings of the "
                                         f"same stream, {dt:.1f} s on 1 of {ncpu} cores (core {core} pinned; "
                                         f"{model})"}
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
