#!/usr/bin/env python
"""Ceiling of the Hogwild q_v round trip on this B200: how many
"updates" per second the SM -> L2 path sustains when every update only loads one q row
(512 B fp32 / 256 B binary16, L2-resident Q) and sends it back as a vector reduction,
with the same warp count, record stream and one-rating-ahead pipelining as
sgd_warp_kernel but none of the SGD arithmetic (the reduced value depends on the load,
as in the real kernel).  GPU only; prints one JSON line and writes
gpurun_out/probe_l2_roundtrip.json.  The item stream is the bench's C3 (or --config)
sorted record stream, so L2 slice hot spots match the real run.

    python tools/probe_l2_roundtrip.py [--config c3] [--warps 4736]
"""
import argparse
import ctypes
import json
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

SRC = r'''
#include <cstdint>
#include <cuda_fp16.h>
// MODE 0: ld + dependent red (fp32 rows), 1: same with binary16 rows,
// 2: ld only (fp32), 3: red only (fp32), 4: records only, 5: TMA bulk reduce only,
// 6: ld + dependent TMA bulk reduce
template <int MODE>
__device__ void body(const int* __restrict__ rv, const float* __restrict__ rr, long long nrec, char* Q, int rowb,
                     long long per_warp, float* sink) {
  const int lane = threadIdx.x & 31;
  const long long w = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
  long long lo = w * per_warp, hi = lo + per_warp;
  if (hi > nrec) hi = nrec;
  if (lo >= hi) return;
  const int lb = (MODE == 1) ? 8 : 16;
  __shared__ float4 stage_all[8][64];
  float4* stage = stage_all[(threadIdx.x >> 5) & 7];
  float acc = 0.f;
  int wv = 0; float wr = 0.f;
  long long wb = lo;
  if (wb + lane < hi) { wv = __ldcs(rv + wb + lane); wr = __ldcs(rr + wb + lane); }
  int cv = __shfl_sync(~0u, wv, 0);
  float cr = __shfl_sync(~0u, wr, 0);
  float4 qc = make_float4(0, 0, 0, 0), qn;
  uint2 hc = make_uint2(0, 0), hn;
  const char* qp = Q + (long long)cv * rowb + lane * lb;
  if (MODE == 0 || MODE == 2 || MODE == 6) qc = __ldcg(reinterpret_cast<const float4*>(qp));
  if (MODE == 1) hc = __ldcg(reinterpret_cast<const uint2*>(qp));
  for (long long j = lo; j < hi; ++j) {
    const long long jn = j + 1;
    int nv = cv; float nr = cr;
    if (jn < hi) {
      if (jn - wb == 32) {
        wb += 32;
        if (wb + lane < hi) { wv = __ldcs(rv + wb + lane); wr = __ldcs(rr + wb + lane); }
      }
      nv = __shfl_sync(~0u, wv, (int)(jn - wb));
      nr = __shfl_sync(~0u, wr, (int)(jn - wb));
    }
    const char* np = Q + (long long)nv * rowb + lane * lb;
    if (jn < hi) {
      if (MODE == 0 || MODE == 2 || MODE == 6) qn = __ldcg(reinterpret_cast<const float4*>(np));
      if (MODE == 1) hn = __ldcg(reinterpret_cast<const uint2*>(np));
    }
    const float s = cr * 1e-30f;  // the reduced value depends on the record and the load
    if (MODE == 0) {
      asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(qp), "f"(qc.x * s),
                   "f"(qc.y * s), "f"(qc.z * s), "f"(qc.w * s) : "memory");
    } else if (MODE == 1) {
      __half2 a = *reinterpret_cast<__half2*>(&hc.x), b = *reinterpret_cast<__half2*>(&hc.y);
      a = __hmul2(a, __float2half2_rn(s)); b = __hmul2(b, __float2half2_rn(s));
      asm volatile("red.relaxed.gpu.global.add.noftz.v2.f16x2 [%0], {%1, %2};" ::"l"(qp),
                   "r"(*reinterpret_cast<unsigned*>(&a)), "r"(*reinterpret_cast<unsigned*>(&b)) : "memory");
    } else if (MODE == 2) {
      acc += qc.x + qc.y + qc.z + qc.w;
    } else if (MODE == 3) {
      asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(qp), "f"(s), "f"(s),
                   "f"(s), "f"(s) : "memory");
    } else if (MODE == 5 || MODE == 6) {
      // TMA bulk reduction of the whole 512 B row from shared memory (async proxy), the
      // warp's staging slot double-buffered; MODE 6 reduces the loaded row (dependent)
      float4* st = stage + ((j & 1) << 5) + lane;
      asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      __syncwarp();
      *st = MODE == 6 ? make_float4(qc.x * s, qc.y * s, qc.z * s, qc.w * s) : make_float4(s, s, s, s);
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) {
        const unsigned sa = (unsigned)__cvta_generic_to_shared(stage + ((j & 1) << 5));
        asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], 512;"
                     :: "l"(Q + (long long)cv * rowb), "r"(sa) : "memory");
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
    } else {
      acc += s + (float)cv;
    }
    qc = qn; hc = hn; qp = np; cv = nv; cr = nr;
  }
  if (MODE == 5 || MODE == 6) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  if (acc == 1.2345f) sink[0] = acc;
}
extern "C" __global__ void __launch_bounds__(256) probe0(const int* rv, const float* rr, long long n, char* Q, int rowb, long long pw, float* s) { body<0>(rv, rr, n, Q, rowb, pw, s); }
extern "C" __global__ void __launch_bounds__(256) probe1(const int* rv, const float* rr, long long n, char* Q, int rowb, long long pw, float* s) { body<1>(rv, rr, n, Q, rowb, pw, s); }
extern "C" __global__ void __launch_bounds__(256) probe2(const int* rv, const float* rr, long long n, char* Q, int rowb, long long pw, float* s) { body<2>(rv, rr, n, Q, rowb, pw, s); }
extern "C" __global__ void __launch_bounds__(256) probe3(const int* rv, const float* rr, long long n, char* Q, int rowb, long long pw, float* s) { body<3>(rv, rr, n, Q, rowb, pw, s); }
extern "C" __global__ void __launch_bounds__(256) probe5(const int* rv, const float* rr, long long n, char* Q, int rowb, long long pw, float* s) { body<5>(rv, rr, n, Q, rowb, pw, s); }
extern "C" __global__ void __launch_bounds__(256) probe6(const int* rv, const float* rr, long long n, char* Q, int rowb, long long pw, float* s) { body<6>(rv, rr, n, Q, rowb, pw, s); }
// MODE 7: binary16 rows, 16 lanes x 16 B per rating, two independent rating streams per
// warp (half-warps), load + dependent red.v4.f16x2
extern "C" __global__ void __launch_bounds__(256) probe7(const int* __restrict__ rv, const float* __restrict__ rr,
                                                         long long nrec, char* Q, int rowb, long long per_group,
                                                         float* sink) {
  const int lane = threadIdx.x & 31, hl = lane & 15, half = lane >> 4;
  const long long grp = ((blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5) * 2 + half;
  long long lo = grp * per_group, hi = lo + per_group;
  if (hi > nrec) hi = nrec;
  const long long n = hi > lo ? hi - lo : 0;
  const long long nmax = per_group;  // both halves loop the same count (lock step)
  int cv = n ? __ldcs(rv + lo) : 0;
  uint4 qc = __ldcg(reinterpret_cast<const uint4*>(Q + (long long)cv * rowb + hl * 16)), qn = qc;
  for (long long j = 0; j < nmax; ++j) {
    const bool live = j < n, nlive = j + 1 < n;
    int nv = cv;
    float r = live ? __ldcs(rr + lo + j) : 0.f;
    if (nlive) nv = __ldcs(rv + lo + j + 1);
    if (nlive) qn = __ldcg(reinterpret_cast<const uint4*>(Q + (long long)nv * rowb + hl * 16));
    if (live) {
      const __half2 sc = __float2half2_rn(r * 1e-30f);
      __half2 a = __hmul2(*reinterpret_cast<__half2*>(&qc.x), sc), b = __hmul2(*reinterpret_cast<__half2*>(&qc.y), sc);
      __half2 c = __hmul2(*reinterpret_cast<__half2*>(&qc.z), sc), d = __hmul2(*reinterpret_cast<__half2*>(&qc.w), sc);
      asm volatile("red.relaxed.gpu.global.add.noftz.v4.f16x2 [%0], {%1, %2, %3, %4};" ::"l"(Q + (long long)cv * rowb + hl * 16),
                   "r"(*reinterpret_cast<unsigned*>(&a)), "r"(*reinterpret_cast<unsigned*>(&b)),
                   "r"(*reinterpret_cast<unsigned*>(&c)), "r"(*reinterpret_cast<unsigned*>(&d)) : "memory");
    }
    qc = qn; cv = nv;
  }
  if (sink[0] == 1.2345f) sink[1] = 0.f;
}
// MODE 8 / 9: fp32 rows in a 64-byte-chunk interleaved layout (chunk j of item v at
// ((j * n + v) * 64): a row's 8 chunks sit in 8 different lines / L2 slices instead of 4),
// MODE 8: red only, MODE 9: load + dependent red
template <int MODE>
__device__ void body_il(const int* __restrict__ rv, const float* __restrict__ rr, long long nrec, char* Q, int n,
                        long long per_warp, float* sink) {
  const int lane = threadIdx.x & 31;
  const long long w = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
  long long lo = w * per_warp, hi = lo + per_warp;
  if (hi > nrec) hi = nrec;
  if (lo >= hi) return;
  const long long off_l = (long long)(lane >> 2) * n * 64 + (lane & 3) * 16;
  int wv = 0; float wr = 0.f;
  long long wb = lo;
  if (wb + lane < hi) { wv = __ldcs(rv + wb + lane); wr = __ldcs(rr + wb + lane); }
  int cv = __shfl_sync(~0u, wv, 0);
  float cr = __shfl_sync(~0u, wr, 0);
  const char* qp = Q + off_l + (long long)cv * 64;
  float4 qc = MODE == 9 ? __ldcg(reinterpret_cast<const float4*>(qp)) : make_float4(0, 0, 0, 0), qn = qc;
  for (long long j = lo; j < hi; ++j) {
    const long long jn = j + 1;
    int nv = cv; float nr = cr;
    if (jn < hi) {
      if (jn - wb == 32) {
        wb += 32;
        if (wb + lane < hi) { wv = __ldcs(rv + wb + lane); wr = __ldcs(rr + wb + lane); }
      }
      nv = __shfl_sync(~0u, wv, (int)(jn - wb));
      nr = __shfl_sync(~0u, wr, (int)(jn - wb));
    }
    const char* np = Q + off_l + (long long)nv * 64;
    if (MODE == 9 && jn < hi) qn = __ldcg(reinterpret_cast<const float4*>(np));
    const float sc = cr * 1e-30f;
    if (MODE == 9)
      asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(qp), "f"(qc.x * sc),
                   "f"(qc.y * sc), "f"(qc.z * sc), "f"(qc.w * sc) : "memory");
    else
      asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(qp), "f"(sc), "f"(sc),
                   "f"(sc), "f"(sc) : "memory");
    qc = qn; qp = np; cv = nv; cr = nr;
  }
  if (sink[0] == 1.2345f) sink[1] = 0.f;
}
extern "C" __global__ void __launch_bounds__(256) probe8(const int* rv, const float* rr, long long n, char* Q, int rowb, long long pw, float* s) { body_il<8>(rv, rr, n, Q, rowb, pw, s); }
extern "C" __global__ void __launch_bounds__(256) probe9(const int* rv, const float* rr, long long n, char* Q, int rowb, long long pw, float* s) { body_il<9>(rv, rr, n, Q, rowb, pw, s); }
extern "C" __global__ void __launch_bounds__(256) probe4(const int* rv, const float* rr, long long n, char* Q, int rowb, long long pw, float* s) { body<4>(rv, rr, n, Q, rowb, pw, s); }
'''

MODES = {0: "ld+red fp32 (512+512 B)", 1: "ld+red binary16 (256+256 B)", 2: "ld only fp32",
         3: "red only fp32", 4: "records only", 5: "bulk reduce only fp32 (TMA, 512 B)",
         6: "ld + dependent bulk reduce fp32 (TMA)", 7: "ld+red binary16, 16 lanes x 16 B, 2 ratings per warp",
         8: "red only fp32, 64 B-chunk interleaved rows", 9: "ld+red fp32, 64 B-chunk interleaved rows"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="c3")
    ap.add_argument("--warps", type=int, default=4736)
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()
    import numpy as np
    import torch
    import synth
    from paper_conf_icpp_huangylhbl21_b200 import Model
    from cuda.bindings import driver as drv

    tmp = tempfile.mkdtemp()
    cu, cubin = os.path.join(tmp, "p.cu"), os.path.join(tmp, "p.cubin")
    open(cu, "w").write(SRC)
    subprocess.check_call(["nvcc", "-O3", "-gencode", "arch=compute_100a,code=sm_100a", "-cubin", "-o", cubin, cu])
    torch.cuda.init()
    torch.zeros(1, device="cuda")
    drv.cuInit(0)
    _, mod = drv.cuModuleLoad(cubin.encode())

    cfg = synth.CONFIGS[args.config]
    (u, v, r), _ = synth.make(cfg)
    k = cfg.k
    with Model(cfg.m, cfg.n, k, cfg.gamma, cfg.lam) as mdl:  # the bench's sorted record stream
        mdl.load(u, v, r)
        mdl.partition(1, (1, 1), "DP0", seed=cfg.seed)
        ru, rv, rr = mdl.records()
    del u, v, r
    rv = torch.from_numpy(rv).cuda()
    rr = torch.from_numpy(rr).cuda()
    nrec = rv.numel()
    out = {"config": args.config, "warps": args.warps, "nrec": nrec, "k": k}
    per_warp = (nrec + args.warps - 1) // args.warps
    Q = torch.zeros(cfg.n * k, dtype=torch.float32, device="cuda")
    sink = torch.zeros(1, device="cuda")
    for mode in range(10):
        _, fn = drv.cuModuleGetFunction(mod, f"probe{mode}".encode())
        rowb = cfg.n if mode in (8, 9) else k * (2 if mode in (1, 7) else 4)  # 8, 9: the item count
        pw = (nrec + 2 * args.warps - 1) // (2 * args.warps) if mode == 7 else per_warp
        vals = [ctypes.c_void_p(rv.data_ptr()), ctypes.c_void_p(rr.data_ptr()), ctypes.c_longlong(nrec),
                ctypes.c_void_p(Q.data_ptr()), ctypes.c_int(rowb), ctypes.c_longlong(pw),
                ctypes.c_void_p(sink.data_ptr())]
        ptrs = (ctypes.c_void_p * len(vals))(*[ctypes.cast(ctypes.pointer(x), ctypes.c_void_p) for x in vals])
        blocks = (args.warps * 32 + 255) // 256
        times = []
        for rep in range(args.reps + 1):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record()
            drv.cuLaunchKernel(fn, blocks, 1, 1, 256, 1, 1, 0, 0, ptrs, 0)
            e1.record()
            torch.cuda.synchronize()
            if rep:
                times.append(e0.elapsed_time(e1) / 1e3)
        t = float(np.median(times))
        out[MODES[mode]] = {"ms": t * 1e3, "G_upd_per_s": nrec / t / 1e9}
    os.makedirs("gpurun_out", exist_ok=True)
    with open("gpurun_out/probe_l2_roundtrip.json", "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
