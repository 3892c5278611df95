// probe.cu -- ceiling of the Hogwild q_v round trip on this device:
// the handle's own sorted record stream, the same warp count as the epoch, one rating
// ahead, and per rating only the q_v traffic of the SGD kernel, none of its arithmetic:
//   mode 0: fp32 vector reductions only (red.v4.f32, 512 B at k = 128) -- the L2 atomic
//           units that bind the fp32 kernel;
//   mode 1: binary16 load + dependent reduction (ld 8 B + red.v2.f16x2 per lane);
//   mode 2: fp32 load + dependent reduction;
//   mode 3: the q_v stream alone, loads only (one row per rating);
//   mode 4: the p_u stream alone: per user run one load of the row and one store of the
//           same values back (the epoch's P traffic; the model is left unchanged).
// Modes 3 and 4 exist for ncu (the L2 hit rate of the Q and of the P stream separately,
// profiles/r02_ncu_l2_split.md).  The reductions go to a scratch copy of Q, never to the model.  bench.py divides the
// SGD kernel's rate by this ceiling (roofline.binding_frac).
#include <cuda_fp16.h>

#include "internal.cuh"

namespace hccmf {
namespace {

template <int MODE, int SLOTS>
__global__ void __launch_bounds__(256) roundtrip_kernel(const int32_t* __restrict__ rv, const float* __restrict__ rr,
                                                        int64_t nrec, char* Q, int rowb, int64_t per_warp,
                                                        float* sink) {
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t lo = w * per_warp;
  const int64_t hi = lo + per_warp < nrec ? lo + per_warp : nrec;
  if (lo >= hi) return;
  constexpr int LB = MODE == 1 ? 8 : 16;  // bytes per lane per slot
  float acc = 0.f;
  int64_t wb = lo;
  int wv = 0;
  float wr = 0.f;
  if (wb + lane < hi) {
    wv = __ldcs(rv + wb + lane);
    wr = __ldcs(rr + wb + lane);
  }
  int cv = __shfl_sync(~0u, wv, 0);
  float cr = __shfl_sync(~0u, wr, 0);
  float4 qc[SLOTS], qn[SLOTS];
  uint2 hc[SLOTS], hn[SLOTS];
#pragma unroll
  for (int s = 0; s < SLOTS; ++s) {
    const char* p = Q + (int64_t)cv * rowb + (s * 32 + lane) * LB;
    if (MODE == 2) qc[s] = __ldcg(reinterpret_cast<const float4*>(p));
    if (MODE == 1) hc[s] = __ldcg(reinterpret_cast<const uint2*>(p));
  }
  for (int64_t j = lo; j < hi; ++j) {
    const int64_t jn = j + 1;
    int nv = cv;
    float nr = cr;
    if (jn < hi) {
      if (jn - wb == 32) {
        wb += 32;
        if (wb + lane < hi) {
          wv = __ldcs(rv + wb + lane);
          wr = __ldcs(rr + wb + lane);
        }
      }
      nv = __shfl_sync(~0u, wv, (int)(jn - wb));
      nr = __shfl_sync(~0u, wr, (int)(jn - wb));
#pragma unroll
      for (int s = 0; s < SLOTS; ++s) {
        const char* p = Q + (int64_t)nv * rowb + (s * 32 + lane) * LB;
        if (MODE == 2) qn[s] = __ldcg(reinterpret_cast<const float4*>(p));
        if (MODE == 1) hn[s] = __ldcg(reinterpret_cast<const uint2*>(p));
      }
    }
    const float sc = cr * 1e-30f;  // depends on the record (and, modes 1-2, on the load)
#pragma unroll
    for (int s = 0; s < SLOTS; ++s) {
      char* p = Q + (int64_t)cv * rowb + (s * 32 + lane) * LB;
      if (MODE == 0) {
        asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(sc), "f"(sc), "f"(sc),
                     "f"(sc)
                     : "memory");
      } else if (MODE == 2) {
        asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(qc[s].x * sc),
                     "f"(qc[s].y * sc), "f"(qc[s].z * sc), "f"(qc[s].w * sc)
                     : "memory");
      } else {
        __half2 a = *reinterpret_cast<__half2*>(&hc[s].x), b = *reinterpret_cast<__half2*>(&hc[s].y);
        const __half2 h2 = __float2half2_rn(sc);
        a = __hmul2(a, h2);
        b = __hmul2(b, h2);
        asm volatile("red.relaxed.gpu.global.add.noftz.v2.f16x2 [%0], {%1, %2};" ::"l"(p),
                     "r"(*reinterpret_cast<unsigned*>(&a)), "r"(*reinterpret_cast<unsigned*>(&b))
                     : "memory");
      }
      if (MODE == 2) qc[s] = qn[s];
      if (MODE == 1) hc[s] = hn[s];
    }
    acc += sc;
    cv = nv;
    cr = nr;
  }
  if (acc == 1.2345f) sink[0] = acc;
}

// modes 3 / 4: one stream of the epoch at a time (same record order and warp split)
template <int MODE, int SLOTS>
__global__ void __launch_bounds__(256) stream_kernel(const int32_t* __restrict__ ru, const int32_t* __restrict__ rv,
                                                     int64_t nrec, const char* Q, char* P, int64_t row0, int rowb,
                                                     int64_t per_warp, float* sink) {
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t lo = w * per_warp;
  const int64_t hi = lo + per_warp < nrec ? lo + per_warp : nrec;
  float acc = 0.f;
  int cu = -1;
  float4 pr[SLOTS];
  for (int64_t j = lo; j < hi; ++j) {
    if (MODE == 3) {
      const int v = __ldcs(rv + j);
#pragma unroll
      for (int s = 0; s < SLOTS; ++s) {
        const float4 x = __ldcg(reinterpret_cast<const float4*>(Q + (int64_t)v * rowb + (s * 32 + lane) * 16));
        acc += x.x + x.y + x.z + x.w;
      }
    } else {
      const int u = __ldcs(ru + j);
      if (u != cu) {
        if (cu >= 0) {
#pragma unroll
          for (int s = 0; s < SLOTS; ++s)
            __stcg(reinterpret_cast<float4*>(P + (int64_t)(cu - row0) * rowb + (s * 32 + lane) * 16), pr[s]);
        }
#pragma unroll
        for (int s = 0; s < SLOTS; ++s)
          pr[s] = __ldcg(reinterpret_cast<const float4*>(P + (int64_t)(u - row0) * rowb + (s * 32 + lane) * 16));
        cu = u;
      }
    }
  }
  if (MODE == 4 && cu >= 0) {
#pragma unroll
    for (int s = 0; s < SLOTS; ++s)
      __stcg(reinterpret_cast<float4*>(P + (int64_t)(cu - row0) * rowb + (s * 32 + lane) * 16), pr[s]);
  }
  if (acc == 1.2345f) sink[0] = acc;
}

// modes 5-7: the q_v round trip through the TMA bulk-copy engine instead of per-lane
// LSU requests: per warp DS shared-memory row slots; lane 0 issues
//   mode 5: bulk reductions only (cp.reduce.async.bulk .add.f32 of the warp's row slot);
//   mode 6: bulk load of q_v (cp.async.bulk + mbarrier, DS - 1 ratings ahead) and the
//           dependent bulk reduction from the same slot;
//   mode 7: per-lane LSU load one rating ahead (as mode 2) + bulk reduction.
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

template <int MODE, int SLOTS, int DS>
__global__ void __launch_bounds__(256) bulk_kernel(const int32_t* __restrict__ rv, const float* __restrict__ rr,
                                                   int64_t nrec, char* Q, int64_t per_warp, float* sink) {
  constexpr int ROWB = SLOTS * 512;
  extern __shared__ __align__(128) unsigned char sm[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  unsigned char* buf = sm + wid * DS * ROWB;
  uint64_t* bar = reinterpret_cast<uint64_t*>(sm + 8 * DS * ROWB) + wid * DS;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t lo = w * per_warp;
  const int64_t hi = lo + per_warp < nrec ? lo + per_warp : nrec;
  if (lo >= hi) return;
  if (MODE == 6 && lane == 0) {
    for (int s = 0; s < DS; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar + s)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  // two record windows: lane l holds ratings wb + l and wb + 32 + l
  int64_t wb = lo;
  int wv0 = 0, wv1 = 0;
  float wr0 = 0.f, wr1 = 0.f;
  if (wb + lane < hi) wv0 = __ldcs(rv + wb + lane), wr0 = __ldcs(rr + wb + lane);
  if (wb + 32 + lane < hi) wv1 = __ldcs(rv + wb + 32 + lane), wr1 = __ldcs(rr + wb + 32 + lane);
  auto vof = [&](int64_t jj) {  // jj in [wb, wb + 64)
    const int o = (int)(jj - wb);
    const int a0 = __shfl_sync(~0u, wv0, o & 31), a1 = __shfl_sync(~0u, wv1, o & 31);
    return o < 32 ? a0 : a1;
  };
  auto issue_load = [&](int64_t jj) {  // lane 0: bulk copy of row v(jj) into slot jj % DS
    const int v = vof(jj);
    const int s = (int)((jj - lo) % DS);
    if (lane == 0) {
      const unsigned b = smem_u32(bar + s);
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(ROWB) : "memory");
      asm volatile(
          "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
              smem_u32(buf + s * ROWB)),
          "l"(Q + (int64_t)v * ROWB), "r"(ROWB), "r"(b)
          : "memory");
    }
  };
  unsigned phase = 0;  // bit s: parity of slot s's next completion
  if (MODE == 6) {
    for (int64_t jj = lo; jj < lo + DS - 1 && jj < hi; ++jj) issue_load(jj);
  }
  float4 qn[SLOTS];
  if (MODE == 7) {
    const int v = vof(lo);
#pragma unroll
    for (int s = 0; s < SLOTS; ++s) qn[s] = __ldcg(reinterpret_cast<const float4*>(Q + (int64_t)v * ROWB + (s * 32 + lane) * 16));
  }
  float acc = 0.f;
  for (int64_t j = lo; j < hi; ++j) {
    if (j - wb == 32) {
      wb += 32;
      wv0 = wv1, wr0 = wr1;
      if (wb + 32 + lane < hi) wv1 = __ldcs(rv + wb + 32 + lane), wr1 = __ldcs(rr + wb + 32 + lane);
    }
    const int cv = vof(j);
    const int o = (int)(j - wb);
    const float cr = __shfl_sync(~0u, o < 32 ? wr0 : wr1, o & 31);
    const int s = (int)((j - lo) % DS);
    float4* slot = reinterpret_cast<float4*>(buf + s * ROWB);
    const float sc = cr * 1e-30f;
    float4 qc[SLOTS];
    if (MODE == 6) {  // wait for the slot's bulk load
      const unsigned b = smem_u32(bar + s);
      const unsigned par = (phase >> s) & 1u;
      asm volatile(
          "{\n .reg .pred P;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n @!P bra WAIT_%=;\n}" ::"r"(b),
          "r"(par)
          : "memory");
      phase ^= 1u << s;
#pragma unroll
      for (int t = 0; t < SLOTS; ++t) qc[t] = slot[t * 32 + lane];
    } else if (MODE == 7) {
#pragma unroll
      for (int t = 0; t < SLOTS; ++t) qc[t] = qn[t];
      if (j + 1 < hi) {
        const int nv = vof(j + 1);
#pragma unroll
        for (int t = 0; t < SLOTS; ++t)
          qn[t] = __ldcg(reinterpret_cast<const float4*>(Q + (int64_t)nv * ROWB + (t * 32 + lane) * 16));
      }
    }
    if (MODE != 6) {  // the slot's previous reduction must have read it
      if (lane == 0) asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(DS - 1) : "memory");
      __syncwarp();
    }
#pragma unroll
    for (int t = 0; t < SLOTS; ++t) {
      float4 d = MODE == 5 ? make_float4(sc, sc, sc, sc)
                           : make_float4(qc[t].x * sc, qc[t].y * sc, qc[t].z * sc, qc[t].w * sc);
      slot[t * 32 + lane] = d;
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
    if (lane == 0) {
      asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.f32 [%0], [%1], %2;" ::"l"(
                       Q + (int64_t)cv * ROWB),
                   "r"(smem_u32(slot)), "r"(ROWB)
                   : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
    if (MODE == 6 && j + DS - 1 < hi) {
      // slot of rating j + DS - 1 = slot of rating j - 1: its reduction (the previous group) must have read it
      if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      issue_load(j + DS - 1);
    }
    acc += sc;
  }
  if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  if (acc == 1.2345f) sink[0] = acc;
}

template <int MODE, int SLOTS>
cudaError_t launch_probe(const int32_t* rv, const float* rr, int64_t nrec, char* Q, int rowb, int64_t warps,
                         float* sink, cudaStream_t st) {
  const int64_t pw = (nrec + warps - 1) / warps;
  const int64_t blocks = (warps * 32 + 255) / 256;
  (note_launch(), roundtrip_kernel<MODE, SLOTS><<<(unsigned)blocks, 256, 0, st>>>(rv, rr, nrec, Q, rowb, pw, sink));
  return cudaGetLastError();
}

}  // namespace

cudaError_t k_probe_roundtrip(int mode, const int32_t* ru, const int32_t* rv, const float* rr, int64_t nrec, int32_t k,
                              int64_t n, float* P, int64_t row0, const float* Qm, int64_t warps, int reps, float* ms,
                              cudaStream_t st) {
  *ms = 0.f;
  if (nrec <= 0 || warps <= 0) return cudaSuccess;
  // slots of 32 lanes: 16 B (fp32) or 8 B (binary16) each
  const int slots = k / 128;
  if (k % 128 != 0 || slots < 1 || slots > 4) return cudaErrorInvalidValue;
  const int rowb = mode == 1 ? k * 2 : k * 4;
  char* Q = nullptr;
  float* sink = nullptr;
  cudaError_t e = cudaMallocAsync((void**)&Q, (size_t)n * rowb, st);
  if (e != cudaSuccess) return e;
  e = cudaMallocAsync((void**)&sink, sizeof(float) * 2, st);
  if (e != cudaSuccess) return e;
  cudaMemsetAsync(Q, 0, (size_t)n * rowb, st);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int64_t pw = (nrec + warps - 1) / warps;
  const unsigned blocks = (unsigned)((warps * 32 + 255) / 256);
  auto once = [&]() -> cudaError_t {
#define PR(M, S) \
  if (mode == M && slots == S) return launch_probe<M, S>(rv, rr, nrec, Q, rowb, warps, sink, st);
    PR(0, 1) PR(0, 2) PR(0, 4) PR(1, 1) PR(1, 2) PR(1, 4) PR(2, 1) PR(2, 2) PR(2, 4)
#undef PR
#define PS(M, S)                                                                                             \
  if (mode == M && slots == S) {                                                                             \
    (note_launch(), stream_kernel<M, S><<<blocks, 256, 0, st>>>(ru, rv, nrec, reinterpret_cast<const char*>(Qm), \
                                                              reinterpret_cast<char*>(P), row0, k * 4, pw, sink)); \
    return cudaGetLastError();                                                                               \
  }
    PS(3, 1) PS(3, 2) PS(3, 4) PS(4, 1) PS(4, 2) PS(4, 4)
#undef PS
#define PB(MD, M, S, D)                                                                                     \
  if (mode == MD && slots == S) {                                                                         \
    const size_t smem = (size_t)8 * D * (S * 512) + 8 * 8 * D;                                            \
    cudaFuncSetAttribute(bulk_kernel<M, S, D>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);   \
    (note_launch(), bulk_kernel<M, S, D><<<blocks, 256, smem, st>>>(rv, rr, nrec, Q, pw, sink));           \
    return cudaGetLastError();                                                                            \
  }
    PB(5, 5, 1, 4) PB(6, 6, 1, 4) PB(7, 7, 1, 2) PB(8, 6, 1, 8) PB(9, 6, 1, 2)
#undef PB
    return cudaErrorInvalidValue;
  };
  e = once();  // warm-up
  if (e == cudaSuccess) {
    cudaEventRecord(a, st);
    for (int i = 0; i < reps && e == cudaSuccess; ++i) e = once();
    cudaEventRecord(b, st);
    cudaEventSynchronize(b);
    float t = 0.f;
    cudaEventElapsedTime(&t, a, b);
    *ms = t / (float)(reps > 0 ? reps : 1);
  }
  cudaEventDestroy(a);
  cudaEventDestroy(b);
  cudaFreeAsync(Q, st);
  cudaFreeAsync(sink, st);
  return e != cudaSuccess ? e : cudaGetLastError();
}

}  // namespace hccmf
