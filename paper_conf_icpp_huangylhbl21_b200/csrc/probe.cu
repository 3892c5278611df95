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
