// eval.cu -- a0 factor init, a8 RMSE, a9 export (un-permute), Q replica average.
#include <cuda_fp16.h>

#include "internal.cuh"

namespace hccmf {
namespace {

constexpr int kT = 256;

inline unsigned grid_for(int64_t n, int64_t cap = 148LL * 64) {
  int64_t b = (n + kT - 1) / kT;
  if (b < 1) b = 1;
  if (b > cap) b = cap;
  return (unsigned)b;
}

// a0 (R5): X[perm[i]][j] = U(H(seed, tag, i, j)) * sqrtf(1/k), original id i
__global__ void init_kernel(uint64_t seed, uint64_t tag, int64_t rows_total, int32_t k, const int32_t* perm,
                            int64_t row0, int64_t rows, float* X) {
  const float sc = sqrtf(1.0f / (float)k);
  const int64_t total = rows_total * k;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = e / k;
    const int32_t j = (int32_t)(e - i * k);
    const int64_t pr = (int64_t)perm[i] - row0;
    if (pr < 0 || pr >= rows) continue;
    X[pr * k + j] = uniform24(hash4(seed, tag, (uint64_t)i, (uint64_t)j)) * sc;
  }
}

__global__ void scatter_kernel(const float4* src, int64_t rows_total, int32_t k4, const int32_t* perm, int64_t row0,
                               int64_t rows, float4* dst) {
  const int64_t total = rows_total * k4;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = e / k4;
    const int32_t j = (int32_t)(e - i * k4);
    const int64_t pr = (int64_t)perm[i] - row0;
    if (pr < 0 || pr >= rows) continue;
    dst[pr * k4 + j] = src[e];
  }
}

__global__ void gather_kernel(const float4* src, int64_t rows_total, int32_t k4, const int32_t* perm, int64_t row0,
                              float4* dst) {
  const int64_t total = rows_total * k4;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < total; e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = e / k4;
    const int32_t j = (int32_t)(e - i * k4);
    dst[e] = src[((int64_t)perm[i] - row0) * k4 + j];
  }
}

// a8: one rating group of L lanes per test rating (same lane mapping as the SGD
// kernel), fp32 dot product, squared error accumulated in fp64 per group in a
// fixed order, then a fixed-order tree per CTA -> partials[blockIdx].
// Each group walks a contiguous chunk of the test set in windows of L ratings: lane sl
// resolves rating w+sl's permuted ids (tu -> perm_row, tv -> perm_col: two dependent
// loads, once per window for L ratings at a time), and the p_u / q_v rows of rating
// j+1 are requested before rating j is reduced.
template <int L, int S>  // S: float4 slots per lane, ceil(k / 4L) rounded up to 1, 2, 4
__global__ void __launch_bounds__(kT) rmse_kernel(const int32_t* __restrict__ tu, const int32_t* __restrict__ tv,
                                                  const float* __restrict__ tr, int64_t nt,
                                                  const int32_t* __restrict__ perm_row,
                                                  const int32_t* __restrict__ perm_col, const float* __restrict__ P,
                                                  int64_t row0, int64_t rows, const float* __restrict__ Q, int32_t k,
                                                  double* partials) {
  constexpr unsigned FM = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const int sl = lane & (L - 1);
  const int64_t group = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) / L;
  const int64_t ngroups = (int64_t)gridDim.x * blockDim.x / L;
  const int64_t chunk = (nt + ngroups - 1) / ngroups;
  const int64_t lo = group * chunk < nt ? group * chunk : nt;
  const int64_t hi = lo + chunk < nt ? lo + chunk : nt;
  double acc = 0.0, cnt = 0.0;
  auto load = [&](int64_t up, int64_t vp, bool act, float4 (&p)[S], float4 (&q)[S]) {
#pragma unroll
    for (int s = 0; s < S; ++s) {
      const int c = (s * L + sl) * 4;
      if (act && c < k) {
        p[s] = __ldcs(reinterpret_cast<const float4*>(P + up * k + c));
        q[s] = __ldg(reinterpret_cast<const float4*>(Q + vp * k + c));
      } else {
        p[s] = q[s] = make_float4(0.f, 0.f, 0.f, 0.f);
      }
    }
  };
  // every group of a warp runs the same number of windows and steps (the shuffles are
  // warp-wide): ceil(chunk / L) windows of L steps, masked past the group's own end
  const int64_t nwin = (chunk + L - 1) / L;
  for (int64_t wi = 0; wi < nwin; ++wi) {
    const int64_t w = lo + wi * L;
    const int64_t idx = w + sl;
    int64_t ul = -1, vl = 0;
    float rl = 0.f;
    if (idx < hi) {
      ul = (int64_t)perm_row[tu[idx]] - row0;
      vl = perm_col[tv[idx]];
      rl = tr[idx];
    }
    const int nw = (int)(hi - w <= 0 ? 0 : (hi - w < L ? hi - w : L));
    float4 pa[S], qa[S], pb[S], qb[S];
    const int64_t up = __shfl_sync(FM, ul, 0, L), vp = __shfl_sync(FM, vl, 0, L);
    float r = __shfl_sync(FM, rl, 0, L);
    bool act = nw > 0 && up >= 0 && up < rows;
    load(up, vp, act, pa, qa);
    auto step = [&](int j, float4 (&pc)[S], float4 (&qc)[S], float4 (&pn)[S], float4 (&qn)[S]) {
      // rating j+1's rows in flight while rating j is reduced
      const int64_t un = __shfl_sync(FM, ul, (j + 1) & (L - 1), L), vn = __shfl_sync(FM, vl, (j + 1) & (L - 1), L);
      const float rn = __shfl_sync(FM, rl, (j + 1) & (L - 1), L);
      const bool actn = j + 1 < nw && un >= 0 && un < rows;
      load(un, vn, actn, pn, qn);
      float d = 0.f;
#pragma unroll
      for (int s = 0; s < S; ++s) {
        d = fmaf(pc[s].x, qc[s].x, d);
        d = fmaf(pc[s].y, qc[s].y, d);
        d = fmaf(pc[s].z, qc[s].z, d);
        d = fmaf(pc[s].w, qc[s].w, d);
      }
#pragma unroll
      for (int o = L / 2; o > 0; o >>= 1) d += __shfl_xor_sync(FM, d, o, L);
      if (act && sl == 0) {
        const double e = (double)r - (double)d;
        acc += e * e;
        cnt += 1.0;
      }
      act = actn;
      r = rn;
    };
    if (L == 1) {
      step(0, pa, qa, pb, qb);
    } else {
#pragma unroll 1
      for (int j = 0; j < L; j += 2) {
        step(j, pa, qa, pb, qb);
        step(j + 1, pb, qb, pa, qa);
      }
    }
  }
  __shared__ double sa[kT], sc[kT];
  sa[threadIdx.x] = acc;
  sc[threadIdx.x] = cnt;
  __syncthreads();
  for (int s = kT / 2; s > 0; s >>= 1) {
    if (threadIdx.x < s) {
      sa[threadIdx.x] += sa[threadIdx.x + s];
      sc[threadIdx.x] += sc[threadIdx.x + s];
    }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    partials[2 * blockIdx.x] = sa[0];
    partials[2 * blockIdx.x + 1] = sc[0];
  }
}

__global__ void rmse_final_kernel(const double* partials, int nb, double* out2) {
  if (threadIdx.x == 0 && blockIdx.x == 0) {
    double s = 0.0, c = 0.0;
    for (int b = 0; b < nb; ++b) {
      s += partials[2 * b];
      c += partials[2 * b + 1];
    }
    out2[0] = s;
    out2[1] = c;
  }
}

__global__ void average_kernel(const float* reps, int32_t G, int64_t count, float* out) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < count; e += (int64_t)gridDim.x * blockDim.x) {
    double s = 0.0;
    for (int g = 0; g < G; ++g) s += (double)reps[(int64_t)g * count + e];
    out[e] = (float)(s / (double)G);
  }
}

// Strategy 2 (L1234-L1249): Q on the wire as IEEE binary16 (round to nearest even).
__global__ void round_half_kernel(float* x, int64_t count) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < count; e += (int64_t)gridDim.x * blockDim.x)
    x[e] = __half2float(__float2half_rn(x[e]));
}
__global__ void pack_half_kernel(const float* x, __half* y, int64_t count) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < count; e += (int64_t)gridDim.x * blockDim.x)
    y[e] = __float2half_rn(x[e]);
}
__global__ void unpack_half_kernel(const __half* y, float* x, int64_t count) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < count; e += (int64_t)gridDim.x * blockDim.x)
    x[e] = __half2float(y[e]);
}
// replicas rounded to binary16, mean in fp64, mean rounded to binary16 (one rounding)
__global__ void average_half_kernel(const float* reps, int32_t G, int64_t count, float* out) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < count; e += (int64_t)gridDim.x * blockDim.x) {
    double s = 0.0;
    for (int g = 0; g < G; ++g) s += (double)__half2float(__float2half_rn(reps[(int64_t)g * count + e]));
    out[e] = __half2float(__double2half(s / (double)G));
  }
}

// Strategy 2 all-reduce on the wire (R25): W binary16 copies of one chunk, `stride`
// halves apart, summed in fp64 in rank order; the mean is rounded once to binary16 --
// the same function as average_half_kernel on the logical backend
__global__ void mean_gathered_half_kernel(const __half* g, int32_t W, int64_t stride, int64_t count, __half* out) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < count; e += (int64_t)gridDim.x * blockDim.x) {
    double s = 0.0;
    for (int r = 0; r < W; ++r) s += (double)__half2float(g[(int64_t)r * stride + e]);
    out[e] = __double2half(s / (double)W);
  }
}

}  // namespace

cudaError_t k_round_half(float* x, int64_t count, cudaStream_t st) {
  if (count <= 0) return cudaSuccess;
  (note_launch(), round_half_kernel<<<grid_for(count), kT, 0, st>>>(x, count));
  return cudaGetLastError();
}
cudaError_t k_pack_half(const float* x, void* y, int64_t count, cudaStream_t st) {
  if (count <= 0) return cudaSuccess;
  (note_launch(), pack_half_kernel<<<grid_for(count), kT, 0, st>>>(x, reinterpret_cast<__half*>(y), count));
  return cudaGetLastError();
}
cudaError_t k_unpack_half(const void* y, float* x, int64_t count, cudaStream_t st) {
  if (count <= 0) return cudaSuccess;
  (note_launch(), unpack_half_kernel<<<grid_for(count), kT, 0, st>>>(reinterpret_cast<const __half*>(y), x, count));
  return cudaGetLastError();
}
cudaError_t k_average_half(const float* reps, int32_t G, int64_t count, float* out, cudaStream_t st) {
  (note_launch(), average_half_kernel<<<grid_for(count), kT, 0, st>>>(reps, G, count, out));
  return cudaGetLastError();
}

cudaError_t k_mean_gathered_half(const void* g, int32_t W, int64_t stride, int64_t count, void* out, cudaStream_t st) {
  if (count <= 0) return cudaSuccess;
  (note_launch(), mean_gathered_half_kernel<<<grid_for(count), kT, 0, st>>>(reinterpret_cast<const __half*>(g), W, stride,
                                                                            count, reinterpret_cast<__half*>(out)));
  return cudaGetLastError();
}

namespace {
__global__ void sum_sq_kernel(const float* __restrict__ r, int64_t n, double* out) {
  double s = 0.0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    s += (double)r[i] * (double)r[i];
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) atomicAdd(out, s);
}
}  // namespace

cudaError_t k_sum_sq(const float* r, int64_t n, double* out, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(out, 0, sizeof(double), st);
  if (e != cudaSuccess || n <= 0) return e;
  (note_launch(), sum_sq_kernel<<<grid_for(n), kT, 0, st>>>(r, n, out));
  return cudaGetLastError();
}

cudaError_t k_init_factors(uint64_t seed, uint64_t tag, int64_t rows_total, int32_t k, const int32_t* perm,
                           int64_t row0, int64_t rows, float* X, cudaStream_t st) {
  if (rows_total == 0) return cudaSuccess;
  (note_launch(), init_kernel<<<grid_for(rows_total * k), kT, 0, st>>>(seed, tag, rows_total, k, perm, row0, rows, X));
  return cudaGetLastError();
}

cudaError_t k_scatter_rows(const float* src, int64_t rows_total, int32_t k, const int32_t* perm, int64_t row0,
                           int64_t rows, float* dst, cudaStream_t st) {
  const int32_t k4 = k / 4;
  (note_launch(), scatter_kernel<<<grid_for(rows_total * k4), kT, 0, st>>>(reinterpret_cast<const float4*>(src), rows_total, k4,
                                                           perm, row0, rows, reinterpret_cast<float4*>(dst)));
  return cudaGetLastError();
}

cudaError_t k_gather_rows(const float* src, int64_t rows_total, int32_t k, const int32_t* perm, int64_t row0,
                          float* dst, cudaStream_t st) {
  const int32_t k4 = k / 4;
  (note_launch(), gather_kernel<<<grid_for(rows_total * k4), kT, 0, st>>>(reinterpret_cast<const float4*>(src), rows_total, k4, perm,
                                                          row0, reinterpret_cast<float4*>(dst)));
  return cudaGetLastError();
}

cudaError_t k_rmse(const int32_t* tu, const int32_t* tv, const float* tr, int64_t nt, const int32_t* perm_row,
                   const int32_t* perm_col, const float* P, int64_t row0, int64_t rows, const float* Q, int32_t k,
                   double* partials, double* out2, cudaStream_t st) {
  const int L = lanes_per_rating(k);
  int S = (k / 4 + L - 1) / L;
  if (S == 3) S = 4;
#define RM(LL, SS)                                                                                              \
  if (L == LL && S == SS) {                                                                                     \
    (note_launch(), rmse_kernel<LL, SS><<<RMSE_BLOCKS, kT, 0, st>>>(tu, tv, tr, nt, perm_row, perm_col, P, row0, \
                                                                   rows, Q, k, partials));                      \
  } else
  RM(1, 1) RM(2, 1) RM(4, 1) RM(8, 1) RM(16, 1) RM(32, 1) RM(32, 2) RM(32, 4)
#undef RM
  return cudaErrorInvalidValue;
  (note_launch(), rmse_final_kernel<<<1, 32, 0, st>>>(partials, RMSE_BLOCKS, out2));
  return cudaGetLastError();
}

cudaError_t k_average(const float* reps, int32_t G, int64_t count, float* out, cudaStream_t st) {
  (note_launch(), average_kernel<<<grid_for(count), kT, 0, st>>>(reps, G, count, out));
  return cudaGetLastError();
}

}  // namespace hccmf
