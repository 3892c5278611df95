// detchain.cu -- the deterministic epoch (a5) as a chain-parallel wavefront.
//
// The DET order (R19: strata of blocks (i, (i+t) mod B), each block in its sorted order,
// L1472-L1474) fixes, for every P row and every Q row, the sequence of updates that touch
// it; any execution that keeps those per-row sequences computes exactly the same numbers
// (each update reads only p_u and q_v).  Inside a block the ratings of one item form a
// chain through q_v, and only consecutive ratings of one user (a user's run is contiguous
// in the sorted block) couple two chains through p_u.  The slab wavefront walks a block's
// ratings one after another; its epoch is the hottest column block's whole serial chain
// (profiles/r01_det_wavefront.md).  Here the warp splits into NG lane groups of L = 32/NG
// lanes, each walking the chains of the items assigned to it (LPT on chain length, per
// segment) in the block's sorted order, with its item's q_v in registers; a rating whose
// user's previous rating sits in another group waits for that group's progress counter.
// Each group's sequence is a subsequence of the sorted order and every dependency points
// back in that order, so the earliest unfinished rating is always ready (no deadlock).
//
// A block is cut into segments of <= SU distinct users (whole user runs); a segment's p_u
// rows sit in shared memory while it runs (copied in with cp.async, the next segment's
// while this one runs; the first segment's while the warp waits for its predecessor) and
// are written back when it ends.  The column block's q rows are staged as in the slab
// wavefront.  Across blocks the hand-off is the slab wavefront's: warp i waits for warp
// i+1's progress flag (cooperative launch: every warp co-resident).
//
// The schedule (records reordered group by group inside each segment, with packed
// dependency words) is built once per partition on the device (k_det_chain_schedule).
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include <cub/cub.cuh>

#include "internal.cuh"

namespace hccmf {
namespace {

constexpr int kCT = 256;
constexpr int kChainWmax = 64;  // items per column block the schedule builder handles
constexpr int kChainRC = 96;    // records per segment (staged in shared memory with its p rows)
#ifndef HCCMF_CHAIN_NW
#define HCCMF_CHAIN_NW 4  // warps (chain groups) per row block: 1, 2 or 4
#endif
constexpr int kNW = HCCMF_CHAIN_NW;
constexpr unsigned kFM = 0xffffffffu;

inline unsigned grid_for(int64_t n, int64_t cap = 148LL * 64) {
  int64_t b = (n + kCT - 1) / kCT;
  if (b < 1) b = 1;
  if (b > cap) b = cap;
  return (unsigned)b;
}

__device__ __forceinline__ int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// meta word of a reordered record: [0,5) p slot (the user's run index in the segment),
// bit 5 has-dependency, [6,8) dependency group, [8,24) dependency index in that group
__device__ __forceinline__ uint32_t pack_meta(int pslot, bool dep, int dg, int di) {
  return (uint32_t)pslot | (dep ? (1u << 5) : 0u) | ((uint32_t)dg << 6) | ((uint32_t)di << 8);
}

// pass 1: runs and segments per block
__global__ void chain_count_kernel(const int32_t* __restrict__ ru, const int64_t* __restrict__ off, int64_t nblk,
                                   int SU, int64_t* nseg, int64_t* nrun) {
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < nblk; b += (int64_t)gridDim.x * blockDim.x) {
    const int64_t lo = off[b], hi = off[b + 1];
    int64_t segs = 0, runs = 0;
    int su = 0;
    int64_t srec = 0;
    for (int64_t j = lo; j < hi;) {
      int64_t e = j + 1;
      while (e < hi && ru[e] == ru[j]) ++e;
      const int64_t len = e - j;
      if (su == 0 || su == SU || srec + len > kChainRC) {
        ++segs;
        su = 0;
        srec = 0;
      }
      ++su;
      srec += len;
      ++runs;
      j = e;
    }
    nseg[b] = segs;
    nrun[b] = runs;
  }
}

// pass 2: reorder each segment group by group (LPT over item chains), dependency words
__global__ void chain_build_kernel(const int32_t* __restrict__ ru, const int32_t* __restrict__ rv,
                                   const float* __restrict__ rr, const int64_t* __restrict__ off, int64_t nblk, int Bc,
                                   int64_t n, int NG, int SU, const int64_t* __restrict__ seg_base,
                                   const int64_t* __restrict__ run_base, int32_t* cv, float* cr, uint32_t* meta,
                                   int64_t* seg_lo, int64_t* seg_run, uint16_t* seg_gend, int32_t* run_user,
                                   int* bad) {
  for (int64_t b = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; b < nblk; b += (int64_t)gridDim.x * blockDim.x) {
    const int64_t lo = off[b], hi = off[b + 1];
    const int64_t cb = b % Bc;
    const int64_t c0 = cdiv(cb * n, Bc), w = cdiv((cb + 1) * n, Bc) - c0;
    if (w > kChainWmax) {
      atomicOr(bad, 1);
      continue;
    }
    int64_t sidx = seg_base[b], ridx = run_base[b];
    int64_t j = lo;
    while (j < hi) {
      // segment [j, se): whole user runs, <= SU users, <= 65535 records
      int64_t se = j;
      int su = 0;
      while (se < hi) {
        int64_t e = se + 1;
        while (e < hi && ru[e] == ru[se]) ++e;
        if (e - se > kChainRC) {  // one user run longer than a segment's record buffer
          atomicOr(bad, 2);
          break;
        }
        if (su == SU || e - j > kChainRC) break;
        run_user[ridx + su] = ru[se];
        ++su;
        se = e;
      }
      if (se == j) {  // (flagged above) never loop: take the run so the pass terminates
        int64_t e = se + 1;
        while (e < hi && ru[e] == ru[se]) ++e;
        run_user[ridx + su] = ru[se];
        ++su;
        se = e;
      }
      seg_lo[sidx] = j;
      seg_run[sidx] = ridx;
      // chain lengths and LPT assignment of items to groups
      int cnt[kChainWmax];
      unsigned char grp[kChainWmax];
      for (int x = 0; x < w; ++x) cnt[x] = 0;
      for (int64_t q = j; q < se; ++q) ++cnt[rv[q] - c0];
      int load[4] = {0, 0, 0, 0};
      unsigned char done[kChainWmax];
      for (int x = 0; x < w; ++x) done[x] = 0;
      for (int it = 0; it < w; ++it) {
        int best = -1;
        for (int x = 0; x < w; ++x)
          if (!done[x] && (best < 0 || cnt[x] > cnt[best])) best = x;
        done[best] = 1;
        int gmin = 0;
        for (int gg = 1; gg < NG; ++gg)
          if (load[gg] < load[gmin]) gmin = gg;
        grp[best] = (unsigned char)gmin;
        load[gmin] += cnt[best];
      }
      int gstart[4], pos[4] = {0, 0, 0, 0};
      int acc = 0;
      for (int gg = 0; gg < 4; ++gg) {
        gstart[gg] = acc;
        if (gg < NG) acc += load[gg];
        seg_gend[sidx * 4 + gg] = (uint16_t)acc;
      }
      // records in sorted order -> their group's next slot
      int pslot = -1, prev_g = 0, prev_i = 0;
      int32_t prev_u = -1;
      for (int64_t q = j; q < se; ++q) {
        const int32_t u = ru[q];
        const bool same = u == prev_u;
        if (!same) ++pslot;
        const int gi = grp[rv[q] - c0];
        const int ii = pos[gi]++;
        const int64_t dst = j + gstart[gi] + ii;
        cv[dst] = rv[q];
        cr[dst] = rr[q];
        meta[dst] = pack_meta(pslot, same, prev_g, prev_i);
        prev_u = u;
        prev_g = gi;
        prev_i = ii;
      }
      ridx += su;
      ++sidx;
      j = se;
    }
  }
}

struct ChainArgs {
  float* P;
  float* Q;
  int64_t row0, n;
  int32_t k;
  float gamma, lambda;
  const int32_t* __restrict__ cv;
  const float* __restrict__ cr;
  const uint32_t* __restrict__ meta;
  const int64_t* __restrict__ blk_seg;
  const int64_t* __restrict__ seg_lo;
  const int64_t* __restrict__ seg_run;
  const uint16_t* __restrict__ seg_gend;
  const int32_t* __restrict__ run_user;
};

// float4 helpers (packed fp32x2 pipe, as in sgd.cu)
__device__ __forceinline__ float2 lo2(float4 a) { return make_float2(a.x, a.y); }
__device__ __forceinline__ float2 hi2(float4 a) { return make_float2(a.z, a.w); }
__device__ __forceinline__ float4 cat2(float2 l, float2 h) { return make_float4(l.x, l.y, h.x, h.y); }
__device__ __forceinline__ float4 f4_fma(float s, float4 a, float4 b) {
  const float2 ss = make_float2(s, s);
  return cat2(__ffma2_rn(ss, lo2(a), lo2(b)), __ffma2_rn(ss, hi2(a), hi2(b)));
}
__device__ __forceinline__ float4 f4_scale(float s, float4 a) {
  const float2 ss = make_float2(s, s);
  return cat2(__fmul2_rn(ss, lo2(a)), __fmul2_rn(ss, hi2(a)));
}
__device__ __forceinline__ float2 f4_dot2(float4 a, float4 b, float2 acc) {
  return __ffma2_rn(hi2(a), hi2(b), __ffma2_rn(lo2(a), lo2(b), acc));
}
__device__ __forceinline__ void cp16(float4* dst, const float4* src) {
  const unsigned d = (unsigned)__cvta_generic_to_shared(dst);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src) : "memory");
}

#ifdef HCCMF_DIAG_TRACE  // diagnostic builds only: per (warp, stratum) %globaltimer stamps + steps
__device__ unsigned g_chain_trace[2048 * 2048 * 4];
__device__ __forceinline__ unsigned ctimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return (unsigned)t;
}
#endif

// One CTA = one row block, NW warps = NW chain groups (all 32 lanes of a warp on one
// rating: VEC float4 of p_u / q_v per lane, k = 128 VEC).  Each warp walks its group's
// records of the segment in the block's sorted order with its item's q_v in registers;
// a record whose user's previous rating belongs to another warp waits for that warp's
// progress counter in shared memory (release / acquire at CTA scope).  The warps' chains
// overlap in the SM's schedulers (a chain step is a dependent instruction chain: the
// dot product's five shuffle levels dominate it).  Shared memory per CTA: the column
// block's q slab (wmax rows), then two segment buffers (SU p rows + kChainRC records each),
// then NW progress counters.  Segments are staged by cp.async one segment ahead (the
// block's first segment while thread 0 waits for the predecessor row block).
template <int NW, int VEC>
__global__ void __launch_bounds__(NW * 32) sgd_wave_chain_kernel(ChainArgs a, int B, int* progress, int wmax, int SU) {
  constexpr int k4 = 32 * VEC;
  constexpr int NT = NW * 32;
  extern __shared__ float4 chain_smem[];
  const int i = blockIdx.x;  // row block
  if (i >= B) return;
  const int tid = threadIdx.x, w = tid >> 5, lane = tid & 31;
  const int bufsz = SU * k4 + (3 * kChainRC) / 4;  // float4 units
  float4* qslab = chain_smem;
  float4* buf0 = qslab + (int64_t)wmax * k4;
  float4* buf1 = buf0 + bufsz;
  int* prog = reinterpret_cast<int*>(buf1 + bufsz);
  const float gam = a.gamma, c1 = 1.f - a.gamma * a.lambda;
  float4* Pg = reinterpret_cast<float4*>(a.P) - a.row0 * k4;
  float4* Qg = reinterpret_cast<float4*>(a.Q);
  const int nb = (i + 1) % B;

  // segment s -> buffer: p rows (16-byte pieces) and records (4-byte copies), spread over
  // the CTA's threads; each thread commits its own copies
  auto issue_seg = [&](int64_t s, float4* buf) {
    const int64_t r0 = a.seg_run[s];
    const int nu = (int)(a.seg_run[s + 1] - r0);
    for (int x = tid; x < nu * k4; x += NT) {
      const int r = x / k4, y = x - r * k4;
      cp16(buf + x, Pg + (int64_t)a.run_user[r0 + r] * k4 + y);
    }
    const int64_t lo = a.seg_lo[s];
    const int nr = (int)(a.seg_lo[s + 1] - lo);
    uint32_t* rec = reinterpret_cast<uint32_t*>(buf + SU * k4);
    for (int x = tid; x < nr; x += NT) {
      const unsigned d0 = (unsigned)__cvta_generic_to_shared(rec + x);
      asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(d0), "l"(a.cv + lo + x) : "memory");
      asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(d0 + 4 * kChainRC), "l"(a.cr + lo + x) : "memory");
      asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(d0 + 8 * kChainRC), "l"(a.meta + lo + x) : "memory");
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };

  for (int t = 0; t < B; ++t) {
    const int c = (i + t) % B;
    const int64_t b = (int64_t)i * B + c;
    const int64_t s0 = a.blk_seg[b], s1 = a.blk_seg[b + 1];
    if (s1 > s0) issue_seg(s0, buf0);  // P rows are this CTA's own: no wait needed
#ifdef HCCMF_DIAG_TRACE
    unsigned steps = 0, polls = 0, segs = (unsigned)(s1 - s0);
    if (tid == 0 && B <= 2048) g_chain_trace[((int64_t)i * B + t) * 4] = ctimer();
#endif
    if (t > 0 && B > 1) {
      if (tid == 0) {
        int seen;
        do {
          asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(seen) : "l"(progress + (int64_t)nb * kProgressStride) : "memory");
          if (seen < t) __nanosleep(64);
        } while (seen < t);
        // acquire pattern (relaxed read + fence.acquire: CCTL.IVALL, no MEMBAR -- a full
        // fence here would also wait for this warp's own outstanding copies and prefetches)
        asm volatile("fence.acquire.gpu;" ::: "memory");
      }
      __syncthreads();
    }
#ifdef HCCMF_DIAG_TRACE
    if (tid == 0 && B <= 2048) g_chain_trace[((int64_t)i * B + t) * 4 + 1] = ctimer();
#endif
    if (s1 > s0) {
      const int qc0 = (int)(((int64_t)c * a.n + B - 1) / B);
      const int qc1 = (int)(((int64_t)(c + 1) * a.n + B - 1) / B);
      for (int x = tid; x < (qc1 - qc0) * k4; x += NT) cp16(qslab + x, Qg + (int64_t)qc0 * k4 + x);
      asm volatile("cp.async.commit_group;" ::: "memory");
      const float4* const qsr = qslab - (int64_t)qc0 * k4 + lane;  // row v: qsr[v * k4 + 32 x]
      float4* const qsw = qslab - (int64_t)qc0 * k4 + lane;
      for (int64_t s = s0; s < s1; ++s) {
        float4* buf = ((s - s0) & 1) ? buf1 : buf0;
        if (s + 1 < s1) {
          issue_seg(s + 1, ((s - s0) & 1) ? buf0 : buf1);
          asm volatile("cp.async.wait_group 1;" ::: "memory");
        } else {
          asm volatile("cp.async.wait_group 0;" ::: "memory");
        }
        if (tid < NW) prog[tid] = 0;
        __syncthreads();
        // ---- the segment: warp w walks its group's records [gs, ge) of the staged buffer
        const int gs = w ? a.seg_gend[s * 4 + w - 1] : 0, ge = a.seg_gend[s * 4 + w];
        const int32_t* rv = reinterpret_cast<const int32_t*>(buf + SU * k4);
        const float* rr = reinterpret_cast<const float*>(rv + kChainRC);
        const uint32_t* rm = reinterpret_cast<const uint32_t*>(rv + 2 * kChainRC);
        float4* const pb = buf + lane;
        int cur_v = -1;
        float4 q[VEC];
        for (int j = gs; j < ge; ++j) {
          const uint32_t m = rm[j];
          const int v = rv[j];
          const float r = rr[j];
          if ((m >> 5) & 1u) {  // the user's previous rating: in another warp's group?
            const int dg = (int)((m >> 6) & 3u), di = (int)(m >> 8);
            if (dg != w) {
              if (lane == 0) {
                int seen;
                do {
                  asm volatile("ld.acquire.cta.shared.s32 %0, [%1];" : "=r"(seen)
                               : "r"((unsigned)__cvta_generic_to_shared(prog + dg)) : "memory");
#ifdef HCCMF_DIAG_TRACE
                  polls += seen <= di;
#endif
                } while (seen <= di);
              }
              __syncwarp();
            }
          }
          if (v != cur_v) {  // chain switch (warp-uniform): park the old q_v, take the new
            if (cur_v >= 0) {
#pragma unroll
              for (int x = 0; x < VEC; ++x) qsw[(int64_t)cur_v * k4 + 32 * x] = q[x];
            }
#pragma unroll
            for (int x = 0; x < VEC; ++x) q[x] = qsr[(int64_t)v * k4 + 32 * x];
            cur_v = v;
          }
          const int ps = (int)(m & 31u);
          float4 p[VEC];
#pragma unroll
          for (int x = 0; x < VEC; ++x) p[x] = pb[ps * k4 + 32 * x];
          float2 dd = make_float2(0.f, 0.f);
#pragma unroll
          for (int x = 0; x < VEC; ++x) dd = f4_dot2(p[x], q[x], dd);
          float d = dd.x + dd.y;
#pragma unroll
          for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(kFM, d, o);
          const float gev = gam * (r - d);
          // p' = (1 - g l) p + g e q ; q' = (1 - g l) q + g e p   (old p, R1)
#pragma unroll
          for (int x = 0; x < VEC; ++x) {
            pb[ps * k4 + 32 * x] = f4_fma(gev, q[x], f4_scale(c1, p[x]));
            q[x] = f4_fma(gev, p[x], f4_scale(c1, q[x]));
          }
          __syncwarp();
          if (lane == 0)
            asm volatile("st.release.cta.shared.s32 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(prog + w)),
                         "r"(j - gs + 1) : "memory");
#ifdef HCCMF_DIAG_TRACE
          ++steps;
#endif
        }
        if (cur_v >= 0) {
#pragma unroll
          for (int x = 0; x < VEC; ++x) qsw[(int64_t)cur_v * k4 + 32 * x] = q[x];
        }
        __syncthreads();
        const int64_t r0 = a.seg_run[s];
        const int nu = (int)(a.seg_run[s + 1] - r0);
        for (int x = tid; x < nu * k4; x += NT) {
          const int rr_ = x / k4, y = x - rr_ * k4;
          __stcg(Pg + (int64_t)a.run_user[r0 + rr_] * k4 + y, buf[x]);
        }
      }
      __syncthreads();
      for (int x = tid; x < (qc1 - qc0) * k4; x += NT) __stcg(Qg + (int64_t)qc0 * k4 + x, qslab[x]);
    }
    __syncthreads();
    if (tid == 0) {
      asm volatile("fence.acq_rel.gpu;" ::: "memory");
      asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(progress + (int64_t)i * kProgressStride), "r"(t + 1) : "memory");
#ifdef HCCMF_DIAG_TRACE
      if (B <= 2048) {
        g_chain_trace[((int64_t)i * B + t) * 4 + 2] = ctimer();
        g_chain_trace[((int64_t)i * B + t) * 4 + 3] = (steps & 0xFFFu) | (min(polls, 0xFFFFu) << 12) | (min(segs, 15u) << 28);
      }
#endif
    }
  }
}

template <int NW, int VEC>
bool chain_geometry_t(int B, int wmax, int k, int* su_out, size_t* smem_out, bool launchable) {
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // every one of the B CTAs resident at once: c CTAs per SM share its shared memory
  const int c = (B + sms - 1) / sms;
  if (c * NW > 64) return false;
  const int64_t per_cta = (int64_t)std::min<size_t>(227 * 1024, 228 * 1024 / c) - 2048;  // static + reserve
  const int64_t row = (int64_t)k * sizeof(float), recb = 12 * (int64_t)kChainRC;
  const int64_t su = (per_cta - wmax * row - 2 * recb - 64) / (2 * row);
  if (su < 4) return false;
  const int SU = (int)std::min<int64_t>(su, 32);
  const size_t smem = (size_t)((wmax + 2 * SU) * row + 2 * recb + 64);
  if (launchable) {
    if (cudaFuncSetAttribute(sgd_wave_chain_kernel<NW, VEC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
        cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, sgd_wave_chain_kernel<NW, VEC>, NW * 32, smem) !=
        cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    if ((int64_t)B > (int64_t)sms * per_sm) return false;
  }
  *su_out = SU;
  *smem_out = smem;
  return true;
}

}  // namespace

// NW = 4 warps per row block (4 chain groups); VEC float4 per lane (k = 128 VEC)
static bool chain_shape(int k, int* NG, int* V) {
  if (k == 128) { *NG = kNW; *V = 1; return true; }
  if (k == 256) { *NG = kNW; *V = 2; return true; }
  return false;
}

bool det_chain_plan(int k, int B, int64_t n, int* NG, int* SU) {
  int ng, v;
  size_t smem;
  if (!chain_shape(k, &ng, &v)) return false;
  const int wmax = (int)((n + B - 1) / B);
  if (wmax > kChainWmax) return false;
  const bool ok = v == 1 ? chain_geometry_t<kNW, 1>(B, wmax, k, SU, &smem, true)
                         : chain_geometry_t<kNW, 2>(B, wmax, k, SU, &smem, true);
  *NG = ng;
  return ok;
}

cudaError_t k_det_chain_schedule(const int32_t* ru, const int32_t* rv, const float* rr, const int64_t* off,
                                 int64_t nblk, int Bc, int64_t n, int NG, int SU, DetChain* out, cudaStream_t st) {
  int64_t *cs = nullptr, *cr = nullptr, *bs = nullptr, *br = nullptr;
  int* bad = nullptr;
  cudaError_t e;
#define CK(x)                        \
  do {                               \
    e = (x);                         \
    if (e != cudaSuccess) return e;  \
  } while (0)
  CK(cudaMallocAsync((void**)&cs, sizeof(int64_t) * (nblk + 1), st));
  CK(cudaMallocAsync((void**)&cr, sizeof(int64_t) * (nblk + 1), st));
  CK(cudaMallocAsync((void**)&bs, sizeof(int64_t) * (nblk + 1), st));
  CK(cudaMallocAsync((void**)&br, sizeof(int64_t) * (nblk + 1), st));
  CK(cudaMallocAsync((void**)&bad, sizeof(int), st));
  CK(cudaMemsetAsync(cs, 0, sizeof(int64_t) * (nblk + 1), st));
  CK(cudaMemsetAsync(cr, 0, sizeof(int64_t) * (nblk + 1), st));
  CK(cudaMemsetAsync(bad, 0, sizeof(int), st));
  (note_launch(), chain_count_kernel<<<grid_for(nblk), kCT, 0, st>>>(ru, off, nblk, SU, cs, cr));
  CK(cudaGetLastError());
  size_t tb = 0;
  void* tmp = nullptr;
  CK(cub::DeviceScan::ExclusiveSum(nullptr, tb, cs, bs, nblk + 1, st));
  CK(cudaMallocAsync(&tmp, tb, st));
  CK(cub::DeviceScan::ExclusiveSum(tmp, tb, cs, bs, nblk + 1, st));
  CK(cub::DeviceScan::ExclusiveSum(tmp, tb, cr, br, nblk + 1, st));
  cudaFreeAsync(tmp, st);
  int64_t tot[2] = {0, 0};
  CK(cudaMemcpyAsync(&tot[0], bs + nblk, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
  CK(cudaMemcpyAsync(&tot[1], br + nblk, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
  int64_t nrec = 0;
  CK(cudaMemcpyAsync(&nrec, off + nblk, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  DetChain d{};
  d.nseg = tot[0];
  d.nrun = tot[1];
  d.nrec = nrec;
  d.NG = NG;
  d.SU = SU;
  CK(cudaMallocAsync((void**)&d.cv, sizeof(int32_t) * (nrec ? nrec : 1), st));
  CK(cudaMallocAsync((void**)&d.cr, sizeof(float) * (nrec ? nrec : 1), st));
  CK(cudaMallocAsync((void**)&d.meta, sizeof(uint32_t) * (nrec ? nrec : 1), st));
  CK(cudaMallocAsync((void**)&d.seg_lo, sizeof(int64_t) * (d.nseg + 1), st));
  CK(cudaMallocAsync((void**)&d.seg_run, sizeof(int64_t) * (d.nseg + 1), st));
  CK(cudaMallocAsync((void**)&d.seg_gend, sizeof(uint16_t) * 4 * (d.nseg ? d.nseg : 1), st));
  CK(cudaMallocAsync((void**)&d.run_user, sizeof(int32_t) * (d.nrun ? d.nrun : 1), st));
  d.blk_seg = bs;
  // sentinels: seg_lo[nseg] = nrec, seg_run[nseg] = nrun
  CK(cudaMemcpyAsync(d.seg_lo + d.nseg, &d.nrec, sizeof(int64_t), cudaMemcpyHostToDevice, st));
  CK(cudaMemcpyAsync(d.seg_run + d.nseg, &d.nrun, sizeof(int64_t), cudaMemcpyHostToDevice, st));
  (note_launch(), chain_build_kernel<<<grid_for(nblk), kCT, 0, st>>>(ru, rv, rr, off, nblk, Bc, n, NG, SU, bs, br, d.cv,
                                                                     d.cr, d.meta, d.seg_lo, d.seg_run, d.seg_gend,
                                                                     d.run_user, bad));
  CK(cudaGetLastError());
  int hbad = 0;
  CK(cudaMemcpyAsync(&hbad, bad, sizeof(int), cudaMemcpyDeviceToHost, st));
  CK(cudaStreamSynchronize(st));
  cudaFreeAsync(cs, st);
  cudaFreeAsync(cr, st);
  cudaFreeAsync(br, st);
  cudaFreeAsync(bad, st);
  *out = d;
  if (hbad) return cudaErrorInvalidValue;
  return cudaSuccess;
#undef CK
}

void det_chain_free(DetChain* d, cudaStream_t st) {
  for (void* p : {(void*)d->cv, (void*)d->cr, (void*)d->meta, (void*)d->seg_lo, (void*)d->seg_run, (void*)d->seg_gend,
                  (void*)d->run_user, (void*)d->blk_seg})
    if (p) cudaFreeAsync(p, st);
  *d = DetChain{};
}

cudaError_t launch_wave_chain(const DetChain& d, float* P, float* Q, int64_t row0, int64_t n, int32_t k, float gamma,
                              float lambda, int B, int* progress, cudaStream_t st) {
  ChainArgs a{};
  a.P = P;
  a.Q = Q;
  a.row0 = row0;
  a.n = n;
  a.k = k;
  a.gamma = gamma;
  a.lambda = lambda;
  a.cv = d.cv;
  a.cr = d.cr;
  a.meta = d.meta;
  a.blk_seg = d.blk_seg;
  a.seg_lo = d.seg_lo;
  a.seg_run = d.seg_run;
  a.seg_gend = d.seg_gend;
  a.run_user = d.run_user;
  const int wmax = (int)((n + B - 1) / B);
  cudaError_t e = cudaMemsetAsync(progress, 0, sizeof(int) * kProgressStride * (size_t)B, st);
  if (e != cudaSuccess) return e;
  int SU = 0, ng = 0, v = 0;
  size_t smem = 0;
  if (!chain_shape(k, &ng, &v) || ng != d.NG) return cudaErrorInvalidValue;
  const bool ok = v == 1 ? chain_geometry_t<kNW, 1>(B, wmax, k, &SU, &smem, true)
                         : chain_geometry_t<kNW, 2>(B, wmax, k, &SU, &smem, true);
  if (!ok || SU != d.SU) return cudaErrorInvalidConfiguration;
  cudaLaunchConfig_t cfg{};
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  cfg.stream = st;
  cfg.gridDim = dim3((unsigned)B);
  cfg.blockDim = dim3(kNW * 32);
  cfg.dynamicSmemBytes = smem;
  note_launch();
  e = v == 1 ? cudaLaunchKernelEx(&cfg, sgd_wave_chain_kernel<kNW, 1>, a, B, progress, wmax, SU)
             : cudaLaunchKernelEx(&cfg, sgd_wave_chain_kernel<kNW, 2>, a, B, progress, wmax, SU);
#ifdef HCCMF_DIAG_TRACE
  if (const char* path = getenv("HCCMF_TRACE_OUT")) {
    static std::vector<unsigned> host(2048 * 2048 * 4);
    cudaStreamSynchronize(st);
    cudaMemcpyFromSymbol(host.data(), g_chain_trace, sizeof(unsigned) * 4 * (size_t)B * B);
    if (FILE* f = fopen(path, "wb")) {
      fwrite(host.data(), sizeof(unsigned), 4 * (size_t)B * B, f);
      fclose(f);
    }
  }
#endif
  return e;
}

}  // namespace hccmf
