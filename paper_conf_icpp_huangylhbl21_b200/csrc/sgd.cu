// sgd.cu -- a5/a6: the per-rating SGD update kernel (the hot loop).
//
// PAPER.md section 2.1 (L198-L219) and Fig. 1: for each observed rating r_uv
//   e   = r_uv - p_u . q_v
//   p_u = p_u + gamma (e q_v - lambda p_u)
//   q_v = q_v + gamma (e p_u - lambda q_v)      (p_u: value before the update, R1)
//
// B200 design:
//  * a "rating group" of L lanes (L = next pow2 of k/4, <= 32) owns one rating at a
//    time; lane l holds the float4 slices (v*L + l) of p_u and q_v, so every
//    factor access is a coalesced 128-bit load/store.  k = 128 -> one rating per
//    warp (L = 32); k = 32 -> four independent rating groups per warp (L = 8).
//  * the dot product is reduced with log2(L) __shfl_xor_sync steps.
//  * a persistent grid pulls tasks (record ranges [lo, hi)) from an atomic
//    queue.  Hogwild tasks are runs of whole users (never split), so p_u is
//    carried in registers across a user's ratings and written back once;
//    q_v races between groups by design (Hogwild!, L216-L219, L1680-L1691).
//    DET tasks are FPSGD blocks of one stratum, which share no rows or columns.
//  * records are read once per epoch with streaming loads (L rating triples per
//    coalesced window, broadcast by shuffles); P/Q go through L2 only (.cg), so a
//    racing group never reads a stale line from its own SM's L1.
//  * rating groups of a warp run in lock step (no divergent shuffles).
#include "internal.cuh"

namespace hccmf {
namespace {

constexpr int kThreads = 256;

template <int L, int VEC, bool FULL>
__device__ __forceinline__ void load_row(const float* row, float4 (&x)[VEC], int sl, int k) {
#pragma unroll
  for (int i = 0; i < VEC; ++i) {
    const int c = (i * L + sl) * 4;
    if (FULL || c < k)
      x[i] = __ldcg(reinterpret_cast<const float4*>(row + c));
    else
      x[i] = make_float4(0.f, 0.f, 0.f, 0.f);
  }
}

template <int L, int VEC, bool FULL>
__device__ __forceinline__ void store_row(float* row, const float4 (&x)[VEC], int sl, int k) {
#pragma unroll
  for (int i = 0; i < VEC; ++i) {
    const int c = (i * L + sl) * 4;
    if (FULL || c < k) __stcg(reinterpret_cast<float4*>(row + c), x[i]);
  }
}

// Hogwild! (Recht et al., the paper's ref [21], L216-L219) applies each update as
// atomic component-wise additions: q_v += delta with one 128-bit vector reduction
// per lane (red.global.add.v4.f32, sm_90+), so racing groups never lose an update
// -- only read a slightly stale q_v.
template <int L, int VEC, bool FULL>
__device__ __forceinline__ void red_row(float* row, const float4 (&d)[VEC], int sl, int k) {
#pragma unroll
  for (int i = 0; i < VEC; ++i) {
    const int c = (i * L + sl) * 4;
    if (FULL || c < k)
      asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(row + c), "f"(d[i].x),
                   "f"(d[i].y), "f"(d[i].z), "f"(d[i].w)
                   : "memory");
  }
}

__device__ __forceinline__ float upd(float a, float b, float e, float g, float lam) {
  // a + gamma * (e * b - lambda * a)
  return a + g * (e * b - lam * a);
}

template <int L, int VEC, bool FULL, bool ATOMIC>
__global__ void __launch_bounds__(kThreads) sgd_kernel(SgdArgs a) {
  constexpr unsigned FM = 0xffffffffu;
  const int lane = threadIdx.x & 31;
  const int sl = lane & (L - 1);
  const int k = a.k;
  const float g = a.gamma, lam = a.lambda;

  int64_t cur = 0, end = 0, wbase = 0;
  bool done = false, have_win = false;
  int wu = 0, wv = 0;
  float wr = 0.f;
  int cu = -1;
  int lastv = -1;  // q_v forwarding: the item this group updated last and its new value
  float4 p[VEC], lastq[VEC];
#pragma unroll
  for (int i = 0; i < VEC; ++i) p[i] = lastq[i] = make_float4(0.f, 0.f, 0.f, 0.f);

  while (true) {
    // ---- task queue: one atomic per rating group, broadcast inside the group
    const bool need = !done && cur >= end;
    unsigned long long t = 0;
    if (need && sl == 0) t = atomicAdd(a.counter, 1ull);
    t = __shfl_sync(FM, t, 0, L);
    if (need) {
      if (cu >= 0) store_row<L, VEC, FULL>(a.P + (int64_t)(cu - a.row0) * k, p, sl, k);
      cu = -1;
      if (t < (unsigned long long)a.n_tasks) {
        cur = a.task_lo[t];
        end = a.task_hi[t];
        have_win = false;
        lastv = -1;
      } else {
        done = true;
      }
    }
    if (__all_sync(FM, done)) break;
    const bool act = !done;  // tasks are never empty

    // ---- record window: L consecutive ratings, one per lane, coalesced
    if (act && (!have_win || cur >= wbase + L)) {
      wbase = cur;
      have_win = true;
      const int64_t idx = cur + sl;
      if (idx < end) {
        wu = __ldcs(a.ru + idx);
        wv = __ldcs(a.rv + idx);
        wr = __ldcs(a.rr + idx);
      }
    }
    const int j = (int)(cur - wbase) & (L - 1);
    const int uu = __shfl_sync(FM, wu, j, L);
    const int vv = __shfl_sync(FM, wv, j, L);
    const float rv = __shfl_sync(FM, wr, j, L);

    // ---- e = r - p.q
    float4 q[VEC];
    float d = 0.f;
    if (act) {
      if (uu != cu) {
        if (cu >= 0) store_row<L, VEC, FULL>(a.P + (int64_t)(cu - a.row0) * k, p, sl, k);
        load_row<L, VEC, FULL>(a.P + (int64_t)(uu - a.row0) * k, p, sl, k);
        cu = uu;
      }
      if (vv == lastv) {  // consecutive ratings of one item (duplicates): serial read-after-write
#pragma unroll
        for (int i = 0; i < VEC; ++i) q[i] = lastq[i];
      } else {
        load_row<L, VEC, FULL>(a.Q + (int64_t)vv * k, q, sl, k);
      }
#pragma unroll
      for (int i = 0; i < VEC; ++i) {
        d = fmaf(p[i].x, q[i].x, d);
        d = fmaf(p[i].y, q[i].y, d);
        d = fmaf(p[i].z, q[i].z, d);
        d = fmaf(p[i].w, q[i].w, d);
      }
    }
#pragma unroll
    for (int o = L / 2; o > 0; o >>= 1) d += __shfl_xor_sync(FM, d, o);

    // ---- p += g(e q - lam p);  q += g(e p_old - lam q)
    if (act) {
      const float e = rv - d;
#pragma unroll
      for (int i = 0; i < VEC; ++i) {
        const float4 pp = p[i], qq = q[i];
        p[i] = make_float4(upd(pp.x, qq.x, e, g, lam), upd(pp.y, qq.y, e, g, lam),
                           upd(pp.z, qq.z, e, g, lam), upd(pp.w, qq.w, e, g, lam));
        // increment gamma (e p_old - lambda q); ATOMIC adds it with a vector red
        const float4 dq = make_float4(g * (e * pp.x - lam * qq.x), g * (e * pp.y - lam * qq.y),
                                      g * (e * pp.z - lam * qq.z), g * (e * pp.w - lam * qq.w));
        lastq[i] = make_float4(qq.x + dq.x, qq.y + dq.y, qq.z + dq.z, qq.w + dq.w);
        q[i] = ATOMIC ? dq : lastq[i];
      }
      lastv = vv;
      if (ATOMIC)
        red_row<L, VEC, FULL>(a.Q + (int64_t)vv * k, q, sl, k);
      else
        store_row<L, VEC, FULL>(a.Q + (int64_t)vv * k, q, sl, k);
      ++cur;
    }
  }
}

template <int L, int VEC, bool FULL>
cudaError_t launch_t(const SgdArgs& a, int64_t warps, cudaStream_t st) {
  constexpr int groups_per_warp = 32 / L;
  int64_t need_warps = (a.n_tasks + groups_per_warp - 1) / groups_per_warp;
  int64_t w = warps < need_warps ? warps : need_warps;
  if (w < 1) return cudaSuccess;
  const int64_t blocks = (w * 32 + kThreads - 1) / kThreads;
  if (a.atomic_q)
    sgd_kernel<L, VEC, FULL, true><<<(unsigned)blocks, kThreads, 0, st>>>(a);
  else
    sgd_kernel<L, VEC, FULL, false><<<(unsigned)blocks, kThreads, 0, st>>>(a);
  return cudaGetLastError();
}

}  // namespace

int lanes_per_rating(int k) {
  const int c4 = k / 4;
  if (c4 >= 32) return 32;
  int L = 1;
  while (L < c4) L <<= 1;
  return L;
}

cudaError_t launch_sgd(const SgdArgs& a, int64_t warps, cudaStream_t st) {
  if (a.n_tasks <= 0) return cudaSuccess;
  const int c4 = a.k / 4;
  if (c4 > 32) {
    const int vec = (c4 + 31) / 32;
    const bool full = (c4 == 32 * vec);
    switch (vec) {
      case 2: return full ? launch_t<32, 2, true>(a, warps, st) : launch_t<32, 2, false>(a, warps, st);
      case 3: return full ? launch_t<32, 3, true>(a, warps, st) : launch_t<32, 3, false>(a, warps, st);
      case 4: return full ? launch_t<32, 4, true>(a, warps, st) : launch_t<32, 4, false>(a, warps, st);
      default: return cudaErrorInvalidValue;
    }
  }
  const int L = lanes_per_rating(a.k);
  const bool full = (L == c4);
  switch (L) {
    case 1: return launch_t<1, 1, true>(a, warps, st);
    case 2: return full ? launch_t<2, 1, true>(a, warps, st) : launch_t<2, 1, false>(a, warps, st);
    case 4: return full ? launch_t<4, 1, true>(a, warps, st) : launch_t<4, 1, false>(a, warps, st);
    case 8: return full ? launch_t<8, 1, true>(a, warps, st) : launch_t<8, 1, false>(a, warps, st);
    case 16: return full ? launch_t<16, 1, true>(a, warps, st) : launch_t<16, 1, false>(a, warps, st);
    case 32: return full ? launch_t<32, 1, true>(a, warps, st) : launch_t<32, 1, false>(a, warps, st);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace hccmf
