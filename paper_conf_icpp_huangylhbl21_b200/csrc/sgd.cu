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
#include <algorithm>

#include "internal.cuh"

namespace hccmf {
namespace {

constexpr int kThreads = 256;

// per-lane slice validity: slot i of lane sl holds elements (i*L + sl)*4 .. +3
template <int L, int VEC>
__device__ __forceinline__ void load_row(const float* row, float4 (&x)[VEC], const bool (&ok)[VEC], int sl) {
#pragma unroll
  for (int i = 0; i < VEC; ++i)
    x[i] = ok[i] ? __ldcg(reinterpret_cast<const float4*>(row + (i * L + sl) * 4)) : make_float4(0.f, 0.f, 0.f, 0.f);
}

template <int L, int VEC>
__device__ __forceinline__ void store_row(float* row, const float4 (&x)[VEC], const bool (&ok)[VEC], int sl) {
#pragma unroll
  for (int i = 0; i < VEC; ++i)
    if (ok[i]) __stcg(reinterpret_cast<float4*>(row + (i * L + sl) * 4), x[i]);
}

// Hogwild! (Recht et al., the paper's ref [21], L216-L219) applies each update as
// atomic component-wise additions: q_v += delta with one 128-bit vector reduction
// per slot (red.global.add.v4.f32, sm_90+), so racing groups never lose an update
// -- they only read a slightly stale q_v.
template <int L, int VEC>
__device__ __forceinline__ void red_row(float* row, const float4 (&d)[VEC], const bool (&ok)[VEC], int sl) {
#pragma unroll
  for (int i = 0; i < VEC; ++i)
    if (ok[i]) {
#ifdef HCCMF_SCALAR_RED
      float* r4 = row + (i * L + sl) * 4;
      atomicAdd(r4 + 0, d[i].x);
      atomicAdd(r4 + 1, d[i].y);
      atomicAdd(r4 + 2, d[i].z);
      atomicAdd(r4 + 3, d[i].w);
#else
      asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(row + (i * L + sl) * 4),
                   "f"(d[i].x), "f"(d[i].y), "f"(d[i].z), "f"(d[i].w)
                   : "memory");
#endif
    }
}

// One kernel for both schedules.  Per rating group (L lanes, lock step inside the
// warp) the loop is software-pipelined one rating deep:
//   iteration j: take rating j+1 from the record window, issue the loads of
//   q_{v(j+1)} and (on a user change) p_{u(j+1)}, then update rating j.
// Hazards: q_{v(j+1)} == q_{v(j)} is forwarded from registers (the serial
// read-after-write), p rows are owned by the group for the whole task.  Record
// windows (WR ratings, coalesced) are double-buffered; the next task id is
// fetched one task ahead.
template <int L, int VEC, bool ATOMIC>
__global__ void __launch_bounds__(kThreads) sgd_kernel(SgdArgs a) {
  constexpr unsigned FM = 0xffffffffu;
  constexpr int RPL = L >= 8 ? 1 : 8 / L;  // records per lane per window
  constexpr int WR = L * RPL;              // records per window
  const int lane = threadIdx.x & 31;
  const int sl = lane & (L - 1);
  const int k = a.k;
  const float g = a.gamma;
  const float c1 = 1.f - a.gamma * a.lambda;  // p' = c1 p + (g e) q
  const float gl = a.gamma * a.lambda;        // dq = (g e) p - (g lambda) q
  const int32_t* __restrict__ ru = a.ru;
  const int32_t* __restrict__ rv = a.rv;
  const float* __restrict__ rr = a.rr;
  float* __restrict__ P = a.P;
  float* __restrict__ Q = a.Q;
  bool ok[VEC];
#pragma unroll
  for (int i = 0; i < VEC; ++i) ok[i] = (i * L + sl) * 4 < k;

  int64_t pos = 0, end = 0, wb = 0;
  bool live = false, done = false;
  int wu0[RPL], wv0[RPL], wu1[RPL], wv1[RPL];
  float wr0[RPL], wr1[RPL];
#pragma unroll
  for (int t = 0; t < RPL; ++t) wu0[t] = wv0[t] = wu1[t] = wv1[t] = 0, wr0[t] = wr1[t] = 0.f;
  int cu = 0, cv = 0;
  float cr = 0.f;
  float4 p[VEC], q[VEC], pn[VEC], qn[VEC];
#pragma unroll
  for (int i = 0; i < VEC; ++i) p[i] = q[i] = pn[i] = qn[i] = make_float4(0.f, 0.f, 0.f, 0.f);

  unsigned long long tnext = 0;
  if (sl == 0) tnext = atomicAdd(a.counter, 1ull);

  auto load_window = [&](int (&wu)[RPL], int (&wv)[RPL], float (&wr)[RPL], int64_t base) {
#pragma unroll
    for (int t = 0; t < RPL; ++t) {
      const int64_t idx = base + t * L + sl;
      if (idx < end) {
        wu[t] = __ldcs(ru + idx);
        wv[t] = __ldcs(rv + idx);
        wr[t] = __ldcs(rr + idx);
      }
    }
  };
  // rating idx (in [wb, wb + WR)) broadcast inside the group; executed by all lanes
  auto fetch = [&](int64_t idx, int& u, int& v, float& r) {
    const int j = (int)(idx - wb) & (WR - 1);
    const int t = j / L, src = j & (L - 1);
    int xu = wu0[0], xv = wv0[0];
    float xr = wr0[0];
#pragma unroll
    for (int tt = 1; tt < RPL; ++tt)
      if (t == tt) xu = wu0[tt], xv = wv0[tt], xr = wr0[tt];
    u = __shfl_sync(FM, xu, src, L);
    v = __shfl_sync(FM, xv, src, L);
    r = __shfl_sync(FM, xr, src, L);
  };

  while (true) {
    // ---- task start (a group whose task ended takes the prefetched id)
    const bool need = !done && !live;
    if (__any_sync(FM, need)) {
      const unsigned long long t = __shfl_sync(FM, tnext, 0, L);
      if (need) {
        if (t < (unsigned long long)a.n_tasks) {
          pos = a.task_lo[t];
          end = a.task_hi[t];
          live = true;
          wb = pos;
          load_window(wu0, wv0, wr0, wb);
          load_window(wu1, wv1, wr1, wb + WR);
          if (sl == 0) tnext = atomicAdd(a.counter, 1ull);
        } else {
          done = true;
        }
      }
      int u0, v0;
      float r0;
      fetch(pos, u0, v0, r0);
      if (need && live) {
        cu = u0;
        cv = v0;
        cr = r0;
        load_row<L, VEC>(P + (int64_t)(cu - a.row0) * k, p, ok, sl);
        load_row<L, VEC>(Q + (int64_t)cv * k, q, ok, sl);
      }
    }
    if (__all_sync(FM, done)) break;

    // ---- look ahead: rating pos+1 and its operands
    const bool has_next = live && (pos + 1 < end);
    if (has_next && pos + 1 >= wb + WR) {  // slide the double-buffered window
#pragma unroll
      for (int t = 0; t < RPL; ++t) wu0[t] = wu1[t], wv0[t] = wv1[t], wr0[t] = wr1[t];
      wb += WR;
      load_window(wu1, wv1, wr1, wb + WR);
    }
    int nu, nv;
    float nr;
    fetch(pos + 1, nu, nv, nr);
    if (has_next) {
      if (nv != cv) load_row<L, VEC>(Q + (int64_t)nv * k, qn, ok, sl);
      if (nu != cu) load_row<L, VEC>(P + (int64_t)(nu - a.row0) * k, pn, ok, sl);
    }

    // ---- e = r - p.q  (four independent partial sums, then log2(L) shuffles)
    float d0 = 0.f, d1 = 0.f, d2 = 0.f, d3 = 0.f;
    if (live) {
#pragma unroll
      for (int i = 0; i < VEC; ++i) {
        d0 = fmaf(p[i].x, q[i].x, d0);
        d1 = fmaf(p[i].y, q[i].y, d1);
        d2 = fmaf(p[i].z, q[i].z, d2);
        d3 = fmaf(p[i].w, q[i].w, d3);
      }
    }
    float d = (d0 + d1) + (d2 + d3);
#pragma unroll
    for (int o = L / 2; o > 0; o >>= 1) d += __shfl_xor_sync(FM, d, o);

    // ---- p' = p + g(e q - lambda p);  q' = q + g(e p - lambda q)   (p: pre-update)
    if (live) {
      const float ge = g * (cr - d);
      float4 dq[VEC];
#pragma unroll
      for (int i = 0; i < VEC; ++i) {
        const float4 pp = p[i], qq = q[i];
        p[i] = make_float4(fmaf(ge, qq.x, c1 * pp.x), fmaf(ge, qq.y, c1 * pp.y), fmaf(ge, qq.z, c1 * pp.z),
                           fmaf(ge, qq.w, c1 * pp.w));
        dq[i] = make_float4(fmaf(ge, pp.x, -gl * qq.x), fmaf(ge, pp.y, -gl * qq.y), fmaf(ge, pp.z, -gl * qq.z),
                            fmaf(ge, pp.w, -gl * qq.w));
        q[i] = make_float4(qq.x + dq[i].x, qq.y + dq[i].y, qq.z + dq[i].z, qq.w + dq[i].w);
      }
      if (ATOMIC)
        red_row<L, VEC>(Q + (int64_t)cv * k, dq, ok, sl);
      else
        store_row<L, VEC>(Q + (int64_t)cv * k, q, ok, sl);
      if (!has_next) {
        store_row<L, VEC>(P + (int64_t)(cu - a.row0) * k, p, ok, sl);
        live = false;
      } else {
        if (nu != cu) {
          store_row<L, VEC>(P + (int64_t)(cu - a.row0) * k, p, ok, sl);
#pragma unroll
          for (int i = 0; i < VEC; ++i) p[i] = pn[i];
        }
        if (nv != cv) {
#pragma unroll
          for (int i = 0; i < VEC; ++i) q[i] = qn[i];
        }
        cu = nu;
        cv = nv;
        cr = nr;
        ++pos;
      }
    }
  }
}

template <int L, int VEC>
cudaError_t launch_t(const SgdArgs& a, int64_t warps, cudaStream_t st) {
  constexpr int groups_per_warp = 32 / L;
  int64_t need_warps = (a.n_tasks + groups_per_warp - 1) / groups_per_warp;
  int64_t w = warps < need_warps ? warps : need_warps;
  if (w < 1) return cudaSuccess;
  // exactly w warps when w < 8 (one partial CTA), else whole CTAs of 8 warps
  const int threads = w < kThreads / 32 ? (int)w * 32 : kThreads;
  const int64_t blocks = (w * 32 + threads - 1) / threads;
  if (a.atomic_q)
    sgd_kernel<L, VEC, true><<<(unsigned)blocks, threads, 0, st>>>(a);
  else
    sgd_kernel<L, VEC, false><<<(unsigned)blocks, threads, 0, st>>>(a);
  return cudaGetLastError();
}

}  // namespace

// Lane geometry: VEC float4 slots per lane, L lanes per
// rating group.  Auto: VEC = 2 for k >= 64 (k = 128: L = 16, two ratings per
// warp), else 1; L is capped at 32 (k = 512 -> VEC = 4); VEC = 3 is rounded up to
// 4 (masked).  VEC = 4 at k = 128 packs 9472 groups on the chip, a concurrency
// at which atomic Hogwild was seen to diverge on the Netflix shape (R14).
void sgd_geometry(int k, int vec_pref, int* L_out, int* VEC_out) {
  const int c4 = k / 4;
  int vec = vec_pref > 0 ? vec_pref : (c4 >= 16 ? 2 : 1);
  if (vec == 3) vec = 4;
  auto pow2 = [](int x) { int l = 1; while (l < x) l <<= 1; return l; };
  int L = std::min(32, pow2((c4 + vec - 1) / vec));
  vec = (c4 + L - 1) / L;
  if (vec == 3) vec = 4;
  if (L < 8 && vec > 1) {  // only VEC = 1 is instantiated below 8 lanes
    vec = 1;
    L = std::min(32, pow2(c4));
    vec = (c4 + L - 1) / L;
    if (vec == 3) vec = 4;
  }
  *L_out = L;
  *VEC_out = vec;
}

int sgd_lanes(int k, int vec_pref) {
  int L, V;
  sgd_geometry(k, vec_pref, &L, &V);
  return L;
}

int lanes_per_rating(int k) {  // RMSE kernel: one float4 slot per lane
  const int c4 = k / 4;
  if (c4 >= 32) return 32;
  int L = 1;
  while (L < c4) L <<= 1;
  return L;
}

cudaError_t launch_sgd(const SgdArgs& a, int64_t warps, cudaStream_t st) {
  if (a.n_tasks <= 0) return cudaSuccess;
  int L, VEC;
  sgd_geometry(a.k, a.vec_pref, &L, &VEC);
#define SGD_CASE(LL, VV) \
  if (L == LL && VEC == VV) return launch_t<LL, VV>(a, warps, st);
  SGD_CASE(1, 1) SGD_CASE(2, 1) SGD_CASE(4, 1)
  SGD_CASE(8, 1) SGD_CASE(8, 2) SGD_CASE(8, 4)
  SGD_CASE(16, 1) SGD_CASE(16, 2) SGD_CASE(16, 4)
  SGD_CASE(32, 1) SGD_CASE(32, 2) SGD_CASE(32, 4)
#undef SGD_CASE
  return cudaErrorInvalidValue;
}

}  // namespace hccmf
