// sgd.cu -- a5/a6: the per-rating SGD update kernel (the hot loop).
//
// PAPER.md section 2.1 (L198-L219) and Fig. 1: for each observed rating r_uv
//   e   = r_uv - p_u . q_v
//   p_u = p_u + gamma (e q_v - lambda p_u)
//   q_v = q_v + gamma (e p_u - lambda q_v)      (p_u: value before the update, R1)
//
// B200 design:
//  * a "rating group" of L lanes owns one rating at a time; lane l holds VEC float4
//    slots (elements (i*L + l)*4 ..) of p_u and q_v, so every factor access is a
//    coalesced 128-bit load/store/red.  k < 128: L = k/4 lanes, 32/L groups per warp in
//    lock step; k = 128 j: one rating per warp (WarpSgd).  The dot product is two packed
//    FFMA2 chains + log2(L) shuffles; all float4 arithmetic runs on the fp32x2 pipe.
//  * a persistent grid pulls tasks (record ranges [lo, hi)) from an atomic queue.
//    Hogwild tasks are runs of whole users, so p_u stays in registers across a
//    user's ratings; DET tasks are the blocks of one stratum (no shared rows or
//    columns).  q_v increments are vector reductions (Hogwild!, L216-L219).
//  * software pipeline, one rating deep: while rating j is updated the record of
//    j+1 is taken from a double-buffered coalesced window and q_{v(j+1)} (and on a
//    user change p_{u(j+1)}) is already in flight.  The loop body is unrolled twice
//    with the current / next q registers swapping roles (no register copies);
//    q_{v(j+1)} == q_{v(j)} is forwarded from registers (serial read-after-write).
//  * 32-bit row offsets and a compile-time full-vector geometry keep the per-rating
//    instruction count low (profiles/).
//  * the warp-per-rating Hogwild loop (k = 128 j) takes its records from a per-warp
//    shared-memory ring filled by cp.async one window of 32 ahead (one broadcast
//    LDS.128 per rating) and carries each row address from its prefetch to its red;
//    an optional deeper q prefetch (D = 2..4) keeps D + 1 rows in flight.
#include <cuda_fp16.h>

#include <algorithm>
#include <type_traits>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "internal.cuh"

namespace hccmf {
namespace {

constexpr int kThreads = 256;
#ifndef HCCMF_WARP_UNROLL  // 2-rating steps per record-ring loop iteration (Hogwild, k = 128 j)
#define HCCMF_WARP_UNROLL 8
#endif
#ifndef HCCMF_WARP_MINB1  // CTAs of 8 warps per SM the k = 128 warp kernel is compiled for (registers)
#define HCCMF_WARP_MINB1 4
#endif
#ifndef HCCMF_NARROW_UNROLL  // R-rating rounds per loop iteration (Hogwild, k = 32 / 64)
#define HCCMF_NARROW_UNROLL 1
#endif
constexpr int kWarpUnroll = HCCMF_WARP_UNROLL, kNarrowUnroll = HCCMF_NARROW_UNROLL;

template <int VEC>
struct Row {
  float4 x[VEC];
};

// Per-lane view of a factor row: slot i of lane sl is float4 index (i*L + sl).
template <int L, int VEC, bool FULL>
struct Lanes {
  bool ok[VEC];
  __device__ __forceinline__ void init(int sl, int k4) {
#pragma unroll
    for (int i = 0; i < VEC; ++i) ok[i] = FULL || (i * L + sl) < k4;
  }
  __device__ __forceinline__ void load(const float4* row, Row<VEC>& r) const {
#pragma unroll
    for (int i = 0; i < VEC; ++i) r.x[i] = (FULL || ok[i]) ? __ldcg(row + i * L) : make_float4(0.f, 0.f, 0.f, 0.f);
  }
  __device__ __forceinline__ void store(float4* row, const Row<VEC>& r) const {
#pragma unroll
    for (int i = 0; i < VEC; ++i)
      if (FULL || ok[i]) __stcg(row + i * L, r.x[i]);
  }
  // Hogwild! applies increments as atomic component-wise additions:
  // one 128-bit vector reduction per slot (red.global.add.v4.f32, sm_90+).
  __device__ __forceinline__ void red(float4* row, const Row<VEC>& d) const {
#pragma unroll
    for (int i = 0; i < VEC; ++i)
      if (FULL || ok[i])
        asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(row + i * L),
                     "f"(d.x[i].x), "f"(d.x[i].y), "f"(d.x[i].z), "f"(d.x[i].w)
                     : "memory");
  }
};

// float4 arithmetic on the sm_100 packed fp32x2 pipe (FFMA2 / FMUL2 / FADD2: two IEEE fp32
// operations per instruction, each correctly rounded as its scalar counterpart)
__device__ __forceinline__ float2 lo2(float4 a) { return make_float2(a.x, a.y); }
__device__ __forceinline__ float2 hi2(float4 a) { return make_float2(a.z, a.w); }
__device__ __forceinline__ float4 cat2(float2 l, float2 h) { return make_float4(l.x, l.y, h.x, h.y); }
__device__ __forceinline__ float4 f4_fma(float s, float4 a, float4 b) {  // s*a + b
  const float2 ss = make_float2(s, s);
  return cat2(__ffma2_rn(ss, lo2(a), lo2(b)), __ffma2_rn(ss, hi2(a), hi2(b)));
}
__device__ __forceinline__ float4 f4_scale(float s, float4 a) {
  const float2 ss = make_float2(s, s);
  return cat2(__fmul2_rn(ss, lo2(a)), __fmul2_rn(ss, hi2(a)));
}
__device__ __forceinline__ float4 f4_add(float4 a, float4 b) {
  return cat2(__fadd2_rn(lo2(a), lo2(b)), __fadd2_rn(hi2(a), hi2(b)));
}
// two fp32 dot-product chains (elements x,z and y,w): acc + a .* b, packed
__device__ __forceinline__ float2 f4_dot2(float4 a, float4 b, float2 acc) {
  return __ffma2_rn(hi2(a), hi2(b), __ffma2_rn(lo2(a), lo2(b), acc));
}
// four binary16 (two half2 words) <-> float4, round to nearest even (storage = 1)
__device__ __forceinline__ uint2 f4_to_h4(float4 a) {
  const __half2 lo = __floats2half2_rn(a.x, a.y), hi = __floats2half2_rn(a.z, a.w);
  return make_uint2(*reinterpret_cast<const unsigned*>(&lo), *reinterpret_cast<const unsigned*>(&hi));
}
// Stochastic rounding (storage = 2, R27).  The random word of element pair c
// (elements 2c, 2c+1) of the q_v write by the update of record i (global index in the
// sorted order) in epoch t is, for even c, r = lowbias32(i*0x9E3779B1 + t*0x85EBCA77 +
// c*0xC2B2AE3D) (mod 2^32; lowbias32 = C. Wellons' 32-bit finaliser) and, for odd c, the
// even neighbour's word times 0x9E3779B1 (one multiply instead of a second finaliser: a
// bijection of the even word, so each 13-bit field stays uniform); element 2c is rounded with
// r[12:0], element 2c+1 with r[28:16] by cvt.rs.f16x2.f32 (sm_100a F2FP.RS):
// y = sign(x) floor((|x| + R13 ulp / 2^13) / ulp) ulp, ulp = the binary16 spacing at |x|.
__device__ __forceinline__ unsigned lowbias32(unsigned x) {
  x ^= x >> 16;
  x *= 0x7FEB352Du;
  x ^= x >> 15;
  x *= 0x846CA68Bu;
  x ^= x >> 16;
  return x;
}
__device__ __forceinline__ unsigned cvt_rs_h2(float hi, float lo, unsigned r) {
  unsigned d;
  asm("cvt.rs.f16x2.f32 %0, %1, %2, %3;" : "=r"(d) : "f"(hi), "f"(lo), "r"(r));
  return d;
}
__device__ __forceinline__ unsigned hsub2_bits(unsigned a, unsigned b) {  // a - b, binary16 x2, RN
  unsigned d;
  asm("sub.rn.f16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
  return d;
}
__device__ __forceinline__ float4 h4_to_f4(uint2 r) {
  const float2 lo = __half22float2(*reinterpret_cast<const __half2*>(&r.x));
  const float2 hi = __half22float2(*reinterpret_cast<const __half2*>(&r.y));
  return make_float4(lo.x, lo.y, hi.x, hi.y);
}

template <int L, int VEC, bool FULL, bool ATOMIC>
struct Group {
  static constexpr unsigned FM = 0xffffffffu;
  static constexpr int RPL = L >= 8 ? 1 : 8 / L;  // records per lane per window
  static constexpr int WR = L * RPL;              // ratings per window

  const SgdArgs& a;
  const int sl, k4;
  const float g, c1, ngl;  // p' = c1 p + (g e) q ;  dq = (g e) p - (g lambda) q
  Lanes<L, VEC, FULL> lanes;
  const float4* Pb;  // lane-adjusted bases: row r, slot i at base + r*k4 + i*L
  const float4* Qb;

  // task / window state (uniform inside the group)
  int64_t wbase = 0;  // record index of window 0
  int jw = 0;         // position of the current rating in window 0
  int left = 0;       // ratings of the task from the current one on
  bool live = false, done = false;
  int wu0[RPL], wv0[RPL], wu1[RPL], wv1[RPL];
  float wr0[RPL], wr1[RPL];
  // current rating
  int cu = 0, cv = 0;
  float cr = 0.f;
  Row<VEC> p, pn;
  unsigned long long tnext = 0;

  __device__ Group(const SgdArgs& args, int sl_)
      : a(args), sl(sl_), k4(args.k >> 2), g(args.gamma), c1(1.f - args.gamma * args.lambda),
        ngl(-args.gamma * args.lambda) {
    lanes.init(sl, k4);
    Pb = reinterpret_cast<const float4*>(a.P) + sl - (int64_t)a.row0 * k4;
    Qb = reinterpret_cast<const float4*>(a.Q) + sl;
#pragma unroll
    for (int t = 0; t < RPL; ++t) wu0[t] = wv0[t] = wu1[t] = wv1[t] = 0, wr0[t] = wr1[t] = 0.f;
  }

  // row addresses with one 32x32->64 multiply-add (ids are non-negative and < 2^31)
  __device__ __forceinline__ const float4* prow(int u) const {
    return reinterpret_cast<const float4*>(reinterpret_cast<const char*>(Pb) +
                                           (unsigned long long)(unsigned)u * (unsigned)(k4 * 16));
  }
  __device__ __forceinline__ const float4* qrow(int v) const {
    return reinterpret_cast<const float4*>(reinterpret_cast<const char*>(Qb) +
                                           (unsigned long long)(unsigned)v * (unsigned)(k4 * 16));
  }

  __device__ __forceinline__ void load_window(int (&wu)[RPL], int (&wv)[RPL], float (&wr)[RPL], int64_t base,
                                              int avail) {
#pragma unroll
    for (int t = 0; t < RPL; ++t) {
      const int j = t * L + sl;
      if (j < avail) {
        wu[t] = __ldcs(a.ru + base + j);
        wv[t] = __ldcs(a.rv + base + j);
        wr[t] = __ldcs(a.rr + base + j);
      }
    }
  }
  // rating at position j of window 0, broadcast inside the group (all lanes execute)
  __device__ __forceinline__ void fetch(int j, int& u, int& v, float& r) const {
    const int t = (j & (WR - 1)) / L, src = j & (L - 1);
    int xu = wu0[0], xv = wv0[0];
    float xr = wr0[0];
#pragma unroll
    for (int tt = 1; tt < RPL; ++tt)
      if (t == tt) xu = wu0[tt], xv = wv0[tt], xr = wr0[tt];
    u = __shfl_sync(FM, xu, src, L);
    v = __shfl_sync(FM, xv, src, L);
    r = __shfl_sync(FM, xr, src, L);
  }

  // Task start for groups that need one (all lanes of the warp execute this).
  __device__ __forceinline__ void refill(Row<VEC>& qc) {
    const bool need = !done && !live;
    if (!__any_sync(FM, need)) return;
    const unsigned long long t = __shfl_sync(FM, tnext, 0, L);
    if (need) {
      if (t < (unsigned long long)a.n_tasks) {
        const int64_t lo = a.task_lo[t], hi = a.task_hi[t];
        wbase = lo;
        jw = 0;
        left = (int)(hi - lo);
        live = true;
        load_window(wu0, wv0, wr0, wbase, left);
        load_window(wu1, wv1, wr1, wbase + WR, left - WR);
        if (sl == 0) tnext = atomicAdd(a.counter, 1ull);
      } else {
        done = true;
      }
    }
    int u0, v0;
    float r0;
    fetch(0, u0, v0, r0);
    if (need && live) {
      cu = u0;
      cv = v0;
      cr = r0;
      lanes.load(prow(cu), p);
      lanes.load(qrow(cv), qc);
    }
  }

  // One pipelined step: update the current rating (q in qc), prefetch the next into qn.
  __device__ __forceinline__ void step(Row<VEC>& qc, Row<VEC>& qn) {
    const bool has_next = live && left > 1;
    // ---- next record (slide the double-buffered window when it is used up)
    int jn = jw + 1;
    if (has_next && jn == WR) {
#pragma unroll
      for (int t = 0; t < RPL; ++t) wu0[t] = wu1[t], wv0[t] = wv1[t], wr0[t] = wr1[t];
      wbase += WR;
      jn = 0;
      load_window(wu1, wv1, wr1, wbase + WR, left - 1 - WR);
    }
    int nu, nv;
    float nr;
    fetch(jn, nu, nv, nr);
    const bool newq = has_next && nv != cv;
    const bool newp = has_next && nu != cu;
    if (newq) lanes.load(qrow(nv), qn);
    if (newp) lanes.load(prow(nu), pn);

    // ---- e = r - p.q
    float2 dd = make_float2(0.f, 0.f);
#pragma unroll
    for (int i = 0; i < VEC; ++i) dd = f4_dot2(p.x[i], qc.x[i], dd);
    float d = dd.x + dd.y;
#pragma unroll
    for (int o = L / 2; o > 0; o >>= 1) d += __shfl_xor_sync(FM, d, o);

    if (live) {
      // ---- p' = c1 p + (g e) q ;  dq = (g e) p - (g lambda) q   (p: pre-update)
      const float ge = g * (cr - d);
      Row<VEC> dq;
#pragma unroll
      for (int i = 0; i < VEC; ++i) {
        dq.x[i] = f4_fma(ge, p.x[i], f4_scale(ngl, qc.x[i]));
        p.x[i] = f4_fma(ge, qc.x[i], f4_scale(c1, p.x[i]));
      }
      float4* qrow_w = const_cast<float4*>(qrow(cv));
      if (ATOMIC) {
        lanes.red(qrow_w, dq);
      } else {
#pragma unroll
        for (int i = 0; i < VEC; ++i) dq.x[i] = f4_add(qc.x[i], dq.x[i]);
        lanes.store(qrow_w, dq);
      }
      if (has_next && !newq) {  // same item next: forward the updated q_v
#pragma unroll
        for (int i = 0; i < VEC; ++i) qn.x[i] = ATOMIC ? f4_add(qc.x[i], dq.x[i]) : dq.x[i];
      }
      if (!has_next || newp) lanes.store(const_cast<float4*>(prow(cu)), p);
      if (newp) p = pn;
      live = has_next;
      cu = nu;
      cv = nv;
      cr = nr;
      jw = jn;
      --left;
    }
  }
};

template <int L, int VEC, bool FULL, bool ATOMIC>
__global__ void __launch_bounds__(kThreads) sgd_kernel(SgdArgs a) {
  Group<L, VEC, FULL, ATOMIC> grp(a, threadIdx.x & (L - 1));
  if (grp.sl == 0) grp.tnext = atomicAdd(a.counter, 1ull);
  Row<VEC> qa, qb;
#pragma unroll
  for (int i = 0; i < VEC; ++i) qa.x[i] = qb.x[i] = grp.p.x[i] = grp.pn.x[i] = make_float4(0.f, 0.f, 0.f, 0.f);
  while (true) {
    grp.refill(qa);  // the current q is always in qa at the top of the body
    if (__all_sync(0xffffffffu, grp.done)) break;
    grp.step(qa, qb);
    grp.step(qb, qa);
  }
}

// Warp-per-rating path (L = 32, k a multiple of 128): one rating group per warp, so
// every branch is warp-uniform and a task is a plain counted loop (no lock step, no
// per-step liveness predicates).  Same pipeline as Group: rating j+1's record and
// q row are in flight while rating j is updated.
// DET slab wavefront: p_u copy distance (ratings) and ring slots (> distance, power of 2)
#ifndef HCCMF_POLL_NS  // the slab wavefront's pause between polls of its predecessor's counter
#define HCCMF_POLL_NS 64
#endif
constexpr unsigned kPollNs = HCCMF_POLL_NS;
#ifndef HCCMF_SLAB_D  // diagnostic builds may move the p_u copy distance (< 16)
#define HCCMF_SLAB_D 12
#endif
constexpr int kSlabD = HCCMF_SLAB_D, kSlabRP = 16;

template <int VEC, bool ATOMIC>
struct WarpSgd {
  static constexpr unsigned FM = 0xffffffffu;
  const SgdArgs& a;
  int lane, k4;
  float g, c1, ngl;
  const float4* __restrict__ Pb;
  const float4* __restrict__ Qb;
  const char* Qhb;  // binary16 Q (storage = 1): lane's 4 halves of slot 0

  __device__ WarpSgd(const SgdArgs& args) : a(args) {
    lane = threadIdx.x & 31;
    k4 = a.k >> 2;
    g = a.gamma;
    c1 = 1.f - a.gamma * a.lambda;
    ngl = -a.gamma * a.lambda;
    Pb = reinterpret_cast<const float4*>(a.P) + lane - (int64_t)a.row0 * k4;
    Qb = reinterpret_cast<const float4*>(a.Q) + lane;
    Qhb = reinterpret_cast<const char*>(a.Q) + lane * 8;
  }
  // 32-bit row offsets: m_local * k/4 and n * k/4 < 2^31
  __device__ __forceinline__ const float4* prow(int u) const {
    return reinterpret_cast<const float4*>(reinterpret_cast<const char*>(Pb) +
                                           (unsigned long long)(unsigned)u * (unsigned)(k4 * 16));
  }
  __device__ __forceinline__ const float4* qrow(int v) const {
    return reinterpret_cast<const float4*>(reinterpret_cast<const char*>(Qb) +
                                           (unsigned long long)(unsigned)v * (unsigned)(k4 * 16));
  }
  __device__ __forceinline__ void ld(const float4* r, float4 (&x)[VEC]) const {
#pragma unroll
    for (int i = 0; i < VEC; ++i) x[i] = __ldcg(r + 32 * i);
  }
  __device__ __forceinline__ void st(const float4* r, const float4 (&x)[VEC]) const {
#pragma unroll
    for (int i = 0; i < VEC; ++i) __stcg(const_cast<float4*>(r) + 32 * i, x[i]);
  }
  // the same store, performed only if `go` (predicated: no branch)
  __device__ __forceinline__ void st_if(const float4* r, const float4 (&x)[VEC], bool go) const {
#pragma unroll
    for (int i = 0; i < VEC; ++i)
      asm volatile("{\n\t.reg .pred P;\n\tsetp.ne.b32 P, %5, 0;\n\t@P st.global.cg.v4.f32 [%0], {%1, %2, %3, %4};\n\t}" ::"l"(
                       r + 32 * i),
                   "f"(x[i].x), "f"(x[i].y), "f"(x[i].z), "f"(x[i].w), "r"((int)go)
                   : "memory");
  }

  // bulk L2 prefetch of one rating's p_u and q_v rows (cp.async.bulk.prefetch, sm_90+)
  __device__ __forceinline__ void prefetch_rows(int u, int v) const {
    const unsigned bytes = (unsigned)k4 * 16u;
    const float4* pr = reinterpret_cast<const float4*>(a.P) + (int64_t)(u - a.row0) * k4;
    const float4* qr = reinterpret_cast<const float4*>(a.Q) + (int64_t)v * k4;
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(pr), "r"(bytes) : "memory");
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(qr), "r"(bytes) : "memory");
  }

  // ---- Hogwild hot loop with a shared-memory record ring ----
  // The warp's next 64 records sit in a per-warp ring of {u, v, r, -} entries filled by
  // cp.async (4-byte copies, one window of 32 records per commit group, one window
  // ahead), so the record of rating j+1 is ONE broadcast LDS.128 instead of three
  // shuffles out of rotating register windows.  Row addresses are formed once with a
  // 32x32->64 multiply-add and carried from the prefetch to the update and the red.
  // q_v row addresses as bytes: fp32 rows of k*4 bytes (lane slot i at +512 i), or
  // binary16 rows of k*2 bytes (QH, storage = 1: lane holds 4 halves = 8 bytes per
  // slot, slot i at +256 i).  The lane offset is folded into the base.
  template <bool QH>
  __device__ __forceinline__ const char* qaddr(int v) const {
    const char* base = QH ? Qhb : reinterpret_cast<const char*>(Qb);
    return base + (unsigned long long)(unsigned)v * (unsigned)(QH ? k4 * 8 : k4 * 16);
  }
  __device__ __forceinline__ const float4* pptr(int u) const {
    return reinterpret_cast<const float4*>(reinterpret_cast<const char*>(Pb) +
                                           (unsigned long long)(unsigned)u * (unsigned)(k4 * 16));
  }
  // q registers hold the row as stored (float4, or 4 binary16 in a uint2 for QH) and are
  // widened only where used, so a prefetched load is not waited on by its conversion
  template <bool QH>
  using QReg = typename std::conditional<QH, uint2, float4>::type;
  template <bool QH>
  static __device__ __forceinline__ float4 widen(const QReg<QH>& x) {
    if constexpr (QH) return h4_to_f4(x); else return x;
  }
  template <bool QH>
  static __device__ __forceinline__ QReg<QH> narrow(const float4& x) {
    if constexpr (QH) return f4_to_h4(x); else return x;
  }
  template <bool QH>
  __device__ __forceinline__ void ldq(const char* q, QReg<QH> (&x)[VEC]) const {
#pragma unroll
    for (int i = 0; i < VEC; ++i) x[i] = __ldcg(reinterpret_cast<const QReg<QH>*>(q + (QH ? 256 : 512) * i));
  }
  template <bool QH>
  __device__ __forceinline__ void stq(const char* q, const QReg<QH> (&x)[VEC]) const {
#pragma unroll
    for (int i = 0; i < VEC; ++i) __stcg(reinterpret_cast<QReg<QH>*>(const_cast<char*>(q) + (QH ? 256 : 512) * i), x[i]);
  }
  // Hogwild!'s component-wise atomic add: red.global.add.v4.f32 (fp32 rows) or
  // red.global.add.noftz.v2.f16x2 of the increment rounded to binary16 (QH)
  template <bool QH>
  __device__ __forceinline__ void redq(const char* q, const QReg<QH> (&d)[VEC]) const {
#pragma unroll
    for (int i = 0; i < VEC; ++i) {
      if constexpr (QH) {
        asm volatile("red.relaxed.gpu.global.add.noftz.v2.f16x2 [%0], {%1, %2};" ::"l"(q + 256 * i), "r"(d[i].x),
                     "r"(d[i].y)
                     : "memory");
      } else {
        asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(q + 512 * i), "f"(d[i].x),
                     "f"(d[i].y), "f"(d[i].z), "f"(d[i].w)
                     : "memory");
      }
    }
  }
  static __device__ __forceinline__ void cp4(const void* dst_smem, const void* src) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(dst_smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(d), "l"(src) : "memory");
  }
  // window w (records 32w .. 32w+31 of the task) -> ring half w & 1
  __device__ __forceinline__ void stage(int4* ring, const int32_t* ru, const int32_t* rv, const float* rr, int w,
                                        int left) const {
    const int idx = w * 32 + lane;
    if (idx < left) {
      int4* e = ring + ((w & 1) << 5) + lane;
      cp4(&e->x, ru + idx);
      cp4(&e->y, rv + idx);
      cp4(&e->z, rr + idx);
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  }
  static __device__ __forceinline__ void wait_all() {
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncwarp();
  }

  template <bool QH, bool SR = false>
  __device__ __forceinline__ void run_ring(int4* ring, int64_t lo, int left) {
    static_assert(!SR || QH, "stochastic rounding needs binary16 storage");
    using QR = QReg<QH>;
    // SR: random word base of rating j = (rec0 + lo + j) * A + t * B (mod 2^32)
    const unsigned rb0 = (unsigned)(a.rec0 + lo) * 0x9E3779B1u + a.epoch * 0x85EBCA77u +
                         (unsigned)(2 * lane) * 0xC2B2AE3Du;
    const int32_t* ru = a.ru + lo;
    const int32_t* rv = a.rv + lo;
    const float* rr = a.rr + lo;
    stage(ring, ru, rv, rr, 0, left);
    wait_all();
    stage(ring, ru, rv, rr, 1, left);  // one window in flight from here on
    int4 rec = ring[0];
    int cu = rec.x, cv = rec.y;
    float cr = __int_as_float(rec.z);
    const float4* pc = pptr(cu);
    const char* qc_p = qaddr<QH>(cv);
    float4 p[VEC], pn[VEC];
    QR qa[VEC], qb[VEC];
    ld(pc, p);
    ldq<QH>(qc_p, qa);

    // one step: update rating j (q in qc_raw at qc_p), prefetch rating j+1 (q into qn)
    auto step = [&](int j, QR (&qc_raw)[VEC], QR (&qn)[VEC], auto has_next_tag, auto may_cross_tag) {
      constexpr bool HAS_NEXT = decltype(has_next_tag)::value;
      constexpr bool MAY_CROSS = decltype(may_cross_tag)::value;
      int nu = 0, nv = 0;
      float nr = 0.f;
      bool fwd = false, newp = false;
      const char* qn_p = qc_p;
      if (HAS_NEXT) {
        const int jn = j + 1;
        if (MAY_CROSS && (jn & 31) == 0) {  // entering window jn/32: it is complete; refill the other half
          wait_all();
          stage(ring, ru, rv, rr, (jn >> 5) + 1, left);
        }
        rec = ring[jn & 63];
        nu = rec.x;
        nv = rec.y;
        nr = __int_as_float(rec.z);
        fwd = nv == cv;
        newp = nu != cu;
        if (!fwd) {
          qn_p = qaddr<QH>(nv);
          ldq<QH>(qn_p, qn);
        }
        if (newp) ld(pptr(nu), pn);
      }
      float4 qc[VEC];
#pragma unroll
      for (int i = 0; i < VEC; ++i) qc[i] = widen<QH>(qc_raw[i]);
      float2 dd = make_float2(0.f, 0.f);
#pragma unroll
      for (int i = 0; i < VEC; ++i) dd = f4_dot2(p[i], qc[i], dd);
      float d = dd.x + dd.y;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(FM, d, o);
      const float ge = g * (cr - d);
      QR w[VEC];  // what is written: the increment (atomic) or the new row (store), as stored
      [[maybe_unused]] QR snew[VEC];  // SR: the new row as stored
#pragma unroll
      for (int i = 0; i < VEC; ++i) {
        if constexpr (SR) {
          // q' = q + dq = c1 q + (g e) p, stochastically rounded to binary16; the atomic
          // increment is q' - q, exact in binary16 (both on q's grid), so a serial run
          // stores exactly q'
          const float4 qq = f4_fma(ge, p[i], f4_scale(c1, qc[i]));
          const unsigned r = rb0 + (unsigned)j * 0x9E3779B1u + (unsigned)(64 * i) * 0xC2B2AE3Du;
          uint2 hs;
          const unsigned w0 = lowbias32(r);  // pair c = 64 i + 2 lane (even); pair c + 1: w0 * 0x9E3779B1
          hs.x = cvt_rs_h2(qq.y, qq.x, w0);
          hs.y = cvt_rs_h2(qq.w, qq.z, w0 * 0x9E3779B1u);
          snew[i] = hs;
          w[i] = ATOMIC ? make_uint2(hsub2_bits(hs.x, qc_raw[i].x), hsub2_bits(hs.y, qc_raw[i].y)) : hs;
        } else {
          const float4 dq = f4_fma(ge, p[i], f4_scale(ngl, qc[i]));
          w[i] = narrow<QH>(ATOMIC ? dq : f4_add(qc[i], dq));
        }
        p[i] = f4_fma(ge, qc[i], f4_scale(c1, p[i]));
      }
      if (ATOMIC)
        redq<QH>(qc_p, w);
      else
        stq<QH>(qc_p, w);
      if (HAS_NEXT) {
        if (fwd) {  // same item next (duplicates): what memory now holds, from registers
#pragma unroll
          for (int i = 0; i < VEC; ++i) {
            if constexpr (SR)
              qn[i] = snew[i];
            else
              qn[i] = ATOMIC ? narrow<QH>(f4_add(qc[i], widen<QH>(w[i]))) : w[i];
          }
        }
        if (newp) {
          st(pc, p);
          pc = pptr(nu);
#pragma unroll
          for (int i = 0; i < VEC; ++i) p[i] = pn[i];
        }
        cu = nu;
        cv = nv;
        cr = nr;
        qc_p = qn_p;
      } else {
        st(pc, p);
      }
    };
    using T = std::true_type;
    using F = std::false_type;
    int j = 0;
#pragma unroll kWarpUnroll
    for (; left - j >= 3; j += 2) {  // j even: only the odd step can enter a new window
      step(j, qa, qb, T{}, F{});
      step(j + 1, qb, qa, T{}, T{});
    }
    if (left - j == 2) {
      step(j, qa, qb, T{}, F{});
      step(j + 1, qb, qa, F{}, F{});
    } else {
      step(j, qa, qb, F{}, F{});
    }
    wait_all();  // no copy may still target the ring when the next task stages
  }

  // all ratings of records [lo, lo + left), left >= 1, in order
  __device__ __forceinline__ void run(int64_t lo, int left) {
    auto ld = [&](const float4* r, float4 (&x)[VEC]) { this->ld(r, x); };
    auto st = [&](const float4* r, const float4 (&x)[VEC]) { this->st(r, x); };
    auto prow = [&](int u) { return this->prow(u); };
    auto qrow = [&](int v) { return this->qrow(v); };
    const int32_t* ru = a.ru + lo;
    const int32_t* rv = a.rv + lo;
    const float* rr = a.rr + lo;
    // double-buffered record windows: lane l holds ratings w*32 + l and w*32 + 32 + l
    int wu0 = 0, wv0 = 0, wu1 = 0, wv1 = 0;
    float wr0 = 0.f, wr1 = 0.f;
    if (lane < left) wu0 = __ldcs(ru + lane), wv0 = __ldcs(rv + lane), wr0 = __ldcs(rr + lane);
    if (lane + 32 < left) wu1 = __ldcs(ru + 32 + lane), wv1 = __ldcs(rv + 32 + lane), wr1 = __ldcs(rr + 32 + lane);
    if (a.prefetch) {  // DET: every rating of the next 64 pulls its p_u / q_v rows into L2 now
      if (lane < left) prefetch_rows(wu0, wv0);
      if (lane + 32 < left) prefetch_rows(wu1, wv1);
    }
    int wb = 0;  // first rating of window 0
    int cu = __shfl_sync(FM, wu0, 0), cv = __shfl_sync(FM, wv0, 0);
    float cr = __shfl_sync(FM, wr0, 0);
    float4 p[VEC], pn[VEC], qa[VEC], qb[VEC];
    ld(prow(cu), p);
    ld(qrow(cv), qa);

    // one step: update rating j (q in qc), prefetch rating j+1 (q into qn); HAS_NEXT static
    auto step = [&](int j, float4 (&qc)[VEC], float4 (&qn)[VEC], auto has_next_tag) {
      constexpr bool HAS_NEXT = decltype(has_next_tag)::value;
      int nu = 0, nv = 0;
      float nr = 0.f;
      bool fwd = false, newp = false;
      if (HAS_NEXT) {
        if (j + 1 - wb == 32) {  // slide the window
          wu0 = wu1, wv0 = wv1, wr0 = wr1;
          wb += 32;
          const int idx = wb + 32 + lane;
          if (idx < left) {
            wu1 = __ldcs(ru + idx), wv1 = __ldcs(rv + idx), wr1 = __ldcs(rr + idx);
            if (a.prefetch) prefetch_rows(wu1, wv1);
          }
        }
        const int src = j + 1 - wb;
        nu = __shfl_sync(FM, wu0, src);
        nv = __shfl_sync(FM, wv0, src);
        nr = __shfl_sync(FM, wr0, src);
        fwd = nv == cv;
        newp = nu != cu;
        if (!fwd) ld(qrow(nv), qn);
        if (newp) ld(prow(nu), pn);
      }
      float2 dd = make_float2(0.f, 0.f);
#pragma unroll
      for (int i = 0; i < VEC; ++i) dd = f4_dot2(p[i], qc[i], dd);
      float d = dd.x + dd.y;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(FM, d, o);
      const float ge = g * (cr - d);
      float4 dq[VEC];
#pragma unroll
      for (int i = 0; i < VEC; ++i) {
        dq[i] = f4_fma(ge, p[i], f4_scale(ngl, qc[i]));
        p[i] = f4_fma(ge, qc[i], f4_scale(c1, p[i]));
      }
      const float4* qw = qrow(cv);
      if (ATOMIC) {
#pragma unroll
        for (int i = 0; i < VEC; ++i)
          asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(qw + 32 * i),
                       "f"(dq[i].x), "f"(dq[i].y), "f"(dq[i].z), "f"(dq[i].w)
                       : "memory");
      } else {
#pragma unroll
        for (int i = 0; i < VEC; ++i) dq[i] = f4_add(qc[i], dq[i]);
        st(qw, dq);
      }
      if (HAS_NEXT) {
        if (fwd) {  // same item next (duplicates): serial read-after-write from registers
#pragma unroll
          for (int i = 0; i < VEC; ++i) qn[i] = ATOMIC ? f4_add(qc[i], dq[i]) : dq[i];
        }
        if (newp) {
          st(prow(cu), p);
#pragma unroll
          for (int i = 0; i < VEC; ++i) p[i] = pn[i];
        }
        cu = nu;
        cv = nv;
        cr = nr;
      } else {
        st(prow(cu), p);
      }
    };
    using T = std::true_type;
    using F = std::false_type;
    int j = 0;
    for (; left - j >= 3; j += 2) {
      step(j, qa, qb, T{});
      step(j + 1, qb, qa, T{});
    }
    if (left - j == 2) {
      step(j, qa, qb, T{});
      step(j + 1, qb, qa, F{});
    } else {
      step(j, qa, qb, F{});
    }
  }

  // DET block with the column block's Q rows resident in shared memory (slab = this
  // warp's copy of rows [c0, c0 + w), lane's slot 0 of row v at slab[(v - c0) k4 + lane]).
  // Nothing else touches those rows while the warp holds the block (disjoint columns
  // within a stratum), so q_v never leaves the SM during the block: every update reads
  // the row from shared memory after the previous update's write (the serial order,
  // duplicates included).  Nothing else touches the block's rows either (the warp owns
  // its row block), and a row's ratings are contiguous in a block (sorted by u'), so the
  // p_u row of every user run is copied D ratings ahead (cp.async, one commit group per
  // rating, wait_group D before use) into a shared-memory ring of RP row slots and
  // written back to HBM when the run ends; a run's row was last written by this warp,
  // before the fence of an earlier block.  Same arithmetic as run() and run_ring(): the
  // factors are bit-identical to the per-stratum launches.
  // Round 2 (C3 DET epoch 45.1 -> 29.3 ms, profiles/r02_det.md).  The block's start is off
  // the wavefront's critical path: the records enter a per-warp shared-memory ring of 4
  // windows of 16 by cp.async (window w + 2 is issued when window w is reached; one LDS.128
  // per rating for the update and one LDS.32 for the p_u copy D ahead, instead of six
  // shuffles out of register windows), and the prologue -- the first windows and the p_u
  // ring fill of the first D ratings, which touch only this warp's own rows -- runs BEFORE
  // wait_load() waits for the predecessor and stages the column block's Q slab.  The last
  // run's p_u row is NOT stored here: it is returned in (last_u, last_p) and the caller
  // stores it after releasing the column block, so the release fence does not wait for it
  // (P rows are this warp's own; the next block's copies follow it in program order).
  template <class WaitLoad>
  __device__ __forceinline__ void run_slab_ring(int64_t lo, int left, float4* slab, int c0, float4* pring, int4* ring,
                                                WaitLoad&& wait_load, int& last_u, float4 (&last_p)[VEC]) {
    constexpr int D = kSlabD, RP = kSlabRP;
    static_assert(RP > D && (RP & (RP - 1)) == 0 && D < 16, "ring: window w + 1 lands before window w is reached");
    const int32_t* ru = a.ru + lo;
    const int32_t* rv = a.rv + lo;
    const float* rr = a.rr + lo;
    auto issue = [&](int w) {  // window w -> ring quarter w & 3 (lane l < 16: record 16 w + l)
      const int idx = w * 16 + lane;
      if (lane < 16 && idx < left) {
        int4* e = ring + ((w & 3) << 4) + lane;
        cp4(&e->x, ru + idx);
        cp4(&e->y, rv + idx);
        cp4(&e->z, rr + idx);
      }
    };
    float4* const sb = slab + lane - (int64_t)c0 * k4;
    float4* const pb = pring + lane;
    auto copy_p = [&](int slot, int u) {  // p_u -> ring slot (this lane's VEC 16-byte pieces)
      const float4* src = prow(u);
#pragma unroll
      for (int i = 0; i < VEC; ++i) {
        const unsigned d = (unsigned)__cvta_generic_to_shared(pb + slot * k4 + 32 * i);
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src + 32 * i) : "memory");
      }
    };
    // the same copy, issued only if `go` (a predicated cp.async: no branch in the loop)
    auto copy_p_if = [&](int slot, int u, bool go) {
      const float4* src = prow(u);
#pragma unroll
      for (int i = 0; i < VEC; ++i) {
        const unsigned d = (unsigned)__cvta_generic_to_shared(pb + slot * k4 + 32 * i);
        asm volatile("{\n\t.reg .pred P;\n\tsetp.ne.b32 P, %2, 0;\n\t@P cp.async.cg.shared.global [%0], [%1], 16;\n\t}" ::"r"(d),
                     "l"(src + 32 * i), "r"((int)go)
                     : "memory");
      }
    };
    // window w reached (w >= 1): windows w and w + 1 have landed (their groups are older
    // than rating j - 1's); w + 1's users' p rows go to L2, window w + 2 is issued
    auto boundary = [&](int w) {
      __syncwarp();
      if (lane < 16 && (w + 1) * 16 + lane < left) prefetch_p(ring[(((w + 1) & 3) << 4) + lane].x);
      issue(w + 2);
    };
    issue(0);
    issue(1);
    asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
    __syncwarp();
    if (lane < 16 && 16 + lane < left) prefetch_p(ring[16 + lane].x);  // window 0: the kernel's look-ahead did it
    issue(2);
    int lastu = -1;
    for (int s = 0; s < D; ++s) {
      if (s < left) {
        const int u = ring[s].x;
        if (u != lastu) copy_p(s & (RP - 1), u);
        lastu = u;
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
    }
    wait_load();  // predecessor done; the slab (and, by wait_group 0, the ring fill) landed
    int cu = -1;  // user whose row is in p
    float4 p[VEC], q[VEC];
    int4 rc = ring[0];       // rating j's record, read one rating ahead (off the q_v chain)
    int un = ring[D].x;      // the user of rating j + D, read one rating ahead as well
    // Issue order matters (one warp issues in order, and on the wavefront's critical path
    // it is alone): rating j's operands are requested first, the look-ahead of rating
    // j + D (compare, predicated p_u copy, commit) sits between the reduction's first two
    // levels, and the next look-ahead's user is read right after this rating's q_v write
    // (a window boundary is handled one rating early so that read always finds it).
#pragma unroll 2
    for (int j = 0; j < left; ++j) {
      const int u = rc.x, v = rc.y;
      const float r = __int_as_float(rc.z);
#ifndef HCCMF_DIAG_NO_DEPBAR
      // groups 0 .. j + D - 1 are committed: at most D - 1 pending = rating j's copy landed
      asm volatile("cp.async.wait_group %0;" ::"n"(D - 1) : "memory");
#endif
      float4* qw = sb + v * k4;
#pragma unroll
      for (int i = 0; i < VEC; ++i) q[i] = qw[32 * i];  // after the previous write: serial order
      {  // a run starts: retire the previous user's row, take this one's (branch-free: every
         // rating's row was copied; inside a run the registers hold the current row)
        const bool newrun = u != cu;
        float4 pr[VEC];
#pragma unroll
        for (int i = 0; i < VEC; ++i) pr[i] = pb[(j & (RP - 1)) * k4 + 32 * i];
        st_if(prow(cu < 0 ? u : cu), p, newrun && cu >= 0);
#pragma unroll
        for (int i = 0; i < VEC; ++i) p[i] = newrun ? pr[i] : p[i];
        cu = u;
      }
      if (j + 1 < left) rc = ring[(j + 1) & 63];  // visible since its window's boundary (j + 1 < j + D)
      float2 dd = make_float2(0.f, 0.f);
#pragma unroll
      for (int i = 0; i < VEC; ++i) dd = f4_dot2(p[i], q[i], dd);
      float d = dd.x + dd.y;
#ifdef HCCMF_DIAG_SHFL_LEVELS  // diagnostic builds only: fewer reduction levels (wrong factors)
      for (int o = 1 << (HCCMF_DIAG_SHFL_LEVELS - 1); o > 0; o >>= 1) {
#else
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
#endif
        d += __shfl_xor_sync(FM, d, o);
        if (o == 16) {  // look-ahead of rating j + D: its user's p_u copy, one commit group
          const int jn = j + D;
          const bool go = jn < left;
          copy_p_if(jn & (RP - 1), un, go);
          asm volatile("cp.async.commit_group;" ::: "memory");
        }
      }
      const float ge = g * (r - d);
#pragma unroll
      for (int i = 0; i < VEC; ++i) {
        const float4 dq = f4_fma(ge, p[i], f4_scale(ngl, q[i]));
        p[i] = f4_fma(ge, q[i], f4_scale(c1, p[i]));
        qw[32 * i] = f4_add(q[i], dq);
      }
      const int jn1 = j + 1 + D;  // the next look-ahead's rating
      if (jn1 < left && (jn1 & 15) == 0) boundary(jn1 >> 4);
      un = ring[jn1 & 63].x;  // beyond the block: a stale entry, never copied
    }
    last_u = cu;
#pragma unroll
    for (int i = 0; i < VEC; ++i) last_p[i] = p[i];
    asm volatile("cp.async.wait_group 0;" ::: "memory");  // nothing may still target the rings
    __syncwarp();  // the record ring is rewritten by the next block's prologue
  }

  // L2 prefetch of one p_u row by the calling lane, line by line (a bulk prefetch takes a
  // uniform operand: one per lane would be a 32-way serialised loop)
  __device__ __forceinline__ void prefetch_p(int u) const {
    const char* pr = reinterpret_cast<const char*>(reinterpret_cast<const float4*>(a.P) + (int64_t)(u - a.row0) * k4);
    for (int o = 0; o < k4 * 16; o += 128) asm volatile("prefetch.global.L2 [%0];" ::"l"(pr + o));
  }

  // Deeper pipeline (D >= 2, Hogwild): the q row of rating j + D is requested while
  // rating j is updated, from a ring of D + 1 register rows (the loop is unrolled
  // D + 1 times so every slot index is static).  Every pending row whose load was
  // issued before this warp's own update of the same item gets the increment added
  // in registers, so one warp alone is exactly serial; p_u keeps the 1-deep prefetch
  // (a user change is rare next to a rating).
  template <int D>
  __device__ __forceinline__ void run_deep(int64_t lo, int left) {
    constexpr int R = D + 1;
    const int32_t* ru = a.ru + lo;
    const int32_t* rv = a.rv + lo;
    const float* rr = a.rr + lo;
    int wu0 = 0, wv0 = 0, wu1 = 0, wv1 = 0;
    float wr0 = 0.f, wr1 = 0.f;
    if (lane < left) wu0 = __ldcs(ru + lane), wv0 = __ldcs(rv + lane), wr0 = __ldcs(rr + lane);
    if (lane + 32 < left) wu1 = __ldcs(ru + 32 + lane), wv1 = __ldcs(rv + 32 + lane), wr1 = __ldcs(rr + 32 + lane);
    int wb = 0;
    int su[R], sv[R];
    float sr[R];
    float4 q[R][VEC], p[VEC], pn[VEC];
#pragma unroll
    for (int s = 0; s < R; ++s) {
      su[s] = sv[s] = 0;
      sr[s] = 0.f;
    }
#pragma unroll
    for (int s = 0; s < D; ++s) {
      if (s < left) {
        su[s] = __shfl_sync(FM, wu0, s);
        sv[s] = __shfl_sync(FM, wv0, s);
        sr[s] = __shfl_sync(FM, wr0, s);
        ld(qrow(sv[s]), q[s]);
      }
    }
    ld(prow(su[0]), p);
    for (int j0 = 0; j0 < left; j0 += R) {
#pragma unroll
      for (int c = 0; c < R; ++c) {
        const int j = j0 + c;
        if (j >= left) break;
        const int ns = (c + D) % R;  // slot of rating j + D
        const int jn = j + D;
        if (jn < left) {
          if (jn - wb == 32) {  // slide the record window
            wu0 = wu1, wv0 = wv1, wr0 = wr1;
            wb += 32;
            const int idx = wb + 32 + lane;
            if (idx < left) wu1 = __ldcs(ru + idx), wv1 = __ldcs(rv + idx), wr1 = __ldcs(rr + idx);
          }
          const int src = jn - wb;
          su[ns] = __shfl_sync(FM, wu0, src);
          sv[ns] = __shfl_sync(FM, wv0, src);
          sr[ns] = __shfl_sync(FM, wr0, src);
          ld(qrow(sv[ns]), q[ns]);
        }
        const int cn = (c + 1) % R;
        const bool has_next = j + 1 < left;
        const bool newp = has_next && su[cn] != su[c];
        if (newp) ld(prow(su[cn]), pn);
        float2 dd = make_float2(0.f, 0.f);
#pragma unroll
        for (int i = 0; i < VEC; ++i) dd = f4_dot2(p[i], q[c][i], dd);
        float d = dd.x + dd.y;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(FM, d, o);
        const float ge = g * (sr[c] - d);
        float4 dq[VEC];
#pragma unroll
        for (int i = 0; i < VEC; ++i) {
          dq[i] = f4_fma(ge, p[i], f4_scale(ngl, q[c][i]));
          p[i] = f4_fma(ge, q[c][i], f4_scale(c1, p[i]));
        }
        const float4* qw = qrow(sv[c]);
        if (ATOMIC) {
#pragma unroll
          for (int i = 0; i < VEC; ++i)
            asm volatile("red.relaxed.gpu.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(qw + 32 * i),
                         "f"(dq[i].x), "f"(dq[i].y), "f"(dq[i].z), "f"(dq[i].w)
                         : "memory");
        } else {
#pragma unroll
          for (int i = 0; i < VEC; ++i) dq[i] = f4_add(q[c][i], dq[i]);
          st(qw, dq);
        }
        // pending rows j+1 .. j+D were all requested before this update
#pragma unroll
        for (int t = 1; t <= D; ++t) {
          const int s = (c + t) % R;
          if (j + t < left && sv[s] == sv[c]) {
#pragma unroll
            for (int i = 0; i < VEC; ++i) q[s][i] = ATOMIC ? f4_add(q[s][i], dq[i]) : dq[i];
          }
        }
        if (!has_next || newp) {
          st(prow(su[c]), p);
          if (newp) {
#pragma unroll
            for (int i = 0; i < VEC; ++i) p[i] = pn[i];
          }
        }
      }
    }
  }
};

// ---- Hogwild for k = 32 / 64 (C2): one rating per warp, lane l holds E = k/32
// consecutive floats of p_u and q_v (one coalesced 4- or 8-byte access per lane; a row is
// 128 / 256 B).  Why not the lane-group kernel (k/4 lanes per rating, 32/L ratings in
// lock step): it waits on every q_v load one rating ahead, so a heavy user's run -- one
// task, serial through p_u -- advanced at ~one L2 round trip per rating and formed the
// epoch's tail (C2's heaviest user has 5,919 ratings).  Here q_v is requested D ratings
// ahead from a register ring (the run_deep scheme: rows loaded before this warp's own
// update of the same item get the increment in registers, so one warp alone is serial),
// and a run advances at the latency of its dot-product chain.
template <int E, bool ATOMIC>
struct NarrowSgd {
  static constexpr unsigned FM = 0xffffffffu;
  const SgdArgs& a;
  int lane, k;
  float g, c1, ngl;
  const float* Pb;
  const float* Qb;
  __device__ NarrowSgd(const SgdArgs& args) : a(args) {
    lane = threadIdx.x & 31;
    k = a.k;
    g = a.gamma;
    c1 = 1.f - a.gamma * a.lambda;
    ngl = -a.gamma * a.lambda;
    Pb = a.P + lane * E - (int64_t)a.row0 * k;
    Qb = a.Q + lane * E;
  }
  // row addresses with one 32x32->64 multiply-add (ids are non-negative and < 2^31)
  __device__ __forceinline__ const float* prow(int u) const {
    return reinterpret_cast<const float*>(reinterpret_cast<const char*>(Pb) +
                                          (unsigned long long)(unsigned)u * (unsigned)(k * 4));
  }
  __device__ __forceinline__ const float* qrow(int v) const {
    return reinterpret_cast<const float*>(reinterpret_cast<const char*>(Qb) +
                                          (unsigned long long)(unsigned)v * (unsigned)(k * 4));
  }
  static __device__ __forceinline__ void ld(const float* r, float (&x)[E]) {
    if constexpr (E == 1) {
      x[0] = __ldcg(r);
    } else {
      const float2 t = __ldcg(reinterpret_cast<const float2*>(r));
      x[0] = t.x, x[1] = t.y;
    }
  }
  static __device__ __forceinline__ void st(const float* r, const float (&x)[E]) {
    if constexpr (E == 1)
      __stcg(const_cast<float*>(r), x[0]);
    else
      __stcg(reinterpret_cast<float2*>(const_cast<float*>(r)), make_float2(x[0], x[1]));
  }
  static __device__ __forceinline__ void red(const float* r, const float (&x)[E]) {
    if constexpr (E == 1)
      asm volatile("red.relaxed.gpu.global.add.f32 [%0], %1;" ::"l"(r), "f"(x[0]) : "memory");
    else
      asm volatile("red.relaxed.gpu.global.add.v2.f32 [%0], {%1, %2};" ::"l"(r), "f"(x[0]), "f"(x[1]) : "memory");
  }

  template <int D>
  __device__ __forceinline__ void run(int64_t lo, int left) {
    constexpr int R = D + 1;
    const int32_t* ru = a.ru + lo;
    const int32_t* rv = a.rv + lo;
    const float* rr = a.rr + lo;
    int wu0 = 0, wv0 = 0, wu1 = 0, wv1 = 0;
    float wr0 = 0.f, wr1 = 0.f;
    if (lane < left) wu0 = __ldcs(ru + lane), wv0 = __ldcs(rv + lane), wr0 = __ldcs(rr + lane);
    if (lane + 32 < left) wu1 = __ldcs(ru + 32 + lane), wv1 = __ldcs(rv + 32 + lane), wr1 = __ldcs(rr + 32 + lane);
    int wb = 0;
    int su[R], sv[R];
    float sr[R];
    float q[R][E], p[E], pn[E];
#pragma unroll
    for (int s = 0; s < R; ++s) {
      su[s] = sv[s] = 0;
      sr[s] = 0.f;
    }
#pragma unroll
    for (int s = 0; s < D; ++s) {
      if (s < left) {
        su[s] = __shfl_sync(FM, wu0, s);
        sv[s] = __shfl_sync(FM, wv0, s);
        sr[s] = __shfl_sync(FM, wr0, s);
        ld(qrow(sv[s]), q[s]);
      }
    }
    ld(prow(su[0]), p);
#pragma unroll kNarrowUnroll
    for (int j0 = 0; j0 < left; j0 += R) {
#pragma unroll
      for (int c = 0; c < R; ++c) {
        const int j = j0 + c;
        if (j >= left) break;
        const int ns = (c + D) % R;  // slot of rating j + D
        const int jn = j + D;
        if (jn < left) {
          if (jn - wb == 32) {  // slide the record window
            wu0 = wu1, wv0 = wv1, wr0 = wr1;
            wb += 32;
            const int idx = wb + 32 + lane;
            if (idx < left) wu1 = __ldcs(ru + idx), wv1 = __ldcs(rv + idx), wr1 = __ldcs(rr + idx);
          }
          const int src = jn - wb;
          su[ns] = __shfl_sync(FM, wu0, src);
          sv[ns] = __shfl_sync(FM, wv0, src);
          sr[ns] = __shfl_sync(FM, wr0, src);
          ld(qrow(sv[ns]), q[ns]);
        }
        const int cn = (c + 1) % R;
        const bool has_next = j + 1 < left;
        const bool newp = has_next && su[cn] != su[c];
        if (newp) ld(prow(su[cn]), pn);
        float d = p[0] * q[c][0];
#pragma unroll
        for (int e = 1; e < E; ++e) d = fmaf(p[e], q[c][e], d);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) d += __shfl_xor_sync(FM, d, o);
        const float ge = g * (sr[c] - d);
        float dq[E];
#pragma unroll
        for (int e = 0; e < E; ++e) {
          dq[e] = fmaf(ge, p[e], ngl * q[c][e]);
          p[e] = fmaf(ge, q[c][e], c1 * p[e]);
        }
        const float* qw = qrow(sv[c]);
        if (ATOMIC) {
          red(qw, dq);
        } else {
#pragma unroll
          for (int e = 0; e < E; ++e) dq[e] = q[c][e] + dq[e];
          st(qw, dq);
        }
        // pending rows j+1 .. j+D were all requested before this update
#pragma unroll
        for (int t = 1; t <= D; ++t) {
          const int s2 = (c + t) % R;
          if (j + t < left && sv[s2] == sv[c]) {
#pragma unroll
            for (int e = 0; e < E; ++e) q[s2][e] = ATOMIC ? q[s2][e] + dq[e] : dq[e];
          }
        }
        if (!has_next || newp) {
          st(prow(su[c]), p);
          if (newp) {
#pragma unroll
            for (int e = 0; e < E; ++e) p[e] = pn[e];
          }
        }
      }
    }
  }
};

template <int E, bool ATOMIC, int D>
__global__ void __launch_bounds__(kThreads) sgd_narrow_kernel(SgdArgs a) {
  constexpr unsigned FM = 0xffffffffu;
  NarrowSgd<E, ATOMIC> w(a);
  unsigned long long tn = 0;
  if (w.lane == 0) tn = atomicAdd(a.counter, 1ull);
  tn = __shfl_sync(FM, tn, 0);
  while (tn < (unsigned long long)a.n_tasks) {
    const int64_t lo = a.task_lo[tn];
    const int left = (int)(a.task_hi[tn] - lo);
    unsigned long long tn2 = 0;
    if (w.lane == 0) tn2 = atomicAdd(a.counter, 1ull);  // next task id, fetched one task ahead
    w.template run<D>(lo, left);
    tn = __shfl_sync(FM, tn2, 0);
  }
}

#ifndef HCCMF_WARP_MINB
#define HCCMF_WARP_MINB 1
#endif
template <int VEC, bool ATOMIC, int D, int QM>  // QM: 0 fp32 Q, 1 binary16 RN, 2 binary16 SR
__global__ void __launch_bounds__(kThreads, (VEC == 1 ? HCCMF_WARP_MINB1 : HCCMF_WARP_MINB)) sgd_warp_kernel(SgdArgs a) {
  constexpr unsigned FM = 0xffffffffu;
  WarpSgd<VEC, ATOMIC> w(a);
  __shared__ int4 sring[kThreads / 32][64];
  int4* ring = sring[threadIdx.x >> 5];
  unsigned long long tn = 0;
  if (w.lane == 0) tn = atomicAdd(a.counter, 1ull);
  tn = __shfl_sync(FM, tn, 0);
  while (tn < (unsigned long long)a.n_tasks) {
    const int64_t lo = a.task_lo[tn];
    const int left = (int)(a.task_hi[tn] - lo);
    unsigned long long tn2 = 0;
    if (w.lane == 0) tn2 = atomicAdd(a.counter, 1ull);  // next task id, fetched one task ahead
    if (D == 1 && QM == 2)
      w.template run_ring<true, true>(ring, lo, left);
    else if (D == 1 && QM == 1)
      w.template run_ring<true>(ring, lo, left);
    else if (D == 1)
      w.template run_ring<false>(ring, lo, left);
    else
      w.template run_deep<D>(lo, left);
    tn = __shfl_sync(FM, tn2, 0);
  }
}

// DET as a wavefront (a5): warp i owns row block i and walks its blocks
// (i, (i+t) mod B) for t = 0..B-1.  Column block (i+t) mod B was last updated by
// row block i+1 at stratum t-1, so warp i waits only for warp i+1's progress
// counter (release/acquire through L2) instead of a grid-wide barrier per stratum;
// the order of updates on every P row and Q row is the strata order of R19.
// All B warps must be co-resident (checked by the launcher).
template <int VEC>
__global__ void __launch_bounds__(kThreads) sgd_wave_kernel(SgdArgs a, const int64_t* __restrict__ off, int B,
                                                            int* progress) {
  // row block i on CTA i mod CTAs, as in sgd_wave_slab_kernel
  const int i = (int)((threadIdx.x >> 5) * gridDim.x + blockIdx.x);
  if (i >= B) return;
  WarpSgd<VEC, false> w(a);
  const int nb = (i + 1) % B;
  for (int t = 0; t < B; ++t) {
    if (t > 0 && B > 1) {
      if (w.lane == 0) {
        int seen;
        do {
          // relaxed polling (an acquire load per poll invalidates the SM's L1 every
          // time: CCTL.IVALL), one acquire fence once the predecessor is seen
          asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(seen) : "l"(progress + (int64_t)nb * kProgressStride) : "memory");
          if (seen < t) __nanosleep(64);
        } while (seen < t);
        // acquire pattern (relaxed read + fence.acquire: CCTL.IVALL, no MEMBAR -- a full
        // fence here would also wait for this warp's own outstanding copies and prefetches)
        asm volatile("fence.acquire.gpu;" ::: "memory");
      }
      __syncwarp();
    }
    const int64_t blk = (int64_t)i * B + (i + t) % B;
    const int64_t lo = off[blk], hi = off[blk + 1];
    if (hi > lo) w.run(lo, (int)(hi - lo));
    __syncwarp();
    if (w.lane == 0) {
      asm volatile("fence.release.gpu;" ::: "memory");  // the warp's writes (ordered by __syncwarp) first
      asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(progress + (int64_t)i * kProgressStride), "r"(t + 1) : "memory");
    }
  }
}

// The same wavefront with the column block's Q rows staged in shared memory
// (WarpSgd::run_slab_ring): per block, the w <= wmax rows of column block c are copied in
// with cp.async (one L2 round trip for the whole slab instead of one per rating),
// updated in place, and written back before the progress counter is released.  The
// next block's records are bulk-prefetched into L2 while this block runs.
// Column block c holds v' with floor(v' B / n) = c, i.e. v' in [ceil(c n / B), ceil((c+1) n / B)).
#ifdef HCCMF_DIAG_TRACE  // diagnostic builds only: %globaltimer stamps per (warp, stratum)
__device__ unsigned g_wave_trace[2048 * 2048 * 3];
__device__ __forceinline__ unsigned gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return (unsigned)t;
}
#endif

template <int VEC>
__global__ void __launch_bounds__(kThreads, 2) sgd_wave_slab_kernel(SgdArgs a, const int64_t* __restrict__ off, int B,
                                                                 int* progress, int64_t n, int wmax) {
  extern __shared__ float4 wave_smem[];
  // row block i -> warp i / CTAs of CTA i mod CTAs: successive row blocks, which hand the
  // column blocks on to each other, run on different SMs rather than sharing one SM's
  // schedulers (C3, B = 2048: 71.5 -> 69.5 ms per step).  Waits go through progress[],
  // so the mapping does not change the order of updates.
  const int i = (int)((threadIdx.x >> 5) * gridDim.x + blockIdx.x);
  if (i >= B) return;
  WarpSgd<VEC, false> w(a);
  const int k4 = a.k >> 2;
  // per warp: the column block's slab (wmax rows), then the p_u ring (kSlabRP rows)
  float4* slab = wave_smem + (int64_t)(threadIdx.x >> 5) * (wmax + kSlabRP) * k4;
  float4* pring = slab + (int64_t)wmax * k4;
  // the per-warp record rings (64 entries) after all warps' slabs and p rings
  int4* rring = reinterpret_cast<int4*>(wave_smem + (int64_t)(blockDim.x >> 5) * (wmax + kSlabRP) * k4) +
                (threadIdx.x >> 5) * 64;
  const float4* Qg = reinterpret_cast<const float4*>(a.Q);
  float4* Qw = reinterpret_cast<float4*>(a.Q);
  const int nb = (i + 1) % B;
  auto prefetch_records = [&](int64_t lo, int64_t hi) {
    if (hi <= lo || w.lane > 2) return;
    const char* base = w.lane == 0 ? reinterpret_cast<const char*>(a.ru)
                                   : (w.lane == 1 ? reinterpret_cast<const char*>(a.rv)
                                                  : reinterpret_cast<const char*>(a.rr));
    const uintptr_t b0 = reinterpret_cast<uintptr_t>(base + 4 * lo) & ~(uintptr_t)15;
    const uintptr_t b1 = (reinterpret_cast<uintptr_t>(base + 4 * hi) + 15) & ~(uintptr_t)15;
    const unsigned bytes = (unsigned)min((uintptr_t)(1u << 20), b1 - b0);
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(b0), "r"(bytes) : "memory");
  };
  const int64_t* row_off = off + (int64_t)i * B;  // block (i, c) = row_off[c] .. row_off[c + 1]
  int last_u = -1;
  float4 last_p[VEC];
  prefetch_records(row_off[i], row_off[i + 1]);
  if (B > 1) prefetch_records(row_off[(i + 1) % B], row_off[(i + 1) % B + 1]);
  for (int t = 0; t < B; ++t) {
    const int c = (i + t) % B;
    const int64_t lo = row_off[c], hi = row_off[c + 1];
    // look-ahead while the predecessor finishes: block t+2's records into L2, and the p_u
    // rows of block t+1's first 64 ratings (its records are in L2 since the last block)
    if (t + 2 < B) {
      const int c2 = (i + t + 2) % B;
      prefetch_records(row_off[c2], row_off[c2 + 1]);
    }
    int nu0 = -1, nu1 = -1;
    if (t + 1 < B) {
      const int c1n = (i + t + 1) % B;
      const int64_t nlo = row_off[c1n], nn = row_off[c1n + 1] - nlo;
      if (w.lane < nn) nu0 = __ldcg(a.ru + nlo + w.lane);
      if (w.lane + 32 < nn) nu1 = __ldcg(a.ru + nlo + 32 + w.lane);
    }
    // the predecessor's release of column block c, then c's Q rows -> slab (cp.async)
    const int c0 = (int)(((int64_t)c * n + B - 1) / B);
    const int rows = (int)(((int64_t)(c + 1) * n + B - 1) / B) - c0;
    auto wait_load = [&]() {
#ifdef HCCMF_DIAG_TRACE
      if (w.lane == 0 && B <= 2048) g_wave_trace[((int64_t)i * B + t) * 3] = gtimer();
#endif
#ifndef HCCMF_DIAG_NOWAIT  // diagnostic builds only: no dependency waits (wrong factors, timing bound)
      if (t > 0 && B > 1) {
        if (w.lane == 0) {
          int seen;
          do {
            // relaxed polling (an acquire load per poll invalidates the SM's L1 every
            // time: CCTL.IVALL), one acquire fence once the predecessor is seen
            asm volatile("ld.relaxed.gpu.global.s32 %0, [%1];" : "=r"(seen) : "l"(progress + (int64_t)nb * kProgressStride) : "memory");
            if (seen < t && kPollNs) __nanosleep(kPollNs);
          } while (seen < t);
          // acquire pattern (relaxed read + fence.acquire: CCTL.IVALL, no MEMBAR -- a full
          // fence here would also wait for this warp's own outstanding copies and prefetches)
          asm volatile("fence.acquire.gpu;" ::: "memory");
        }
        __syncwarp();
      }
#endif
#ifdef HCCMF_DIAG_TRACE
      if (w.lane == 0 && B <= 2048) g_wave_trace[((int64_t)i * B + t) * 3 + 1] = gtimer();
#endif
      if (hi > lo) {
        for (int r = 0; r < rows; ++r) {
#pragma unroll
          for (int s = 0; s < VEC; ++s) {
            const unsigned d = (unsigned)__cvta_generic_to_shared(slab + r * k4 + w.lane + 32 * s);
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d),
                         "l"(Qg + (int64_t)(c0 + r) * k4 + w.lane + 32 * s)
                         : "memory");
          }
        }
        asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
      }
      // the next block's first 64 users' p_u rows -> L2 (its prologue copies hit there)
      if (nu0 >= 0) w.prefetch_p(nu0);
      if (nu1 >= 0) w.prefetch_p(nu1);
    };
    if (hi > lo) {
      w.run_slab_ring(lo, (int)(hi - lo), slab, c0, pring, rring, wait_load, last_u, last_p);
      for (int r = 0; r < rows; ++r) {
#pragma unroll
        for (int s = 0; s < VEC; ++s)
          __stcg(Qw + (int64_t)(c0 + r) * k4 + w.lane + 32 * s, slab[r * k4 + w.lane + 32 * s]);
      }
    } else {
      wait_load();
    }
    __syncwarp();
    if (w.lane == 0) {
      asm volatile("fence.release.gpu;" ::: "memory");  // the warp's writes (ordered by __syncwarp) first
      asm volatile("st.relaxed.gpu.global.s32 [%0], %1;" ::"l"(progress + (int64_t)i * kProgressStride), "r"(t + 1) : "memory");
#ifdef HCCMF_DIAG_TRACE
      if (B <= 2048) g_wave_trace[((int64_t)i * B + t) * 3 + 2] = gtimer();
#endif
    }
    if (last_u >= 0) {  // the block's last p_u run, after the release (see run_slab_ring)
      w.st(w.prow(last_u), last_p);
      last_u = -1;
    }
  }
}

template <int L, int VEC, bool FULL>
cudaError_t launch_t(const SgdArgs& a, int64_t warps, cudaStream_t st) {
  constexpr int groups_per_warp = 32 / L;
  int64_t need_warps = (a.n_tasks + groups_per_warp - 1) / groups_per_warp;
  int64_t w = warps < need_warps ? warps : need_warps;
  if (w < 1) return cudaSuccess;
  // exactly w warps when w < 8 (one partial CTA), else whole CTAs of 8 warps
  const int threads = w < kThreads / 32 ? (int)w * 32 : kThreads;
  const int64_t blocks = (w * 32 + threads - 1) / threads;
  if (L == 32 && FULL) {  // warp-per-rating specialisation
    const int depth = a.depth < 1 ? 1 : a.depth;  // auto: one rating ahead
#define WARP_CASE(DD, QQ)                                                     \
  if (depth == DD && a.qhalf == QQ) {                                         \
    if (a.atomic_q)                                                           \
      (note_launch(), sgd_warp_kernel<VEC, true, DD, QQ><<<(unsigned)blocks, threads, 0, st>>>(a));  \
    else                                                                      \
      (note_launch(), sgd_warp_kernel<VEC, false, DD, QQ><<<(unsigned)blocks, threads, 0, st>>>(a)); \
    return cudaGetLastError();                                                \
  }
    WARP_CASE(1, 0) WARP_CASE(2, 0) WARP_CASE(3, 0) WARP_CASE(4, 0) WARP_CASE(1, 1) WARP_CASE(1, 2)
#undef WARP_CASE
    return cudaErrorInvalidValue;
  }
  if (a.qhalf) return cudaErrorInvalidValue;  // binary16 Q: warp-per-rating geometry only
  if (a.atomic_q)
    (note_launch(), sgd_kernel<L, VEC, FULL, true><<<(unsigned)blocks, threads, 0, st>>>(a));
  else
    (note_launch(), sgd_kernel<L, VEC, FULL, false><<<(unsigned)blocks, threads, 0, st>>>(a));
  return cudaGetLastError();
}

}  // namespace

// Lane geometry: VEC float4 slots per lane, L lanes per rating group.  Auto: one
// rating per warp (L = 32) once k >= 128 (k = 128: VEC = 1, k = 256: 2, k = 512: 4),
// the warp-per-rating kernel; below, L = k/4 lanes and 32/L groups per warp in lock
// step.  At equal rating groups in flight (equal Hogwild staleness) one group per
// warp was fastest on C3 (tools/sweep_hogwild.py: 7.7 vs 5.8 G upd/s).
void sgd_geometry(int k, int vec_pref, int* L_out, int* VEC_out) {
  const int c4 = k / 4;
  int vec = vec_pref > 0 ? vec_pref : std::max(1, std::min(4, c4 / 32));
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

bool wave_supported(int k, int vec_pref, int B) {
  int L, VEC;
  sgd_geometry(k, vec_pref, &L, &VEC);
  if (L != 32 || L * VEC * 4 != k) return false;
  int dev = 0, sms = 0, per_sm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaError_t e = cudaSuccess;
  switch (VEC) {
    case 1: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, sgd_wave_kernel<1>, kThreads, 0); break;
    case 2: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, sgd_wave_kernel<2>, kThreads, 0); break;
    case 4: e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, sgd_wave_kernel<4>, kThreads, 0); break;
    default: return false;
  }
  if (e != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  // co-residency with head room: at most half of the resident warps
  return (int64_t)B * 2 <= (int64_t)sms * per_sm * (kThreads / 32);
}

// The wavefront kernels spin on progress counters of warps in other CTAs, so every CTA
// must be resident at once: they are launched cooperatively, and the driver either
// guarantees co-residency (whatever else the device runs) or fails the launch with
// cudaErrorCooperativeLaunchTooLarge, on which the caller runs the per-stratum launches.
template <typename... KArgs, typename... Args>
cudaError_t launch_cooperative(void (*kernel)(KArgs...), unsigned blocks, unsigned threads, size_t smem,
                               cudaStream_t st, Args... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(blocks);
  cfg.blockDim = dim3(threads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeCooperative;
  attr[0].val.cooperative = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  note_launch();
  return cudaLaunchKernelEx(&cfg, kernel, args...);
}

cudaError_t launch_wave(const SgdArgs& a, const int64_t* off, int B, int* progress, cudaStream_t st) {
  int L, VEC;
  sgd_geometry(a.k, a.vec_pref, &L, &VEC);
  cudaError_t e = cudaMemsetAsync(progress, 0, sizeof(int) * kProgressStride * (size_t)B, st);
  if (e != cudaSuccess) return e;
  const unsigned blocks = (unsigned)(((int64_t)B * 32 + kThreads - 1) / kThreads);
  switch (VEC) {
    case 1: return launch_cooperative(sgd_wave_kernel<1>, blocks, kThreads, 0, st, a, off, B, progress);
    case 2: return launch_cooperative(sgd_wave_kernel<2>, blocks, kThreads, 0, st, a, off, B, progress);
    case 4: return launch_cooperative(sgd_wave_kernel<4>, blocks, kThreads, 0, st, a, off, B, progress);
    default: return cudaErrorInvalidValue;
  }
}

namespace {
// slab wavefront geometry: warps per CTA and dynamic shared memory, or false if the
// column blocks' rows do not fit or the B warps cannot all be co-resident
template <int VEC>
bool slab_geometry_t(int k, int B, int64_t n, int* wpc_out, size_t* smem_out) {
  const int64_t wmax = (n + B - 1) / B;
  const size_t per_warp = (size_t)(wmax + kSlabRP) * k * sizeof(float) + 64 * sizeof(int4);
  constexpr size_t kBudget = 160 * 1024;
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // the widest CTA (8, 4, 2, 1 warps) whose occupancy keeps all B warps co-resident (every
  // warp waits on its successor) with 10 % head room: narrower CTAs pack the shared memory
  // of an SM more tightly when the slabs are wide (C3 at B = 1536: 8 warps -> 1 CTA per SM)
  for (int wpc = kThreads / 32; wpc >= 1; wpc >>= 1) {
    if (wpc * per_warp > kBudget) continue;
    const size_t smem = wpc * per_warp;
    if (cudaFuncSetAttribute(sgd_wave_slab_kernel<VEC>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
        cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    int per_sm = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, sgd_wave_slab_kernel<VEC>, wpc * 32, smem) !=
        cudaSuccess) {
      cudaGetLastError();
      return false;
    }
    if ((int64_t)B * 10 <= (int64_t)sms * per_sm * wpc * 9) {
      *wpc_out = wpc;
      *smem_out = smem;
      return true;
    }
  }
  return false;
}
}  // namespace

bool wave_slab_supported(int k, int vec_pref, int B, int64_t n) {
  int L, VEC, wpc;
  size_t smem;
  sgd_geometry(k, vec_pref, &L, &VEC);
  if (L != 32 || L * VEC * 4 != k) return false;
  switch (VEC) {
    case 1: return slab_geometry_t<1>(k, B, n, &wpc, &smem);
    case 2: return slab_geometry_t<2>(k, B, n, &wpc, &smem);
    case 4: return slab_geometry_t<4>(k, B, n, &wpc, &smem);
    default: return false;
  }
}

cudaError_t launch_wave_slab(const SgdArgs& a, const int64_t* off, int B, int* progress, int64_t n, cudaStream_t st) {
  int L, VEC, wpc = 0;
  size_t smem = 0;
  sgd_geometry(a.k, a.vec_pref, &L, &VEC);
  cudaError_t e = cudaMemsetAsync(progress, 0, sizeof(int) * kProgressStride * (size_t)B, st);
  if (e != cudaSuccess) return e;
  const int wmax = (int)((n + B - 1) / B);
#define SLAB_CASE(V)                                                                                        \
  case V:                                                                                                   \
    if (!slab_geometry_t<V>(a.k, B, n, &wpc, &smem)) return cudaErrorInvalidConfiguration;                 \
    e = launch_cooperative(sgd_wave_slab_kernel<V>, (unsigned)((B + wpc - 1) / wpc), (unsigned)(wpc * 32), smem, st, \
                           a, off, B, progress, n, wmax);                                                  \
    if (e != cudaSuccess) return e;                                                                       \
    break;
  switch (VEC) {
    SLAB_CASE(1)
    SLAB_CASE(2)
    SLAB_CASE(4)
    default: return cudaErrorInvalidValue;
  }
#undef SLAB_CASE
#ifdef HCCMF_DIAG_TRACE
  if (const char* path = getenv("HCCMF_TRACE_OUT")) {
    static std::vector<unsigned> host(2048 * 2048 * 3);
    cudaStreamSynchronize(st);
    cudaMemcpyFromSymbol(host.data(), g_wave_trace, sizeof(unsigned) * 3 * (size_t)B * B);
    if (FILE* f = fopen(path, "wb")) {
      fwrite(host.data(), sizeof(unsigned), 3 * (size_t)B * B, f);
      fclose(f);
    }
  }
#endif
  return cudaGetLastError();
}

// Hogwild with k = 32 or 64 (auto geometry, fp32 Q) runs one rating per warp (NarrowSgd)
static bool narrow_hogwild(int k, int vec_pref) { return vec_pref == 0 && (k == 32 || k == 64); }

int hogwild_groups_per_warp(int k, int vec_pref) {
  return narrow_hogwild(k, vec_pref) ? 1 : 32 / sgd_lanes(k, vec_pref);
}

static cudaError_t launch_narrow(const SgdArgs& a, int64_t warps, cudaStream_t st) {
  int64_t w = std::min<int64_t>(warps, a.n_tasks);
  if (w < 1) return cudaSuccess;
  const int threads = w < kThreads / 32 ? (int)w * 32 : kThreads;
  const unsigned blocks = (unsigned)((w * 32 + threads - 1) / threads);
  const int depth = a.depth < 1 ? 4 : a.depth;  // auto: 4 ratings ahead
#define NARROW_CASE(EE, DD)                                                                       \
  if (a.k == 32 * EE && depth == DD) {                                                            \
    if (a.atomic_q)                                                                               \
      (note_launch(), sgd_narrow_kernel<EE, true, DD><<<blocks, threads, 0, st>>>(a));           \
    else                                                                                          \
      (note_launch(), sgd_narrow_kernel<EE, false, DD><<<blocks, threads, 0, st>>>(a));          \
    return cudaGetLastError();                                                                    \
  }
  NARROW_CASE(1, 1) NARROW_CASE(1, 2) NARROW_CASE(1, 3) NARROW_CASE(1, 4)
  NARROW_CASE(2, 1) NARROW_CASE(2, 2) NARROW_CASE(2, 3) NARROW_CASE(2, 4)
#undef NARROW_CASE
  return cudaErrorInvalidValue;
}

cudaError_t launch_sgd(const SgdArgs& a, int64_t warps, cudaStream_t st) {
  if (a.n_tasks <= 0) return cudaSuccess;
  if (!a.prefetch && !a.qhalf && narrow_hogwild(a.k, a.vec_pref)) return launch_narrow(a, warps, st);
  int L, VEC;
  sgd_geometry(a.k, a.vec_pref, &L, &VEC);
  const bool full = (L * VEC * 4 == a.k);
#define SGD_CASE(LL, VV) \
  if (L == LL && VEC == VV) return full ? launch_t<LL, VV, true>(a, warps, st) : launch_t<LL, VV, false>(a, warps, st);
  SGD_CASE(1, 1) SGD_CASE(2, 1) SGD_CASE(4, 1)
  SGD_CASE(8, 1) SGD_CASE(8, 2) SGD_CASE(8, 4)
  SGD_CASE(16, 1) SGD_CASE(16, 2) SGD_CASE(16, 4)
  SGD_CASE(32, 1) SGD_CASE(32, 2) SGD_CASE(32, 4)
#undef SGD_CASE
  return cudaErrorInvalidValue;
}

}  // namespace hccmf
