// api.cu -- the C ABI (include/hccmf.h) and the host runtime around the kernels:
// argument checks, device memory, the partition planner (DP0/DP1/DP2), SGD
// launch plans for every (schedule, sync) pair, the ring / all-reduce Q
// synchronisation over NCCL, and export.
#include <algorithm>
#include <functional>
#include <queue>
#include <chrono>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>

#include <nccl.h>

#include "internal.cuh"

using namespace hccmf;

namespace {

thread_local std::string g_err;

hccmf_status fail(hccmf_t h, hccmf_status st, const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  if (h) {
    h->err = buf;
    if (st == HCCMF_ECUDA || st == HCCMF_ENCCL) h->sticky = st;
  }
  g_err = buf;
  return st;
}

#define CU(h, call)                                                                                   \
  do {                                                                                                \
    cudaError_t e_ = (call);                                                                          \
    if (e_ != cudaSuccess) {                                                                          \
      if (e_ == cudaErrorMemoryAllocation) {                                                          \
        cudaGetLastError();                                                                           \
        return fail(h, HCCMF_ENOMEM, "%s: out of device memory (%s:%d)", #call, __FILE__, __LINE__);  \
      }                                                                                               \
      return fail(h, HCCMF_ECUDA, "%s: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__, __LINE__); \
    }                                                                                                 \
  } while (0)

// a data-plane call (comm.cuh: NCCL or loopback); failures are sticky HCCMF_ENCCL
#define CM(h, call)                                                                                   \
  do {                                                                                                \
    if ((call) != 0)                                                                                  \
      return fail(h, HCCMF_ENCCL, "%s [%s] (%s:%d)", (h)->comm->err.c_str(), (h)->comm->backend(), __FILE__, \
                  __LINE__);                                                                          \
  } while (0)

#define ENTER(h)                                      \
  do {                                                \
    if (!(h)) return fail(nullptr, HCCMF_EINVAL, "NULL handle"); \
    if ((h)->sticky != HCCMF_OK) return (h)->sticky;  \
    CU(h, cudaSetDevice((h)->device));                \
  } while (0)

// Every device buffer of a handle comes from the device's stream-ordered pool on the
// handle's stream.  The pool keeps its mapped memory (release threshold = max, set in
// make_ctx), so repeated jobs and the syncs inside one partition reuse it instead of
// mapping and unmapping gigabytes (C3 partition: 550 -> see DESIGN.md section 8).
template <typename T>
cudaError_t dmalloc(hccmf_t h, T** p, size_t count) {
  const size_t bytes = sizeof(T) * (count ? count : 1);
  cudaError_t e = cudaMallocAsync((void**)p, bytes, h->stream);
  if (e == cudaSuccess) h->device_bytes += bytes;
  return e;
}
template <typename T>
void dfree(hccmf_t h, T*& p, size_t count) {
  if (p) {
    cudaFreeAsync((void*)p, h->stream);
    h->device_bytes -= sizeof(T) * (count ? count : 1);
  }
  p = nullptr;
}

hccmf_status finish(hccmf_t h) {
  CU(h, cudaGetLastError());
  if (h->sync_stream) CU(h, cudaStreamSynchronize(h->stream));
  return HCCMF_OK;
}

// HCCMF_PROFILE=1: per-phase wall times of the preprocessing on stderr (syncs the stream)
struct PhaseTimer {
  bool on;
  cudaStream_t st;
  std::chrono::steady_clock::time_point t0;
  explicit PhaseTimer(cudaStream_t s) : on(getenv("HCCMF_PROFILE") != nullptr), st(s) {
    if (on) cudaStreamSynchronize(st);
    t0 = std::chrono::steady_clock::now();
  }
  void mark(const char* what) {
    if (!on) return;
    cudaStreamSynchronize(st);
    const auto t1 = std::chrono::steady_clock::now();
    fprintf(stderr, "[hccmf] %-28s %9.3f ms\n", what, std::chrono::duration<double, std::milli>(t1 - t0).count());
    t0 = t1;
  }
};

int bitlen(uint64_t x) {  // bits needed to represent x (0 -> 0)
  int b = 0;
  while (x) { ++b; x >>= 1; }
  return b;
}

int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

hccmf_status check_problem(int64_t m, int64_t n, int32_t k, float gamma, float lambda) {
  if (m < 1 || m >= (1LL << 31) || n < 1 || n >= (1LL << 31))
    return fail(nullptr, HCCMF_EINVAL, "m, n must be in [1, 2^31)");
  if (k < 4 || k > 512 || k % 4 != 0) return fail(nullptr, HCCMF_EINVAL, "k must be a multiple of 4 in [4, 512]");
  if (!(gamma > 0.f) || !std::isfinite(gamma)) return fail(nullptr, HCCMF_EINVAL, "gamma must be finite and > 0");
  if (!(lambda >= 0.f) || !std::isfinite(lambda)) return fail(nullptr, HCCMF_EINVAL, "lambda must be finite and >= 0");
  return HCCMF_OK;
}

hccmf_status make_ctx(int64_t m, int64_t n, int32_t k, float gamma, float lambda, int device, hccmf_t* out) {
  hccmf_t h = new hccmf_ctx();
  h->m = m;
  h->n = n;
  h->k = k;
  h->gamma = gamma;
  h->lambda = lambda;
  h->device = device;
  cudaError_t e = cudaSetDevice(device);
  // a blocking stream: the handle's work is ordered after the legacy default stream, so
  // device inputs a caller produced there (e.g. with torch) are complete before we copy
  if (e == cudaSuccess) e = cudaStreamCreate(&h->stream);
  if (e != cudaSuccess) {
    hccmf_status st = fail(nullptr, HCCMF_ECUDA, "no usable CUDA device: %s", cudaGetErrorString(e));
    cudaGetLastError();
    delete h;
    return st;
  }
  h->own_stream = true;
  // Keep what the stream-ordered pool maps (a release threshold of 0 unmaps and remaps
  // gigabytes at every stream synchronisation; HCCMF_TRIM=1 trims at destroy).
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, device) == cudaSuccess) {
    uint64_t keep = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
  }
  cudaGetLastError();
  *out = h;
  return HCCMF_OK;
}

void trim_pool(hccmf_t h) {
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, h->device) == cudaSuccess) {
    cudaStreamSynchronize(h->stream);
    cudaMemPoolTrimTo(pool, 0);
  }
  cudaGetLastError();
}

// ----------------------------------------------------------- DP planners
// Independent host implementation of section 3.3 (the oracle has its own).
void plan_dp0(int G, const double* t, std::vector<double>& x) {  // Eq. 6
  x.assign(G, 0.0);
  for (int i = 0; i < G; ++i) {
    double s = 0.0;
    for (int j = 0; j < G; ++j) s += t[i] / t[j];
    x[i] = 1.0 / s;
  }
}

void plan_dp1(int G, std::vector<double>& x, std::vector<double> t) {  // Alg. 1, R11
  for (int it = 0; it < 8; ++it) {
    double tbar = 0.0, tmin = t[0], dev = 0.0;
    for (int s = 0; s < G; ++s) tbar += t[s];
    tbar /= (double)G;
    for (int s = 0; s < G; ++s) {
      tmin = std::min(tmin, t[s]);
      dev = std::max(dev, std::fabs(t[s] - tbar));
    }
    if (dev / tmin <= 0.1) break;
    double sum = 0.0;
    for (int s = 0; s < G; ++s) sum += x[s] * tbar / t[s];
    for (int s = 0; s < G; ++s) {
      const double xn = (x[s] * tbar / t[s]) / sum;
      t[s] = t[s] * xn / x[s];
      x[s] = xn;
    }
  }
}

void plan_dp2(int G, std::vector<double>& x, const double* t, double t_sync) {  // Eq. 7, R12
  const int smed = (G - 1) / 2;
  const double tmed = t[smed];
  double sum = 0.0;
  std::vector<double> y(G);
  for (int s = 0; s < G; ++s) {
    double Ts = tmed + (double)(s - smed) * t_sync;
    if (Ts < 0.0) Ts = 0.0;
    y[s] = x[s] * Ts / t[s];
    sum += y[s];
  }
  for (int s = 0; s < G; ++s) x[s] = y[s] / sum;
}


void free_partition(hccmf_t h) {
  for (auto& p : h->plans) {
    dfree(h, p.d_lo, p.n_tasks);
    dfree(h, p.d_hi, p.n_tasks);
  }
  h->plans.clear();
  dfree(h, h->d_task_lo, h->n_tasks);
  dfree(h, h->d_task_hi, h->n_tasks);
  h->n_tasks = 0;
  dfree(h, h->d_u, h->local_nnz);
  dfree(h, h->d_v, h->local_nnz);
  dfree(h, h->d_r, h->local_nnz);
  dfree(h, h->d_perm_row, h->m);
  dfree(h, h->d_perm_col, h->n);
  dfree(h, h->d_P, h->rows * h->k);
  dfree(h, h->d_Q, h->n * h->k);
  dfree(h, h->d_Qrep, (size_t)h->n * h->k * (h->shard_hi - h->shard_lo));
  dfree(h, h->d_Qh, (size_t)h->n * h->k);
  dfree(h, h->d_counters, h->n_counters);
  h->n_counters = 0;
  dfree(h, h->d_blk_off, h->nblk_local + 1);
  dfree(h, h->d_progress, (size_t)h->Br * kProgressStride);
  det_chain_free(&h->det_chain, h->stream);
  h->local_nnz = 0;
  h->rows = 0;
  h->blk_task_off.clear();
}

// ------------------------------------------------------------ timeline (HCCMF_OPT_TIMELINE)
void timeline_clear(hccmf_t h) {
  for (auto& r : h->timeline) {
    cudaEventDestroy(r.a);
    cudaEventDestroy(r.b);
  }
  h->timeline.clear();
}
// open a row: its start event is recorded now on `st`; returns the row index (-1: off)
int timeline_begin(hccmf_t h, int kind, int stage, int block, cudaStream_t st) {
  if (!h->opt_timeline) return -1;
  hccmf_ctx::TimelineRow r{kind, stage, block, nullptr, nullptr};
  if (cudaEventCreate(&r.a) != cudaSuccess || cudaEventCreate(&r.b) != cudaSuccess) {
    cudaGetLastError();
    return -1;
  }
  cudaEventRecord(r.a, st);
  h->timeline.push_back(r);
  return (int)h->timeline.size() - 1;
}
void timeline_end(hccmf_t h, int row, cudaStream_t st) {
  if (row >= 0) cudaEventRecord(h->timeline[row].b, st);
}

// ------------------------------------------------------------ SGD plans
// The a5/a6/a7 schedule as block lists (pure host logic, also exported through
// hccmf_schedule so multi-process tests can run it without a device):
// launches in order; blocks inside one launch share no P rows and no Q columns
// (DET) or no users (HOGWILD), so running them concurrently is the serial
// order of DESIGN.md R19.
struct BlockLaunch {
  std::vector<int64_t> blocks;
  int32_t qrep, stage, phase = 0;
};

const char* schedule_blocks(int G, int Br, int Bc, int sched, int sync, int shard_lo, int shard_hi,
                            std::vector<BlockLaunch>& out, int* n_stages, int phases = 1) {
  out.clear();
  *n_stages = 1;
  auto blk = [&](int64_t s, int64_t rb, int64_t cb) { return (s * Br + rb) * Bc + cb; };
  const int eff_sync = (G == 1) ? HCCMF_SYNC_NONE : sync;
  if (eff_sync == HCCMF_SYNC_NONE && G != 1) return "sync NONE needs n_shards == 1";
  if (sched == HCCMF_SCHED_DET) {
    if (eff_sync == HCCMF_SYNC_RING) {
      if (Bc != G * Br) return "DET+RING needs grid_cols == n_shards * grid_rows";
      const int c = Br;
      *n_stages = G;
      for (int t = 0; t < G; ++t)
        for (int t2 = 0; t2 < c; ++t2) {
          BlockLaunch L{{}, 0, t};
          for (int s = shard_lo; s < shard_hi; ++s) {
            const int g = (s + t) % G;
            for (int i = 0; i < c; ++i) L.blocks.push_back(blk(s, i, (int64_t)g * c + (i + t2) % c));
          }
          out.push_back(L);
        }
    } else {
      if (Br != Bc) return "DET needs grid_rows == grid_cols (sync NONE/ALLREDUCE)";
      const int c = Br;
      for (int s = shard_lo; s < shard_hi; ++s)
        for (int t2 = 0; t2 < c; ++t2) {
          BlockLaunch L{{}, s - shard_lo, 0};
          for (int i = 0; i < c; ++i) L.blocks.push_back(blk(s, i, (i + t2) % c));
          out.push_back(L);
        }
    }
  } else {
    if (eff_sync == HCCMF_SYNC_RING) {
      if (Bc % G != 0) return "HOGWILD+RING needs grid_cols % n_shards == 0";
      const int c = Bc / G;
      *n_stages = G;
      for (int t = 0; t < G; ++t)
        for (int j = 0; j < c; ++j) {
          BlockLaunch L{{}, 0, t};
          for (int s = shard_lo; s < shard_hi; ++s) {
            const int g = (s + t) % G;
            for (int rb = 0; rb < Br; ++rb) L.blocks.push_back(blk(s, rb, (int64_t)g * c + j));
          }
          out.push_back(L);
        }
    } else if (eff_sync == HCCMF_SYNC_ALLREDUCE_AVG && phases > 1) {
      // sub-epoch sync (R22): round ph runs row blocks [ph Br/phases, (ph+1) Br/phases)
      if (Br % phases != 0) return "sync phases must divide grid_rows";
      const int per = Br / phases;
      for (int ph = 0; ph < phases; ++ph)
        for (int s = shard_lo; s < shard_hi; ++s)
          for (int cb = 0; cb < Bc; ++cb) {
            BlockLaunch L{{}, s - shard_lo, 0, ph};
            for (int rb = ph * per; rb < (ph + 1) * per; ++rb) L.blocks.push_back(blk(s, rb, cb));
            out.push_back(L);
          }
    } else {
      // column-block-major phases: a user's p_u is touched by one task per launch
      for (int s = shard_lo; s < shard_hi; ++s)
        for (int cb = 0; cb < Bc; ++cb) {
          BlockLaunch L{{}, s - shard_lo, 0};
          for (int rb = 0; rb < Br; ++rb) L.blocks.push_back(blk(s, rb, cb));
          out.push_back(L);
        }
    }
  }
  return nullptr;
}

// Q rows [a, b) of ring column group g (columns of column blocks [g c, (g+1) c))
void ring_cols(int64_t n, int G, int Br, int Bc, int sched, int g, int64_t* a, int64_t* b) {
  const int c = (sched == HCCMF_SCHED_DET) ? Br : Bc / G;
  *a = ceil_div((int64_t)g * c * n, Bc);
  *b = ceil_div((int64_t)(g + 1) * c * n, Bc);
}

hccmf_status build_plan(hccmf_t h, int sched, int sync, Plan** out) {
  for (auto& p : h->plans)
    if (p.sched == sched && p.sync == sync && p.phases == (sched == HCCMF_SCHED_HOGWILD ? (int)h->opt_phases : 1)) {
      *out = &p;
      return HCCMF_OK;
    }
  std::vector<BlockLaunch> bl;
  Plan pl;
  pl.sched = sched;
  pl.sync = sync;
  const char* msg = schedule_blocks(h->G, h->Br, h->Bc, sched, sync, h->shard_lo, h->shard_hi, bl, &pl.n_stages,
                                    sched == HCCMF_SCHED_HOGWILD ? (int)h->opt_phases : 1);
  if (msg) return fail(h, HCCMF_EINVAL, "%s", msg);
  pl.phases = sched == HCCMF_SCHED_HOGWILD ? (int)h->opt_phases : 1;
  // DET: one task per non-empty block, from the host block offsets.  HOGWILD: the blocks'
  // task ranges of the device task list, gathered on the device (segment tables only)
  std::vector<int64_t> lo, hi, seg_src, seg_dst;
  int64_t total = 0;
  for (const BlockLaunch& L : bl) {
    const int64_t t0 = total;
    for (int64_t b : L.blocks) {
      if (sched == HCCMF_SCHED_DET) {
        const int64_t a = h->block_off[b] - h->rec0, e = h->block_off[b + 1] - h->rec0;
        if (e > a) {
          lo.push_back(a);
          hi.push_back(e);
          ++total;
        }
      } else {
        const int64_t j = b - h->blk0;
        const int64_t cnt = h->blk_task_off[j + 1] - h->blk_task_off[j];
        if (cnt > 0) {
          seg_src.push_back(h->blk_task_off[j]);
          seg_dst.push_back(total);
          total += cnt;
        }
      }
    }
    std::vector<int64_t> cbs;
    for (int64_t b : L.blocks) cbs.push_back(b % h->Bc);
    std::sort(cbs.begin(), cbs.end());
    cbs.erase(std::unique(cbs.begin(), cbs.end()), cbs.end());
    int64_t items = 0;
    for (int64_t cb : cbs) items += ceil_div((cb + 1) * h->n, h->Bc) - ceil_div(cb * h->n, h->Bc);
    pl.launches.push_back(Launch{t0, total - t0, L.qrep, L.stage, L.phase, items});
  }
  pl.n_tasks = total;
  CU(h, dmalloc(h, &pl.d_lo, pl.n_tasks));
  CU(h, dmalloc(h, &pl.d_hi, pl.n_tasks));
  if (sched == HCCMF_SCHED_DET && pl.n_tasks) {
    CU(h, cudaMemcpyAsync(pl.d_lo, lo.data(), sizeof(int64_t) * pl.n_tasks, cudaMemcpyHostToDevice, h->stream));
    CU(h, cudaMemcpyAsync(pl.d_hi, hi.data(), sizeof(int64_t) * pl.n_tasks, cudaMemcpyHostToDevice, h->stream));
  } else if (pl.n_tasks) {
    CU(h, k_gather_tasks(seg_src.data(), seg_dst.data(), (int64_t)seg_src.size(), total, h->d_task_lo, h->d_task_hi,
                         pl.d_lo, pl.d_hi, h->stream));
  }
  if ((int64_t)pl.launches.size() > h->n_counters) {
    dfree(h, h->d_counters, h->n_counters);
    h->n_counters = (int64_t)pl.launches.size();
    CU(h, dmalloc(h, &h->d_counters, h->n_counters));
  }
  CU(h, cudaStreamSynchronize(h->stream));
  h->plans.push_back(pl);
  *out = &h->plans.back();
  return HCCMF_OK;
}

// Hogwild concurrency (R14, R28, R32): the rating groups in flight set how stale a
// q_v read can be.  A read that misses tau concurrent updates of its item is a delayed gradient
// step; on the per-rating quadratic in q_v (curvature ~ |p_u|^2 + lambda, and |p_u|^2 grows to
// the rating scale) the delay is harmless while tau * gamma * (r_rms + lambda) stays small.  With
// the items of a launch hit uniformly, tau ~ groups / items, so the cap is
//   groups <= items * kappa / (gamma (r_rms + lambda)),   kappa = opt_staleness * 1e-4 (0.006),
// calibrated on the measured stability edge (C4, ratings 0..100, lambda 1: stable at
// tau gamma (r_rms + lambda) = 0.0077 and 0.0097, divergent at 0.0155, and one epoch-1 NaN in
// ~100 runs of C4 at 5 % size at 0.008 -- hence 0.006, 25 % inside it; C3 runs at 0.0048).
// opt_conflict > 0 replaces it by the fixed items / opt_conflict of round 1.  Never more
// than 32 resident warps per SM.
int64_t auto_warps(hccmf_t h, int64_t items_in_play) {
  if (h->opt_warps > 0) return h->opt_warps;
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, h->device);
#ifndef HCCMF_WARPS_PER_SM
#define HCCMF_WARPS_PER_SM 32  // resident warps of the warp-per-rating kernel (64 registers: 4 CTAs of 8)
#endif
  int64_t w = (int64_t)sms * HCCMF_WARPS_PER_SM;
  const int64_t groups_per_warp = hogwild_groups_per_warp(h->k, (int)h->opt_vec);
  int64_t groups = -1;
  if (h->opt_conflict > 0) {
    groups = items_in_play / h->opt_conflict;
  } else if (h->opt_staleness > 0) {
    const double denom = (double)h->gamma * (h->r_rms + (double)h->lambda);
    const double g = denom > 0.0 ? (double)items_in_play * (double)h->opt_staleness * 1e-4 / denom : 1e18;
    groups = (int64_t)std::min(g, 1e15);
  }
  if (groups >= 0) w = std::min(w, std::max<int64_t>(1, groups / groups_per_warp));
  return w;
}

// column-group row range [a, b) of Q for ring group g
void ring_group_cols(hccmf_t h, int sched, int g, int64_t* a, int64_t* b) {
  ring_cols(h->n, h->G, h->Br, h->Bc, sched, g, a, b);
}

hccmf_status wire_reserve(hccmf_t h, size_t halves, bool* grown = nullptr) {  // send + recv staging, binary16
  const size_t bytes = 2 * halves * 2;
  if (grown) *grown = false;
  if (h->wire_bytes >= bytes) return HCCMF_OK;
  if (grown) *grown = true;
  if (h->d_wire) {  // the comm stream may still read the old staging buffer
    if (h->comm_stream) CU(h, cudaStreamSynchronize(h->comm_stream));
    cudaFreeAsync(h->d_wire, h->stream);
  }
  h->d_wire = nullptr;
  h->wire_bytes = 0;
  CU(h, cudaMallocAsync(&h->d_wire, bytes, h->stream));
  h->wire_bytes = bytes;
  return HCCMF_OK;
}

// one ring transfer of Q rows [sa, sb) to `prev` and [ra, rb) from `next`, fp32 or binary16
hccmf_status ring_transfer(hccmf_t h, int64_t sa, int64_t sb, int64_t ra, int64_t rb, int prev, int next,
                           cudaStream_t cs, int site) {
  const size_t ns = (size_t)(sb - sa) * h->k, nr = (size_t)(rb - ra) * h->k;
  h->comm_counts[site] += 1;
  Comm* c = h->comm;
  if (!h->opt_wire16) {
    CM(h, c->group_start());
    if (ns) CM(h, c->send(h->d_Q + sa * h->k, ns * sizeof(float), prev, cs));
    if (nr) CM(h, c->recv(h->d_Q + ra * h->k, nr * sizeof(float), next, cs));
    CM(h, c->group_end());
    return HCCMF_OK;
  }
  h->comm_counts[SITE_RING_WIRE16] += 1;
  // Strategy 2: pack to binary16, ship half the bytes, unpack (all on the comm stream)
  const size_t cap = (size_t)h->n * h->k;
  bool grown = false;
  hccmf_status st = wire_reserve(h, cap, &grown);
  if (st != HCCMF_OK) return st;
  // a new staging buffer (stream-ordered on the handle's stream) is ready before cs uses it;
  // afterwards transfers never wait for the compute stream (hidden synchronisation)
  if (grown && cs != h->stream) CU(h, cudaStreamSynchronize(h->stream));
  char* sendb = static_cast<char*>(h->d_wire);
  char* recvb = sendb + cap * 2;
  CU(h, k_pack_half(h->d_Q + sa * h->k, sendb, (int64_t)ns, cs));
  CM(h, c->group_start());
  if (ns) CM(h, c->send(sendb, ns * 2, prev, cs));
  if (nr) CM(h, c->recv(recvb, nr * 2, next, cs));
  CM(h, c->group_end());
  CU(h, k_unpack_half(recvb, h->d_Q + ra * h->k, (int64_t)nr, cs));
  return HCCMF_OK;
}

hccmf_status ring_exchange(hccmf_t h, int sched, int t) {
  const int G = h->G, s = h->rank;
  const int g_send = (s + t) % G, g_recv = (s + t + 1) % G;
  int64_t sa, sb, ra, rb;
  ring_group_cols(h, sched, g_send, &sa, &sb);
  ring_group_cols(h, sched, g_recv, &ra, &rb);
  const int prev = (s - 1 + G) % G, next = (s + 1) % G;
  const int row = timeline_begin(h, 2, t, -1, h->stream);
  hccmf_status st = ring_transfer(h, sa, sb, ra, rb, prev, next, h->stream, SITE_RING_STAGE);
  timeline_end(h, row, h->stream);
  return st;
}

// Hidden synchronisation (L1143-L1172) with asynchronous computing-transmission
// (L1251-L1269): HOGWILD ring stages are launched one column block at a time; as soon
// as column block j of stage t is done, the comm stream ships it to shard s-1 and
// receives column block j of the next group from s+1, overlapping the transfer with
// the compute of blocks j+1.. of the same stage.  Stage t+1's block j waits only for
// its own block's receive.
hccmf_status ring_exchange_block(hccmf_t h, int t, int j, cudaStream_t cs) {
  const int G = h->G, s = h->rank, c = h->Bc / G;
  auto rows = [&](int g, int64_t* a, int64_t* b) {
    const int64_t cb = (int64_t)g * c + j;
    *a = ceil_div(cb * h->n, h->Bc);
    *b = ceil_div((cb + 1) * h->n, h->Bc);
  };
  int64_t sa, sb, ra, rb;
  rows((s + t) % G, &sa, &sb);
  rows((s + t + 1) % G, &ra, &rb);
  const int prev = (s - 1 + G) % G, next = (s + 1) % G;
  const int row = timeline_begin(h, 1, t, j, cs);
  hccmf_status st = ring_transfer(h, sa, sb, ra, rb, prev, next, cs, SITE_RING_BLOCK);
  timeline_end(h, row, cs);
  return st;
}

// after ring epochs rank s holds only group s of Q: broadcast every group from its owner
hccmf_status materialize_q(hccmf_t h) {
  if (h->world <= 1 || h->q_ring_sched < 0) return HCCMF_OK;
  h->comm_counts[SITE_MATERIALIZE_Q] += 1;
  CM(h, h->comm->group_start());
  for (int g = 0; g < h->G; ++g) {
    int64_t a, b;
    ring_group_cols(h, h->q_ring_sched, g, &a, &b);
    if (b > a)
      CM(h, h->comm->broadcast(h->d_Q + a * h->k, h->d_Q + a * h->k, sizeof(float) * (size_t)(b - a) * h->k, g,
                               h->stream));
  }
  CM(h, h->comm->group_end());
  h->q_ring_sched = -1;
  return HCCMF_OK;
}

// Strategy 2 all-reduce (R25): Q = binary16( sum_s binary16(Q_s) / G ), the sum in fp64
// in rank order -- the function the oracle (orc_epoch_wire16) and the logical backend
// (average_half_kernel) compute, with only binary16 on the wire.  Chunk c of the packed
// copy (C = ceil(nk / G) halves, zero padded) belongs to rank c: an all-to-all ships
// every rank's chunk c to rank c, which reduces its G copies and rounds once; an
// all-gather returns the rounded chunks.  Wire bytes per rank 4 (G-1)/G nk, half of an
// fp32 ring all-reduce; reducing in binary16 inside NCCL would round at every hop.
hccmf_status allreduce_q16(hccmf_t h, cudaStream_t s) {
  const int G = h->G, me = h->rank;
  const int64_t nk = h->n * h->k;
  const int64_t C = (nk + G - 1) / G;
  h->comm_counts[SITE_ALLREDUCE_Q16] += 1;
  hccmf_status w = wire_reserve(h, (size_t)C * G);
  if (w != HCCMF_OK) return w;
  uint16_t* packed = static_cast<uint16_t*>(h->d_wire);  // G x C halves
  uint16_t* gath = packed + (size_t)C * G;                // G x C halves: rank r's copy of my chunk
  if (C * G > nk) CU(h, cudaMemsetAsync(packed + nk, 0, sizeof(uint16_t) * (size_t)(C * G - nk), s));
  CU(h, k_pack_half(h->d_Q, packed, nk, s));
  Comm* c = h->comm;
  CM(h, c->group_start());
  for (int p = 0; p < G; ++p)
    if (p != me) {
      CM(h, c->send(packed + (size_t)p * C, sizeof(uint16_t) * C, p, s));
      CM(h, c->recv(gath + (size_t)p * C, sizeof(uint16_t) * C, p, s));
    }
  CM(h, c->group_end());
  CU(h, cudaMemcpyAsync(gath + (size_t)me * C, packed + (size_t)me * C, sizeof(uint16_t) * C,
                        cudaMemcpyDeviceToDevice, s));
  CU(h, k_mean_gathered_half(gath, G, C, C, packed + (size_t)me * C, s));
  CM(h, c->allgather(packed + (size_t)me * C, packed, sizeof(uint16_t) * C, s));
  CU(h, k_unpack_half(packed, h->d_Q, nk, s));
  return HCCMF_OK;
}

}  // namespace

// ======================================================================== ABI
extern "C" {

const char* hccmf_version(void) { return "hccmf 0.1 sm_100a"; }

int64_t hccmf_kernel_launches(void) { return hccmf::g_kernel_launches.load(std::memory_order_relaxed); }

const char* hccmf_last_error(hccmf_t h) { return h ? h->err.c_str() : g_err.c_str(); }

hccmf_status hccmf_create(int64_t m, int64_t n, int32_t k, float gamma, float lambda, hccmf_t* out) {
  if (!out) return fail(nullptr, HCCMF_EINVAL, "out is NULL");
  *out = nullptr;
  hccmf_status st = check_problem(m, n, k, gamma, lambda);
  if (st != HCCMF_OK) return st;
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(nullptr, HCCMF_ECUDA, "no CUDA device: %s", cudaGetErrorString(e));
  }
  return make_ctx(m, n, k, gamma, lambda, dev, out);
}

hccmf_status hccmf_nccl_unique_id(void* out128) {
  if (!out128) return fail(nullptr, HCCMF_EINVAL, "out is NULL");
  ncclUniqueId id;
  ncclResult_t r = ncclGetUniqueId(&id);
  if (r != ncclSuccess) return fail(nullptr, HCCMF_ENCCL, "ncclGetUniqueId: %s", ncclGetErrorString(r));
  static_assert(sizeof(ncclUniqueId) == 128, "NCCL unique id is 128 bytes");
  memcpy(out128, &id, sizeof(id));
  return HCCMF_OK;
}

hccmf_status hccmf_create_dist(int64_t m, int64_t n, int32_t k, float gamma, float lambda, const void* nccl_unique_id,
                               int32_t rank, int32_t world, int32_t device, hccmf_t* out) {
  if (!out || !nccl_unique_id) return fail(nullptr, HCCMF_EINVAL, "NULL argument");
  *out = nullptr;
  if (world < 1 || rank < 0 || rank >= world || device < 0) return fail(nullptr, HCCMF_EINVAL, "bad rank/world/device");
  hccmf_status st = check_problem(m, n, k, gamma, lambda);
  if (st != HCCMF_OK) return st;
  st = make_ctx(m, n, k, gamma, lambda, device, out);
  if (st != HCCMF_OK) return st;
  hccmf_t h = *out;
  h->rank = rank;
  h->world = world;
  std::string why;
  h->comm = make_nccl_comm(nccl_unique_id, rank, world, device, &why);
  if (!h->comm) {
    st = fail(nullptr, HCCMF_ENCCL, "%s", why.c_str());
    hccmf_destroy(h);
    *out = nullptr;
    return st;
  }
  return HCCMF_OK;
}

hccmf_status hccmf_create_loopback(int64_t m, int64_t n, int32_t k, float gamma, float lambda, hccmf_hub_t hub,
                                   int32_t rank, int32_t device, hccmf_t* out) {
  if (!out || !hub) return fail(nullptr, HCCMF_EINVAL, "NULL argument");
  *out = nullptr;
  hccmf_status st = check_problem(m, n, k, gamma, lambda);
  if (st != HCCMF_OK) return st;
  std::string why;
  Comm* c = make_loopback_comm(hub, rank, device, &why);
  if (!c) return fail(nullptr, HCCMF_EINVAL, "loopback: %s", why.c_str());
  st = make_ctx(m, n, k, gamma, lambda, device, out);
  if (st != HCCMF_OK) {
    delete c;
    return st;
  }
  (*out)->rank = rank;
  (*out)->world = c->world;
  (*out)->comm = c;
  return HCCMF_OK;
}

hccmf_status hccmf_comm_counts(hccmf_t h, int64_t* counts, int32_t n, int32_t* n_sites) {
  if (!h) return fail(nullptr, HCCMF_EINVAL, "NULL handle");
  if (n_sites) *n_sites = N_COMM_SITES;
  for (int i = 0; i < n && i < N_COMM_SITES; ++i) counts[i] = h->comm_counts[i];
  return HCCMF_OK;
}

hccmf_status hccmf_set_stream(hccmf_t h, void* stream) {
  ENTER(h);
  if (h->own_stream && h->stream) {
    CU(h, cudaStreamSynchronize(h->stream));
    cudaStreamDestroy(h->stream);
  }
  h->stream = (cudaStream_t)stream;
  h->own_stream = false;
  return HCCMF_OK;
}

hccmf_status hccmf_set_option(hccmf_t h, int32_t option, int64_t value) {
  ENTER(h);
  switch (option) {
    case HCCMF_OPT_HOGWILD_WARPS:
      if (value < 0) return fail(h, HCCMF_EINVAL, "warps must be >= 0");
      h->opt_warps = value;
      return HCCMF_OK;
    case HCCMF_OPT_TASK_RATINGS:
      if (value < 1) return fail(h, HCCMF_EINVAL, "task ratings must be >= 1");
      h->opt_task = value;
      return HCCMF_OK;
    case HCCMF_OPT_SYNC_STREAM:
      h->sync_stream = value != 0;
      return HCCMF_OK;
    case HCCMF_OPT_HOGWILD_ATOMIC:
      h->opt_atomic = value != 0;
      return HCCMF_OK;
    case HCCMF_OPT_L2_PERSIST:
      h->opt_l2persist = value != 0;
      return HCCMF_OK;
    case HCCMF_OPT_WIRE_FP16:
      h->opt_wire16 = value != 0;
      return HCCMF_OK;
    case HCCMF_OPT_STORAGE:
      if (value < 0 || value > 2) return fail(h, HCCMF_EINVAL, "storage must be 0 (fp32), 1 (binary16 Q) or 2 (binary16 Q, stochastic rounding)");
      h->storage = (int32_t)value;
      return HCCMF_OK;
    case HCCMF_OPT_PREFETCH_DEPTH:
      if (value < 0 || value > 4) return fail(h, HCCMF_EINVAL, "prefetch depth must be in [0, 4] (0 = auto)");
      h->opt_depth = value;
      return HCCMF_OK;
    case HCCMF_OPT_SYNC_PHASES:
      if (value < 1) return fail(h, HCCMF_EINVAL, "sync phases must be >= 1");
      h->opt_phases = value;
      return HCCMF_OK;
    case HCCMF_OPT_DET_WAVE:
      if (value < 0 || value > 3) return fail(h, HCCMF_EINVAL, "det_wave must be 0, 1, 2 or 3");
      h->opt_wave = (int)value;
      return HCCMF_OK;
    case HCCMF_OPT_VEC:
      if (value != 0 && value != 1 && value != 2 && value != 4) return fail(h, HCCMF_EINVAL, "vec must be 0, 1, 2 or 4");
      h->opt_vec = value;
      return HCCMF_OK;
    case HCCMF_OPT_HEAVY_FIRST:
      h->opt_heavy = value;
      return HCCMF_OK;
    case HCCMF_OPT_TIMELINE:
      h->opt_timeline = value != 0;
      if (!h->opt_timeline) timeline_clear(h);
      return HCCMF_OK;
    case HCCMF_OPT_STALENESS:
      if (value < 0) return fail(h, HCCMF_EINVAL, "staleness budget must be >= 0");
      h->opt_staleness = value;
      return HCCMF_OK;
    case HCCMF_OPT_CONFLICT_RATIO:
      if (value < 0) return fail(h, HCCMF_EINVAL, "conflict ratio must be >= 0");
      h->opt_conflict = value;
      return HCCMF_OK;
    default:
      return fail(h, HCCMF_EINVAL, "unknown option %d", option);
  }
}

void hccmf_destroy(hccmf_t h) {
  if (!h) return;
  cudaSetDevice(h->device);
  if (h->stream) cudaStreamSynchronize(h->stream);
  free_partition(h);
  dfree(h, h->d_in_u, h->nnz_in);
  dfree(h, h->d_in_v, h->nnz_in);
  dfree(h, h->d_in_r, h->nnz_in);
  dfree(h, h->d_partials, 2 * RMSE_BLOCKS);
  dfree(h, h->d_scalar, 2);
  if (h->d_wire) cudaFreeAsync(h->d_wire, h->stream);
  timeline_clear(h);
  for (auto e : h->ev_done) cudaEventDestroy(e);
  for (auto e : h->ev_recv) cudaEventDestroy(e);
  if (h->comm_stream) {
    cudaStreamSynchronize(h->comm_stream);
    cudaStreamDestroy(h->comm_stream);
  }
  delete h->comm;
  if (getenv("HCCMF_TRIM")) trim_pool(h);
  if (h->stream) cudaStreamSynchronize(h->stream);
  if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
  delete h;
}

namespace {
hccmf_status load_impl(hccmf_t h, const int32_t* u, const int32_t* v, const float* r, int64_t nnz, bool sliced) {
  if (nnz < 0) return fail(h, HCCMF_EINVAL, "nnz must be >= 0");
  if (nnz > 0 && (!u || !v || !r)) return fail(h, HCCMF_EINVAL, "NULL rating array");
  free_partition(h);
  dfree(h, h->d_in_u, h->nnz_in);
  dfree(h, h->d_in_v, h->nnz_in);
  dfree(h, h->d_in_r, h->nnz_in);
  if (h->transposed) {  // back to the caller's orientation
    std::swap(h->m, h->n);
    h->transposed = false;
  }
  h->state = 0;
  h->nnz = nnz;
  h->nnz_in = nnz;
  h->sliced = sliced && h->world > 1;
  CU(h, dmalloc(h, &h->d_in_u, nnz));
  CU(h, dmalloc(h, &h->d_in_v, nnz));
  CU(h, dmalloc(h, &h->d_in_r, nnz));
  if (!h->d_scalar) CU(h, dmalloc(h, &h->d_scalar, 2));
  if (nnz) {
    CU(h, cudaMemcpyAsync(h->d_in_u, u, sizeof(int32_t) * nnz, cudaMemcpyDefault, h->stream));
    CU(h, cudaMemcpyAsync(h->d_in_v, v, sizeof(int32_t) * nnz, cudaMemcpyDefault, h->stream));
    CU(h, cudaMemcpyAsync(h->d_in_r, r, sizeof(float) * nnz, cudaMemcpyDefault, h->stream));
    unsigned int* flag = reinterpret_cast<unsigned int*>(h->d_scalar);
    CU(h, cudaMemsetAsync(flag, 0, sizeof(unsigned int), h->stream));
    CU(h, k_validate(h->d_in_u, h->d_in_v, h->d_in_r, nnz, h->m, h->n, flag, h->stream));
    unsigned int bad = 0;
    CU(h, cudaMemcpyAsync(&bad, flag, sizeof(bad), cudaMemcpyDeviceToHost, h->stream));
    CU(h, cudaStreamSynchronize(h->stream));
    if (bad) {
      h->nnz = 0;
      h->nnz_in = 0;
      return fail(h, HCCMF_ERANGE, "invalid ratings:%s%s%s", (bad & 1) ? " u out of [0,m)" : "",
                  (bad & 2) ? " v out of [0,n)" : "", (bad & 4) ? " non-finite r" : "");
    }
  }
  h->state = 1;
  return finish(h);
}
}  // namespace

hccmf_status hccmf_load_ratings(hccmf_t h, const int32_t* u, const int32_t* v, const float* r, int64_t nnz) {
  ENTER(h);
  return load_impl(h, u, v, r, nnz, false);
}

hccmf_status hccmf_load_ratings_slice(hccmf_t h, const int32_t* u, const int32_t* v, const float* r,
                                      int64_t nnz_local) {
  ENTER(h);
  return load_impl(h, u, v, r, nnz_local, true);
}

hccmf_status hccmf_partition(hccmf_t h, const hccmf_partition_opts* o) {
  ENTER(h);
  if (!o) return fail(h, HCCMF_EINVAL, "opts is NULL");
  if (h->state < 1 || !h->d_in_u) return fail(h, HCCMF_ESTATE, "partition needs load_ratings first");
  const int G = o->n_shards;
  if (G < 1) return fail(h, HCCMF_EINVAL, "n_shards must be >= 1");
  if (h->world > 1 && G != h->world) return fail(h, HCCMF_EINVAL, "n_shards must equal the world size");
  if (o->grid_rows < 1 || o->grid_cols < 1) return fail(h, HCCMF_EINVAL, "grid must be >= 1 x 1");
  if (o->storage < 0 || o->storage > 2) return fail(h, HCCMF_EINVAL, "storage must be 0 (fp32), 1 (binary16 Q) or 2 (binary16 Q, stochastic rounding)");
  if (o->strategy < HCCMF_DP0 || o->strategy > HCCMF_DP2) return fail(h, HCCMF_EINVAL, "bad strategy");
  if ((o->strategy != HCCMF_DP0) && !o->t_meas) return fail(h, HCCMF_EINVAL, "DP1/DP2 need t_meas");
  if (o->grid_dim < 0 || o->grid_dim > 2) return fail(h, HCCMF_EINVAL, "grid_dim must be 0, 1 or 2");
  free_partition(h);
  // row grid or column grid (L881-L886): a column grid is the row grid of R^T with
  // the roles of P and Q swapped; only the caller-facing calls swap back
  {
    const int64_t rows_now = h->transposed ? h->n : h->m, cols_now = h->transposed ? h->m : h->n;
    const bool want_t = o->grid_dim == 1 || (o->grid_dim == 2 && cols_now > rows_now);
    if (want_t != h->transposed) {
      std::swap(h->d_in_u, h->d_in_v);
      std::swap(h->m, h->n);
      h->transposed = want_t;
    }
  }
  if (G > h->m) return fail(h, HCCMF_EINVAL, "n_shards must be <= the number of grid rows");

  // ---- a3 partition fractions (host planner, section 3.3)
  std::vector<double> x(G, 1.0 / G);
  if (o->x)
    for (int s = 0; s < G; ++s) x[s] = o->x[s];
  if (o->strategy == HCCMF_DP0 && o->t_meas) plan_dp0(G, o->t_meas, x);
  if (o->strategy == HCCMF_DP1) plan_dp1(G, x, std::vector<double>(o->t_meas, o->t_meas + G));
  if (o->strategy == HCCMF_DP2) plan_dp2(G, x, o->t_meas, o->t_sync);
  for (int s = 0; s < G; ++s)
    if (!(x[s] >= 0.0) || !std::isfinite(x[s])) return fail(h, HCCMF_EINVAL, "partition fractions must be >= 0");
  h->x = x;
  h->G = G;
  h->Br = o->grid_rows;
  h->Bc = o->grid_cols;
  h->seed = o->seed;
  h->storage = o->storage;
  const int64_t m = h->m, n = h->n;
  int64_t nnz = h->nnz_in;  // ratings held now (the global COO, or this rank's slice)
  cudaStream_t st = h->stream;

  PhaseTimer timer(h->stream);
  // ---- a2 shuffle
  CU(h, dmalloc(h, &h->d_perm_row, m));
  CU(h, dmalloc(h, &h->d_perm_col, n));
  CU(h, k_perm(h->seed, 1, m, h->d_perm_row, st));
  if (o->col_balance) {
    // R30: degree-balanced column blocks -- item degrees (global under sliced ingest), then
    // least-loaded placement in order of (degree desc, id asc), ties to the lowest block
    unsigned long long* dDeg = nullptr;
    CU(h, cudaMallocAsync((void**)&dDeg, sizeof(unsigned long long) * n, st));
    CU(h, k_item_degree(h->d_in_v, h->nnz_in, n, dDeg, st));
    if (h->sliced) {
      h->comm_counts[SITE_INGEST_HIST] += 1;
      CM(h, h->comm->allreduce(dDeg, dDeg, (size_t)n, DType::u64, ROp::sum, st));
    }
    std::vector<unsigned long long> deg(n);
    CU(h, cudaMemcpyAsync(deg.data(), dDeg, sizeof(unsigned long long) * n, cudaMemcpyDeviceToHost, st));
    CU(h, cudaStreamSynchronize(st));
    cudaFreeAsync(dDeg, st);
    std::vector<int32_t> order(n), pc(n);
    for (int64_t x = 0; x < n; ++x) order[x] = (int32_t)x;
    std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return deg[a] > deg[b]; });
    const int64_t Bc = o->grid_cols;
    std::vector<int64_t> used(Bc, 0);
    using LB = std::pair<unsigned long long, int64_t>;  // (load, block): least load, then lowest block
    std::priority_queue<LB, std::vector<LB>, std::greater<LB>> heap;
    for (int64_t c = 0; c < Bc; ++c)
      if (ceil_div((c + 1) * n, Bc) > ceil_div(c * n, Bc)) heap.push({0ull, c});
    for (int64_t x = 0; x < n; ++x) {
      const LB top = heap.top();
      heap.pop();
      const int64_t c = top.second, start = ceil_div(c * n, Bc), width = ceil_div((c + 1) * n, Bc) - start;
      pc[order[x]] = (int32_t)(start + used[c]);
      if (++used[c] < width) heap.push({top.first + deg[order[x]], c});
    }
    CU(h, cudaMemcpyAsync(h->d_perm_col, pc.data(), sizeof(int32_t) * n, cudaMemcpyHostToDevice, st));
    CU(h, cudaStreamSynchronize(st));
  } else {
    CU(h, k_perm(h->seed, 2, n, h->d_perm_col, st));
  }

  timer.mark("a2 shuffle");
  // ---- a3 row histogram, prefix, boundaries
  // (one shard: the bounds are [0, m] whatever the histogram -- skip it, C5: 3.1 B atomics)
  unsigned long long* dS = nullptr;
  if (G > 1) {
    CU(h, cudaMallocAsync((void**)&dS, sizeof(unsigned long long) * (m + 1), st));
    CU(h, k_row_prefix(h->d_in_u, nnz, h->d_perm_row, m, dS, st));
  }
  if (h->sliced) {  // the global prefix is the sum of the ranks' prefixes
    h->comm_counts[SITE_INGEST_HIST] += 1;
    CM(h, h->comm->allreduce(dS, dS, (size_t)m + 1, DType::u64, ROp::sum, st));
    unsigned long long tot = 0;
    CU(h, cudaMemcpyAsync(&tot, dS + m, sizeof(tot), cudaMemcpyDeviceToHost, st));
    CU(h, cudaStreamSynchronize(st));
    h->nnz = (int64_t)tot;
  }
  const int64_t nnz_glob = h->sliced ? h->nnz : nnz;
  std::vector<int64_t> targets(G > 1 ? G - 1 : 1, 0), rstar(G > 1 ? G - 1 : 1, 0);
  double cum = 0.0;
  for (int s = 1; s < G; ++s) {
    cum += x[s - 1];
    targets[s - 1] = llround((double)nnz_glob * cum);
  }
  h->bounds.assign(G + 1, 0);
  h->bounds[G] = (int32_t)m;
  if (G > 1) {
    int64_t *dT = nullptr, *dR = nullptr;
    CU(h, cudaMallocAsync((void**)&dT, sizeof(int64_t) * (G - 1), st));
    CU(h, cudaMallocAsync((void**)&dR, sizeof(int64_t) * (G - 1), st));
    CU(h, cudaMemcpyAsync(dT, targets.data(), sizeof(int64_t) * (G - 1), cudaMemcpyHostToDevice, st));
    CU(h, k_bound_search(dS, m, dT, G - 1, dR, st));
    CU(h, cudaMemcpyAsync(rstar.data(), dR, sizeof(int64_t) * (G - 1), cudaMemcpyDeviceToHost, st));
    CU(h, cudaStreamSynchronize(st));
    cudaFreeAsync(dT, st);
    cudaFreeAsync(dR, st);
    for (int s = 1; s < G; ++s) h->bounds[s] = (int32_t)std::max<int64_t>(h->bounds[s - 1], rstar[s - 1]);
  }
  if (dS) cudaFreeAsync(dS, st);
  int32_t* dB = nullptr;
  CU(h, cudaMallocAsync((void**)&dB, sizeof(int32_t) * (G + 1), st));
  CU(h, cudaMemcpyAsync(dB, h->bounds.data(), sizeof(int32_t) * (G + 1), cudaMemcpyHostToDevice, st));

  timer.mark("a3 histogram+bounds");
  if (h->sliced) {
    // ---- sliced ingest: every rating to the rank that owns its (permuted) row.  Each
    // source's ratings stay in input order and arrive in rank order, so the received
    // sequence is the global COO restricted to this shard, in global order.
    h->comm_counts[SITE_INGEST_EXCHANGE] += 1;
    const int me = h->rank;
    int32_t *xu = nullptr, *xv = nullptr;
    float* xr = nullptr;
    CU(h, dmalloc(h, &xu, nnz));
    CU(h, dmalloc(h, &xv, nnz));
    CU(h, dmalloc(h, &xr, nnz));
    std::vector<int64_t> mine(G), all((size_t)G * G);
    CU(h, k_shard_split(h->d_in_u, h->d_in_v, h->d_in_r, nnz, h->d_perm_row, dB, G, xu, xv, xr, mine.data(), st));
    dfree(h, h->d_in_u, nnz);
    dfree(h, h->d_in_v, nnz);
    dfree(h, h->d_in_r, nnz);
    int64_t* dcnt = nullptr;
    CU(h, cudaMallocAsync((void**)&dcnt, sizeof(int64_t) * G * G, st));
    CU(h, cudaMemcpyAsync(dcnt + (size_t)me * G, mine.data(), sizeof(int64_t) * G, cudaMemcpyHostToDevice, st));
    CM(h, h->comm->allgather(dcnt + (size_t)me * G, dcnt, sizeof(int64_t) * G, st));
    CU(h, cudaMemcpyAsync(all.data(), dcnt, sizeof(int64_t) * G * G, cudaMemcpyDeviceToHost, st));
    CU(h, cudaStreamSynchronize(st));
    cudaFreeAsync(dcnt, st);
    std::vector<int64_t> soff(G + 1, 0), roff(G + 1, 0);  // send offsets (by dest), recv offsets (by source)
    for (int p = 0; p < G; ++p) {
      soff[p + 1] = soff[p] + all[(size_t)me * G + p];
      roff[p + 1] = roff[p] + all[(size_t)p * G + me];
    }
    const int64_t got = roff[G];
    CU(h, dmalloc(h, &h->d_in_u, got));
    CU(h, dmalloc(h, &h->d_in_v, got));
    CU(h, dmalloc(h, &h->d_in_r, got));
    Comm* c = h->comm;
    CM(h, c->group_start());
    for (int p = 0; p < G; ++p) {
      if (p == me) continue;
      const int64_t ns = soff[p + 1] - soff[p], nr = roff[p + 1] - roff[p];
      if (ns) {
        CM(h, c->send(xu + soff[p], 4 * ns, p, st));
        CM(h, c->send(xv + soff[p], 4 * ns, p, st));
        CM(h, c->send(xr + soff[p], 4 * ns, p, st));
      }
      if (nr) {
        CM(h, c->recv(h->d_in_u + roff[p], 4 * nr, p, st));
        CM(h, c->recv(h->d_in_v + roff[p], 4 * nr, p, st));
        CM(h, c->recv(h->d_in_r + roff[p], 4 * nr, p, st));
      }
    }
    CM(h, c->group_end());
    if (const int64_t nm = soff[me + 1] - soff[me]) {
      CU(h, cudaMemcpyAsync(h->d_in_u + roff[me], xu + soff[me], 4 * nm, cudaMemcpyDeviceToDevice, st));
      CU(h, cudaMemcpyAsync(h->d_in_v + roff[me], xv + soff[me], 4 * nm, cudaMemcpyDeviceToDevice, st));
      CU(h, cudaMemcpyAsync(h->d_in_r + roff[me], xr + soff[me], 4 * nm, cudaMemcpyDeviceToDevice, st));
    }
    dfree(h, xu, nnz);
    dfree(h, xv, nnz);
    dfree(h, xr, nnz);
    nnz = got;
    h->nnz_in = got;
    timer.mark("sliced ingest exchange");
  }
  // ---- a4 geometry + stable sort
  BlockGeom g{};
  g.G = G;
  g.Br = h->Br;
  g.Bc = h->Bc;
  g.m = m;
  g.n = n;
  int64_t maxr = 1;
  for (int s = 0; s < G; ++s) maxr = std::max<int64_t>(maxr, ceil_div((int64_t)h->bounds[s + 1] - h->bounds[s], h->Br));
  const int64_t nblk = (int64_t)G * h->Br * h->Bc;
  g.bu = bitlen((uint64_t)(maxr - 1));
  g.bv = bitlen((uint64_t)(ceil_div(n, h->Bc) - 1));
  g.bb = bitlen((uint64_t)(nblk - 1));
  g.seed = h->seed;
  if (g.bb + g.bu + g.bv > 64) return fail(h, HCCMF_ERANGE, "sort key needs %d > 64 bits", g.bb + g.bu + g.bv);
  h->geom = g;
  int32_t *su = nullptr, *sv = nullptr;
  float* sr = nullptr;
  int64_t* dOff = nullptr;
  CU(h, dmalloc(h, &su, nnz));
  CU(h, dmalloc(h, &sv, nnz));
  CU(h, dmalloc(h, &sr, nnz));
  CU(h, cudaMallocAsync((void**)&dOff, sizeof(int64_t) * (nblk + 1), st));
  timer.mark("a4 alloc records");
  CU(h, k_block_sort(g, dB, h->d_perm_row, h->d_perm_col, h->d_in_u, h->d_in_v, h->d_in_r, nnz, su, sv, sr, dOff, st));
  timer.mark("a4 key+sort+decode");
  if (h->sliced) {  // global block offsets = the sum of the ranks' (local) offsets
    h->comm_counts[SITE_INGEST_BLOCKS] += 1;
    CM(h, h->comm->allreduce(dOff, dOff, (size_t)nblk + 1, DType::i64, ROp::sum, st));
  }
  h->block_off.assign(nblk + 1, 0);
  CU(h, cudaMemcpyAsync(h->block_off.data(), dOff, sizeof(int64_t) * (nblk + 1), cudaMemcpyDeviceToHost, st));
  CU(h, cudaStreamSynchronize(st));
  cudaFreeAsync(dOff, st);
  cudaFreeAsync(dB, st);
  dfree(h, h->d_in_u, nnz);
  dfree(h, h->d_in_v, nnz);
  dfree(h, h->d_in_r, nnz);
  timer.mark("a4 offsets + free input");
  // ---- local shard(s)
  const int64_t bps = (int64_t)h->Br * h->Bc;
  if (h->world > 1) {
    h->shard_lo = h->rank;
    h->shard_hi = h->rank + 1;
  } else {
    h->shard_lo = 0;
    h->shard_hi = G;
  }
  h->blk0 = h->shard_lo * bps;
  h->nblk_local = (h->shard_hi - h->shard_lo) * bps;
  h->rec0 = h->block_off[h->blk0];
  h->local_nnz = h->block_off[h->blk0 + h->nblk_local] - h->rec0;
  if (h->sliced) {  // the sorted records are exactly this shard's
    if (h->local_nnz != nnz)
      return fail(h, HCCMF_ESTATE, "sliced ingest: %lld records received, %lld in the shard's blocks",
                  (long long)nnz, (long long)h->local_nnz);
    h->d_u = su;
    h->d_v = sv;
    h->d_r = sr;
  } else if (h->world > 1) {
    CU(h, dmalloc(h, &h->d_u, h->local_nnz));
    CU(h, dmalloc(h, &h->d_v, h->local_nnz));
    CU(h, dmalloc(h, &h->d_r, h->local_nnz));
    if (h->local_nnz) {
      CU(h, cudaMemcpyAsync(h->d_u, su + h->rec0, 4 * h->local_nnz, cudaMemcpyDeviceToDevice, st));
      CU(h, cudaMemcpyAsync(h->d_v, sv + h->rec0, 4 * h->local_nnz, cudaMemcpyDeviceToDevice, st));
      CU(h, cudaMemcpyAsync(h->d_r, sr + h->rec0, 4 * h->local_nnz, cudaMemcpyDeviceToDevice, st));
    }
    CU(h, cudaStreamSynchronize(st));
    dfree(h, su, nnz);
    dfree(h, sv, nnz);
    dfree(h, sr, nnz);
  } else {
    h->d_u = su;
    h->d_v = sv;
    h->d_r = sr;
  }
  h->row0 = h->bounds[h->shard_lo];
  h->rows = (int64_t)h->bounds[h->shard_hi] - h->row0;

  timer.mark("local shard");
  {  // rating scale of the shard (R32: the Hogwild staleness budget)
    double* dss = nullptr;
    CU(h, cudaMallocAsync((void**)&dss, sizeof(double), st));
    CU(h, k_sum_sq(h->d_r, h->local_nnz, dss, st));
    double ss = 0.0;
    CU(h, cudaMemcpyAsync(&ss, dss, sizeof(double), cudaMemcpyDeviceToHost, st));
    CU(h, cudaStreamSynchronize(st));
    cudaFreeAsync(dss, st);
    h->r_rms = h->local_nnz > 0 ? std::sqrt(ss / (double)h->local_nnz) : 0.0;
  }
  // ---- Hogwild tasks: user-aligned runs of ~opt_task ratings inside each block
  std::vector<int64_t> loc_off(h->nblk_local + 1);
  for (int64_t j = 0; j <= h->nblk_local; ++j) loc_off[j] = h->block_off[h->blk0 + j] - h->rec0;
  int64_t* dLoc = nullptr;
  CU(h, cudaMallocAsync((void**)&dLoc, sizeof(int64_t) * (h->nblk_local + 1), st));
  CU(h, cudaMemcpyAsync(dLoc, loc_off.data(), sizeof(int64_t) * (h->nblk_local + 1), cudaMemcpyHostToDevice, st));
  int64_t nt = 0;
  CU(h, k_build_tasks(h->d_u, h->local_nnz, dLoc, h->nblk_local, h->opt_task, h->opt_heavy, &h->d_task_lo, &h->d_task_hi, &nt, st));
  h->device_bytes += 2 * sizeof(int64_t) * (nt ? nt : 1);
  h->n_tasks = nt;
  cudaFreeAsync(dLoc, st);
  // local block offsets stay on the device for the DET wavefront
  CU(h, dmalloc(h, &h->d_blk_off, h->nblk_local + 1));
  CU(h, cudaMemcpyAsync(h->d_blk_off, loc_off.data(), sizeof(int64_t) * (h->nblk_local + 1), cudaMemcpyHostToDevice, st));
  CU(h, dmalloc(h, &h->d_progress, (size_t)h->Br * kProgressStride));
  // tasks are grouped by block (LPT order inside a block): the first task of every block
  h->blk_task_off.assign(h->nblk_local + 1, 0);
  CU(h, k_task_block_offsets(h->d_task_lo, nt, h->d_blk_off, h->nblk_local, h->blk_task_off.data(), st));

  timer.mark("hogwild tasks");
  // ---- factors
  CU(h, dmalloc(h, &h->d_P, h->rows * h->k));
  CU(h, dmalloc(h, &h->d_Q, h->n * h->k));
  if (!h->d_partials) CU(h, dmalloc(h, &h->d_partials, 2 * RMSE_BLOCKS));
  h->q_ring_sched = -1;
  h->state = 2;
  timer.mark("factors alloc");
  return finish(h);
}

hccmf_status hccmf_init_factors(hccmf_t h, uint64_t seed) {
  ENTER(h);
  if (h->state < 2) return fail(h, HCCMF_ESTATE, "init_factors needs partition first");
  // R5: users draw from tag 3, items from tag 4, whatever the grid orientation
  const uint64_t trow = h->transposed ? 4 : 3, tcol = h->transposed ? 3 : 4;
  CU(h, k_init_factors(seed, trow, h->m, h->k, h->d_perm_row, h->row0, h->rows, h->d_P, h->stream));
  CU(h, k_init_factors(seed, tcol, h->n, h->k, h->d_perm_col, 0, h->n, h->d_Q, h->stream));
  h->q_ring_sched = -1;
  h->state = 3;
  h->epoch = 0;
  return finish(h);
}

hccmf_status hccmf_set_factors(hccmf_t h, const float* P, const float* Q) {
  ENTER(h);
  if (h->state < 2) return fail(h, HCCMF_ESTATE, "set_factors needs partition first");
  if (!P || !Q) return fail(h, HCCMF_EINVAL, "P and Q are required");
  if (h->transposed) std::swap(P, Q);
  const size_t mk = (size_t)h->m * h->k, nk = (size_t)h->n * h->k;
  float* tmp = nullptr;
  CU(h, cudaMallocAsync((void**)&tmp, sizeof(float) * std::max(mk, nk), h->stream));
  CU(h, cudaMemcpyAsync(tmp, P, sizeof(float) * mk, cudaMemcpyDefault, h->stream));
  CU(h, k_scatter_rows(tmp, h->m, h->k, h->d_perm_row, h->row0, h->rows, h->d_P, h->stream));
  CU(h, cudaMemcpyAsync(tmp, Q, sizeof(float) * nk, cudaMemcpyDefault, h->stream));
  CU(h, k_scatter_rows(tmp, h->n, h->k, h->d_perm_col, 0, h->n, h->d_Q, h->stream));
  cudaFreeAsync(tmp, h->stream);
  h->q_ring_sched = -1;
  h->state = 3;
  h->epoch = 0;
  return finish(h);
}

hccmf_status hccmf_train_epoch(hccmf_t h, hccmf_sched sched, hccmf_sync sync) {
  ENTER(h);
  if (h->state < 3) return fail(h, HCCMF_ESTATE, "train_epoch needs factors (init_factors or set_factors)");
  if (sched != HCCMF_SCHED_DET && sched != HCCMF_SCHED_HOGWILD) return fail(h, HCCMF_EINVAL, "bad schedule");
  if (sync < HCCMF_SYNC_NONE || sync > HCCMF_SYNC_ALLREDUCE_AVG) return fail(h, HCCMF_EINVAL, "bad sync");
  const int G = h->G;
  if (h->storage >= 1) {  // binary16 Q lives in the warp-per-rating kernel (one rating per warp)
    int L = 0, VEC = 0;
    sgd_geometry(h->k, (int)h->opt_vec, &L, &VEC);
    if (L != 32 || L * VEC * 4 != h->k)
      return fail(h, HCCMF_EINVAL, "binary16 Q storage needs one rating per warp (k a multiple of 128, vec = k/128)");
  }
  int chain_ng = 0, chain_su = 0;
  if (sched == HCCMF_SCHED_DET && G == 1 && h->opt_wave == 3 && h->storage == 0 && h->Br == h->Bc && h->Br > 1 &&
      h->local_nnz > 0 && det_chain_plan(h->k, h->Br, h->n, &chain_ng, &chain_su)) {
    // DET as the chain-parallel wavefront: the same per-row update sequences as the strata (R19)
    DetChain& dc = h->det_chain;
    if (dc.B != h->Br || dc.NG != chain_ng || dc.SU != chain_su) {
      det_chain_free(&dc, h->stream);
      cudaError_t e = k_det_chain_schedule(h->d_u, h->d_v, h->d_r, h->d_blk_off, h->nblk_local, h->Bc, h->n, chain_ng,
                                           chain_su, &dc, h->stream);
      if (e != cudaSuccess) {
        det_chain_free(&dc, h->stream);
        CU(h, e);
      }
      dc.B = h->Br;
    }
    cudaError_t e = launch_wave_chain(dc, h->d_P, h->d_Q, h->row0, h->n, h->k, h->gamma, h->lambda, h->Br,
                                      h->d_progress, h->stream);
    if (e == cudaSuccess) {
      h->det_path = 3;
      ++h->epoch;
      return finish(h);
    }
    if (e != cudaErrorCooperativeLaunchTooLarge) CU(h, e);
    cudaGetLastError();
  }
  const bool wave_slab = sched == HCCMF_SCHED_DET && G == 1 && (h->opt_wave == 1 || h->opt_wave == 3) && h->storage == 0 &&
                         h->Br == h->Bc && h->Br > 1 && wave_slab_supported(h->k, (int)h->opt_vec, h->Br, h->n);
  if (wave_slab || (sched == HCCMF_SCHED_DET && G == 1 && h->opt_wave && h->storage == 0 && h->Br == h->Bc &&
                    h->Br > 1 && wave_supported(h->k, (int)h->opt_vec, h->Br))) {
    // DET as one wavefront kernel: same order of updates as the strata (R19)
    SgdArgs a{};
    a.ru = h->d_u;
    a.rv = h->d_v;
    a.rr = h->d_r;
    a.P = h->d_P;
    a.Q = h->d_Q;
    a.row0 = h->row0;
    a.k = h->k;
    a.gamma = h->gamma;
    a.lambda = h->lambda;
    a.vec_pref = (int32_t)h->opt_vec;
    a.prefetch = 1;
    cudaError_t e = wave_slab ? launch_wave_slab(a, h->d_blk_off, h->Br, h->d_progress, h->n, h->stream)
                              : launch_wave(a, h->d_blk_off, h->Br, h->d_progress, h->stream);
    if (e == cudaSuccess) {
      h->det_path = wave_slab ? 1 : 2;
      ++h->epoch;
      return finish(h);
    }
    // the cooperative launch could not make every CTA co-resident (another workload holds
    // SMs): nothing ran; the per-stratum launches below compute the same epoch
    if (e != cudaErrorCooperativeLaunchTooLarge) CU(h, e);
    cudaGetLastError();
  }
  Plan* pl = nullptr;
  hccmf_status st = build_plan(h, sched, sync, &pl);
  if (st != HCCMF_OK) return st;
  if (sched == HCCMF_SCHED_DET) h->det_path = 0;
  timeline_clear(h);
  const int eff_sync = (G == 1) ? HCCMF_SYNC_NONE : sync;
  const bool dist = h->world > 1;
  const int64_t nk = h->n * h->k;
  cudaStream_t s = h->stream;
  if (eff_sync != HCCMF_SYNC_RING || h->q_ring_sched != sched) {
    st = materialize_q(h);
    if (st != HCCMF_OK) return st;
  }
  const int nrep = h->shard_hi - h->shard_lo;
  auto replicate = [&]() -> hccmf_status {  // logical all-reduce: every shard starts from Q
    if (!h->d_Qrep) CU(h, dmalloc(h, &h->d_Qrep, (size_t)nk * nrep));
    for (int r = 0; r < nrep; ++r)
      CU(h, cudaMemcpyAsync(h->d_Qrep + (size_t)r * nk, h->d_Q, sizeof(float) * nk, cudaMemcpyDeviceToDevice, s));
    return HCCMF_OK;
  };
  auto average = [&]() -> hccmf_status {  // the server's sync (L549-L557): Q = mean of the shards' Q
    const int trow = timeline_begin(h, 3, -1, -1, s);
    struct End {
      hccmf_t h;
      int row;
      cudaStream_t s;
      ~End() { timeline_end(h, row, s); }
    } end_{h, trow, s};
    if (dist && h->opt_wire16) {  // Strategy 2: the copies travel and come back as binary16
      hccmf_status w = allreduce_q16(h, s);
      if (w != HCCMF_OK) return w;
    } else if (dist) {
      h->comm_counts[SITE_ALLREDUCE_Q] += 1;
      CM(h, h->comm->allreduce(h->d_Q, h->d_Q, (size_t)nk, DType::f32, ROp::avg, s));
    } else if (h->opt_wire16) {
      CU(h, k_average_half(h->d_Qrep, nrep, nk, h->d_Q, s));
    } else {
      CU(h, k_average(h->d_Qrep, nrep, nk, h->d_Q, s));
    }
    return HCCMF_OK;
  };
  // logical ring + Strategy 2: every column group moves once per stage, i.e. all of Q
  // passes through binary16 at each stage boundary
  const bool logical_wire = !dist && eff_sync == HCCMF_SYNC_RING && h->opt_wire16;
  // Storage = 1 (R26): while launches run, the binary16 copy d_Qh of rows [qh_a, qh_b)
  // of the fp32 matrix qh_of is the authoritative Q; it is rounded in before the first
  // launch that needs it and written back (exactly: binary16 values are fp32 values)
  // before anything else reads or moves Q (a ring transfer, an average, the next
  // replica, the end of the epoch).
  float* qh_of = nullptr;
  int64_t qh_a = 0, qh_b = 0;
  if (h->storage >= 1 && !h->d_Qh) CU(h, dmalloc(h, &h->d_Qh, (size_t)nk));
  auto qh_flush = [&]() -> hccmf_status {
    if (qh_of && qh_b > qh_a)
      CU(h, k_unpack_half(h->d_Qh + qh_a * h->k, qh_of + qh_a * h->k, (qh_b - qh_a) * h->k, s));
    qh_of = nullptr;
    return HCCMF_OK;
  };
  auto qh_enter = [&](float* q, int64_t a0, int64_t b0) -> hccmf_status {
    if (qh_of == q && qh_a == a0 && qh_b == b0) return HCCMF_OK;
    hccmf_status f = qh_flush();
    if (f != HCCMF_OK) return f;
    if (b0 > a0) CU(h, k_pack_half(q + a0 * h->k, h->d_Qh + a0 * h->k, (b0 - a0) * h->k, s));
    qh_of = q;
    qh_a = a0;
    qh_b = b0;
    return HCCMF_OK;
  };
  if (eff_sync == HCCMF_SYNC_ALLREDUCE_AVG && !dist) {
    st = replicate();
    if (st != HCCMF_OK) return st;
  }
  CU(h, cudaMemsetAsync(h->d_counters, 0, sizeof(unsigned long long) * pl->launches.size(), s));
  SgdArgs a{};
  a.ru = h->d_u;
  a.rv = h->d_v;
  a.rr = h->d_r;
  a.P = h->d_P;
  a.row0 = h->row0;
  a.k = h->k;
  a.gamma = h->gamma;
  a.lambda = h->lambda;
  a.atomic_q = (sched == HCCMF_SCHED_HOGWILD && h->opt_atomic) ? 1 : 0;
  a.vec_pref = (int32_t)h->opt_vec;
  a.prefetch = sched == HCCMF_SCHED_DET ? 1 : 0;
  a.depth = (sched == HCCMF_SCHED_HOGWILD && h->storage == 0) ? (int32_t)h->opt_depth : 1;
  a.qhalf = h->storage;
  a.rec0 = h->rec0;
  a.epoch = h->epoch;
  const int L = sgd_lanes(h->k, (int)h->opt_vec);
  if (dist && eff_sync == HCCMF_SYNC_RING && sched == HCCMF_SCHED_HOGWILD) {
    const size_t ne = (size_t)G * (h->Bc / G);
    if (pl->launches.size() != ne) return fail(h, HCCMF_EINVAL, "ring plan: one launch per column block expected");
    if (!h->comm_stream) CU(h, cudaStreamCreateWithFlags(&h->comm_stream, cudaStreamNonBlocking));
    while (h->ev_done.size() < ne) {
      cudaEvent_t a0, a1;
      CU(h, cudaEventCreateWithFlags(&a0, cudaEventDisableTiming));
      CU(h, cudaEventCreateWithFlags(&a1, cudaEventDisableTiming));
      h->ev_done.push_back(a0);
      h->ev_recv.push_back(a1);
    }
    // the comm stream must not run ahead of work already queued on the compute stream
    CU(h, cudaEventRecord(h->ev_done[0], s));
    CU(h, cudaStreamWaitEvent(h->comm_stream, h->ev_done[0], 0));
  }
  // Keep Q resident in L2 across the epoch: a persisting access-policy
  // window over Q on the launch stream, so the 1.2 GB record stream and the P rows
  // do not evict q_v lines between a group's load and its red.
  const bool persist = h->opt_l2persist && sched == HCCMF_SCHED_HOGWILD;
  if (persist) {
    int max_win = 0, max_persist = 0;
    cudaDeviceGetAttribute(&max_win, cudaDevAttrMaxAccessPolicyWindowSize, h->device);
    cudaDeviceGetAttribute(&max_persist, cudaDevAttrMaxPersistingL2CacheSize, h->device);
    const size_t qbytes = sizeof(float) * (size_t)nk;
    const size_t win = std::min(qbytes, (size_t)std::max(0, max_win));
    if (win > 0 && max_persist > 0) {
      cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, std::min(win, (size_t)max_persist));
      cudaStreamAttrValue v{};
      v.accessPolicyWindow.base_ptr = h->d_Q;
      v.accessPolicyWindow.num_bytes = win;
      v.accessPolicyWindow.hitRatio = std::min(1.0f, (float)max_persist / (float)win);
      v.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
      v.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
      cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v);
    }
    cudaGetLastError();
  }
  int stage = 0;
  int phase = 0;
  for (size_t li = 0; li < pl->launches.size(); ++li) {
    const Launch& ln = pl->launches[li];
    if (eff_sync == HCCMF_SYNC_ALLREDUCE_AVG && ln.phase != phase) {  // sub-epoch sync (R22)
      st = qh_flush();
      if (st != HCCMF_OK) return st;
      st = average();
      if (st != HCCMF_OK) return st;
      if (!dist) {
        st = replicate();
        if (st != HCCMF_OK) return st;
      }
      phase = ln.phase;
    }
    const bool pipelined = dist && eff_sync == HCCMF_SYNC_RING && sched == HCCMF_SCHED_HOGWILD;
    int jblk = 0;  // column block of this launch inside its stage (HOGWILD ring plans: one each)
    if (pipelined) {
      jblk = (int)(li % (size_t)(h->Bc / G));
      if (ln.stage > 0) CU(h, cudaStreamWaitEvent(s, h->ev_recv[(size_t)(ln.stage - 1) * (h->Bc / G) + jblk], 0));
    } else if (dist && eff_sync == HCCMF_SYNC_RING) {
      if (stage < ln.stage) {
        st = qh_flush();
        if (st != HCCMF_OK) return st;
      }
      while (stage < ln.stage) {
        st = ring_exchange(h, sched, stage++);
        if (st != HCCMF_OK) return st;
      }
    } else if (logical_wire) {  // binary16 storage: Q is already binary16, the rounding is the identity
      for (; stage < ln.stage; ++stage)
        if (h->storage == 0) CU(h, k_round_half(h->d_Q, nk, s));
    }
    a.Q = (eff_sync == HCCMF_SYNC_ALLREDUCE_AVG && !dist) ? h->d_Qrep + (size_t)ln.qrep * nk : h->d_Q;
    if (h->storage >= 1) {
      // rows this launch may touch: its column block (pipelined ring), its column group
      // (stage-wise ring), else all of Q
      int64_t ra = 0, rb = h->n;
      if (pipelined) {
        const int64_t cb = (int64_t)((h->rank + ln.stage) % G) * (h->Bc / G) + jblk;
        ra = ceil_div(cb * h->n, h->Bc);
        rb = ceil_div((cb + 1) * h->n, h->Bc);
      } else if (dist && eff_sync == HCCMF_SYNC_RING) {
        ring_group_cols(h, sched, (h->rank + ln.stage) % G, &ra, &rb);
      }
      st = qh_enter(a.Q, ra, rb);
      if (st != HCCMF_OK) return st;
      a.Q = reinterpret_cast<float*>(h->d_Qh);
    }
    a.task_lo = pl->d_lo + ln.t0;
    a.task_hi = pl->d_hi + ln.t0;
    a.n_tasks = ln.nt;
    a.counter = h->d_counters + li;
    // DET: one rating group per block of the stratum; HOGWILD: persistent grid
    // Hogwild races only on the Q rows of the launch's column blocks (R14, R28)
    const int64_t warps = (sched == HCCMF_SCHED_DET) ? (ln.nt * L + 31) / 32 : auto_warps(h, ln.items);
    const int trow = timeline_begin(h, 0, ln.stage, pipelined ? jblk : (int)li, s);
    CU(h, launch_sgd(a, warps, s));
    timeline_end(h, trow, s);
    if (pipelined) {
      st = qh_flush();  // the block travels as fp32 (or binary16 wire) right after its launch
      if (st != HCCMF_OK) return st;
      const size_t e = (size_t)ln.stage * (h->Bc / G) + jblk;
      CU(h, cudaEventRecord(h->ev_done[e], s));
      CU(h, cudaStreamWaitEvent(h->comm_stream, h->ev_done[e], 0));
      st = ring_exchange_block(h, ln.stage, jblk, h->comm_stream);
      if (st != HCCMF_OK) return st;
      CU(h, cudaEventRecord(h->ev_recv[e], h->comm_stream));
    }
  }
  st = qh_flush();
  if (st != HCCMF_OK) return st;
  if (dist && eff_sync == HCCMF_SYNC_RING && sched == HCCMF_SCHED_HOGWILD) {
    // every transfer of the last stage lands before the epoch ends (shard s holds group s)
    const int c = h->Bc / G;
    for (int j = 0; j < c; ++j) CU(h, cudaStreamWaitEvent(s, h->ev_recv[(size_t)(G - 1) * c + j], 0));
    h->q_ring_sched = sched;
  } else if (dist && eff_sync == HCCMF_SYNC_RING) {
    while (stage < pl->n_stages) {
      st = ring_exchange(h, sched, stage++);
      if (st != HCCMF_OK) return st;
    }
    h->q_ring_sched = sched;
  }
  if (persist) {  // drop the window again: the stream may be the caller's
    cudaStreamAttrValue v{};
    v.accessPolicyWindow.num_bytes = 0;
    cudaStreamSetAttribute(s, cudaStreamAttributeAccessPolicyWindow, &v);
    cudaGetLastError();
  }
  if (logical_wire)
    for (; stage < pl->n_stages; ++stage) CU(h, k_round_half(h->d_Q, nk, s));
  if (eff_sync == HCCMF_SYNC_ALLREDUCE_AVG) {
    st = average();
    if (st != HCCMF_OK) return st;
  }
  ++h->epoch;
  return finish(h);
}

hccmf_status hccmf_rmse(hccmf_t h, const int32_t* u, const int32_t* v, const float* r, int64_t nt, double* out) {
  ENTER(h);
  if (!out) return fail(h, HCCMF_EINVAL, "out is NULL");
  if (h->state < 3) return fail(h, HCCMF_ESTATE, "rmse needs factors");
  if (nt < 0 || (nt > 0 && (!u || !v || !r))) return fail(h, HCCMF_EINVAL, "bad test set");
  if (h->transposed) std::swap(u, v);
  hccmf_status st = materialize_q(h);
  if (st != HCCMF_OK) return st;
  cudaStream_t s = h->stream;
  int32_t *du = nullptr, *dv = nullptr;
  float* dr = nullptr;
  CU(h, cudaMallocAsync((void**)&du, 4 * (nt ? nt : 1), s));
  CU(h, cudaMallocAsync((void**)&dv, 4 * (nt ? nt : 1), s));
  CU(h, cudaMallocAsync((void**)&dr, 4 * (nt ? nt : 1), s));
  if (nt) {
    CU(h, cudaMemcpyAsync(du, u, 4 * nt, cudaMemcpyDefault, s));
    CU(h, cudaMemcpyAsync(dv, v, 4 * nt, cudaMemcpyDefault, s));
    CU(h, cudaMemcpyAsync(dr, r, 4 * nt, cudaMemcpyDefault, s));
    unsigned int* flag = reinterpret_cast<unsigned int*>(h->d_partials);
    CU(h, cudaMemsetAsync(flag, 0, sizeof(unsigned int), s));
    CU(h, k_validate(du, dv, dr, nt, h->m, h->n, flag, s));
    unsigned int bad = 0;
    CU(h, cudaMemcpyAsync(&bad, flag, sizeof(bad), cudaMemcpyDeviceToHost, s));
    CU(h, cudaStreamSynchronize(s));
    if (bad) {
      cudaFreeAsync(du, s);
      cudaFreeAsync(dv, s);
      cudaFreeAsync(dr, s);
      return fail(h, HCCMF_ERANGE, "invalid test ratings");
    }
  }
  CU(h, k_rmse(du, dv, dr, nt, h->d_perm_row, h->d_perm_col, h->d_P, h->row0, h->rows, h->d_Q, h->k, h->d_partials,
               h->d_scalar, s));
  if (h->world > 1) {
    h->comm_counts[SITE_RMSE] += 1;
    CM(h, h->comm->allreduce(h->d_scalar, h->d_scalar, 2, DType::f64, ROp::sum, s));
  }
  double sc[2] = {0.0, 0.0};
  CU(h, cudaMemcpyAsync(sc, h->d_scalar, sizeof(sc), cudaMemcpyDeviceToHost, s));
  CU(h, cudaStreamSynchronize(s));
  cudaFreeAsync(du, s);
  cudaFreeAsync(dv, s);
  cudaFreeAsync(dr, s);
  *out = sc[1] > 0.0 ? std::sqrt(sc[0] / sc[1]) : 0.0;
  return finish(h);
}

hccmf_status hccmf_get_factors(hccmf_t h, float* P, float* Q) {
  ENTER(h);
  if (h->state < 3) return fail(h, HCCMF_ESTATE, "get_factors needs factors");
  if (h->transposed) std::swap(P, Q);
  cudaStream_t s = h->stream;
  const size_t mk = (size_t)h->m * h->k, nk = (size_t)h->n * h->k;
  if (P) {
    float* full = h->d_P;
    float* tmp = nullptr;
    if (h->world > 1) {  // final push of P (L1205-L1206): every shard's rows to every rank
      CU(h, cudaMallocAsync((void**)&full, sizeof(float) * mk, s));
      h->comm_counts[SITE_EXPORT_P] += 1;
      CM(h, h->comm->group_start());
      for (int g = 0; g < h->G; ++g) {
        const int64_t a = h->bounds[g], b = h->bounds[g + 1];
        if (b > a) {
          const float* src = (g == h->rank) ? h->d_P : full + a * h->k;
          CM(h, h->comm->broadcast(src, full + a * h->k, sizeof(float) * (size_t)(b - a) * h->k, g, s));
        }
      }
      CM(h, h->comm->group_end());
    }
    CU(h, cudaMallocAsync((void**)&tmp, sizeof(float) * mk, s));
    CU(h, k_gather_rows(full, h->m, h->k, h->d_perm_row, 0, tmp, s));
    CU(h, cudaMemcpyAsync(P, tmp, sizeof(float) * mk, cudaMemcpyDefault, s));
    CU(h, cudaStreamSynchronize(s));
    cudaFreeAsync(tmp, s);
    if (full != h->d_P) cudaFreeAsync(full, s);
  }
  if (Q) {
    hccmf_status st = materialize_q(h);
    if (st != HCCMF_OK) return st;
    float* tmp = nullptr;
    CU(h, cudaMallocAsync((void**)&tmp, sizeof(float) * nk, s));
    CU(h, k_gather_rows(h->d_Q, h->n, h->k, h->d_perm_col, 0, tmp, s));
    CU(h, cudaMemcpyAsync(Q, tmp, sizeof(float) * nk, cudaMemcpyDefault, s));
    CU(h, cudaStreamSynchronize(s));
    cudaFreeAsync(tmp, s);
  }
  return finish(h);
}

hccmf_status hccmf_get_partition(hccmf_t h, int32_t* bounds, int64_t* block_off, int32_t* perm_row, int32_t* perm_col) {
  ENTER(h);
  if (h->state < 2) return fail(h, HCCMF_ESTATE, "get_partition needs partition");
  if (bounds) memcpy(bounds, h->bounds.data(), sizeof(int32_t) * h->bounds.size());
  if (block_off) memcpy(block_off, h->block_off.data(), sizeof(int64_t) * h->block_off.size());
  if (perm_row) CU(h, cudaMemcpyAsync(perm_row, h->d_perm_row, 4 * h->m, cudaMemcpyDefault, h->stream));
  if (perm_col) CU(h, cudaMemcpyAsync(perm_col, h->d_perm_col, 4 * h->n, cudaMemcpyDefault, h->stream));
  CU(h, cudaStreamSynchronize(h->stream));
  return finish(h);
}

hccmf_status hccmf_get_records(hccmf_t h, int32_t* u, int32_t* v, float* r) {
  ENTER(h);
  if (h->state < 2) return fail(h, HCCMF_ESTATE, "get_records needs partition");
  const int64_t c = h->local_nnz;
  if (c) {
    if (u) CU(h, cudaMemcpyAsync(u, h->d_u, 4 * c, cudaMemcpyDefault, h->stream));
    if (v) CU(h, cudaMemcpyAsync(v, h->d_v, 4 * c, cudaMemcpyDefault, h->stream));
    if (r) CU(h, cudaMemcpyAsync(r, h->d_r, 4 * c, cudaMemcpyDefault, h->stream));
  }
  CU(h, cudaStreamSynchronize(h->stream));
  return finish(h);
}

hccmf_status hccmf_get_fractions(hccmf_t h, double* x) {
  ENTER(h);
  if (h->state < 2) return fail(h, HCCMF_ESTATE, "get_fractions needs partition");
  if (!x) return fail(h, HCCMF_EINVAL, "x is NULL");
  memcpy(x, h->x.data(), sizeof(double) * h->x.size());
  return HCCMF_OK;
}

hccmf_status hccmf_schedule(int32_t G, int32_t Br, int32_t Bc, int64_t n, int32_t sched, int32_t sync, int32_t shard,
                            int64_t* blocks, int64_t* n_blocks, int64_t* launch_off, int32_t* launch_stage,
                            int64_t* n_launches, int64_t* ring) {
  if (G < 1 || Br < 1 || Bc < 1 || n < 1 || !n_blocks || !n_launches || shard < -1 || shard >= G)
    return fail(nullptr, HCCMF_EINVAL, "bad schedule arguments");
  const int lo = shard < 0 ? 0 : shard, hi = shard < 0 ? G : shard + 1;
  std::vector<BlockLaunch> bl;
  int n_stages = 1;
  const char* msg = schedule_blocks(G, Br, Bc, sched, sync, lo, hi, bl, &n_stages);
  if (msg) return fail(nullptr, HCCMF_EINVAL, "%s", msg);
  int64_t nb = 0;
  for (const auto& L : bl) nb += (int64_t)L.blocks.size();
  const int64_t cap_b = *n_blocks, cap_l = *n_launches;
  *n_blocks = nb;
  *n_launches = (int64_t)bl.size();
  if (!blocks || !launch_off || cap_b < nb || cap_l < (int64_t)bl.size()) return HCCMF_OK;  // size query
  int64_t k = 0;
  for (size_t i = 0; i < bl.size(); ++i) {
    launch_off[i] = k;
    if (launch_stage) launch_stage[i] = bl[i].stage;
    for (int64_t b : bl[i].blocks) blocks[k++] = b;
  }
  launch_off[bl.size()] = k;
  if (ring && sync == HCCMF_SYNC_RING && G > 1)
    for (int t = 0; t < G; ++t) {
      const int s = lo;
      ring_cols(n, G, Br, Bc, sched, (s + t) % G, &ring[4 * t + 0], &ring[4 * t + 1]);
      ring_cols(n, G, Br, Bc, sched, (s + t + 1) % G, &ring[4 * t + 2], &ring[4 * t + 3]);
    }
  return HCCMF_OK;
}

hccmf_status hccmf_cost_model(int32_t p, int64_t m, int64_t n, int64_t nnz, int32_t k, const double* B,
                              const double* Bbus, double B_server, int32_t t, int32_t q_only, int32_t elem_bytes,
                              double lambda_sync, double* x, double* T_i, double* T_sync, double* T,
                              int32_t* strategy) {
  if (p < 1 || m < 1 || n < 1 || nnz < 0 || k < 1 || !B || !Bbus || !x || !T_i || !T_sync || !T || !strategy ||
      !(B_server > 0.0) || t < 0 || elem_bytes < 1)
    return fail(nullptr, HCCMF_EINVAL, "bad cost model arguments");
  for (int i = 0; i < p; ++i)
    if (!(B[i] > 0.0) || !(Bbus[i] > 0.0)) return fail(nullptr, HCCMF_EINVAL, "bandwidths must be > 0");
  // section 3.2: bytes per rating 16k + 4 (L741-L742); parameters moved D k elem (R18)
  const double D = q_only ? (double)n : (double)(m + n);
  const double per_rating = 16.0 * k + 4.0;
  std::vector<double> Te(p);
  for (int i = 0; i < p; ++i) Te[i] = (double)nnz * per_rating / B[i];  // independent execution time
  std::vector<double> xv;
  plan_dp0(p, Te.data(), xv);  // Eq. 6
  double Tmax = 0.0;
  for (int i = 0; i < p; ++i) {
    x[i] = xv[i];
    T_i[i] = xv[i] * (double)nnz * per_rating / B[i] + 2.0 * elem_bytes * k * D / Bbus[i];  // Eq. 2
    Tmax = std::max(Tmax, T_i[i]);
  }
  *T_sync = 3.0 * t * elem_bytes * k * D / B_server;  // Eq. 3
  if (Tmax / *T_sync >= lambda_sync) {  // Eq. 5: synchronisation negligible -> balance (DP1)
    *T = Tmax;
    *strategy = HCCMF_DP1;
  } else {  // hide the synchronisation (DP2)
    *T = Tmax + *T_sync;
    *strategy = HCCMF_DP2;
  }
  return HCCMF_OK;
}

hccmf_status hccmf_timeline(hccmf_t h, double* rows, int64_t cap, int64_t* n) {
  ENTER(h);
  if (!n) return fail(h, HCCMF_EINVAL, "n is NULL");
  *n = (int64_t)h->timeline.size();
  if (h->timeline.empty() || !rows) return HCCMF_OK;
  CU(h, cudaStreamSynchronize(h->stream));
  if (h->comm_stream) CU(h, cudaStreamSynchronize(h->comm_stream));
  const cudaEvent_t t0 = h->timeline[0].a;
  for (int64_t i = 0; i < *n && i < cap; ++i) {
    const auto& r = h->timeline[i];
    float a = 0.f, b = 0.f;
    CU(h, cudaEventElapsedTime(&a, t0, r.a));
    CU(h, cudaEventElapsedTime(&b, t0, r.b));
    double* o = rows + 5 * i;
    o[0] = r.kind;
    o[1] = r.stage;
    o[2] = r.block;
    o[3] = a;
    o[4] = b;
  }
  return HCCMF_OK;
}

hccmf_status hccmf_probe_roundtrip(hccmf_t h, int32_t mode, int64_t warps, int32_t reps, double* ms) {
  ENTER(h);
  if (!ms || mode < 0 || mode > 9 || warps < 0 || reps < 1) return fail(h, HCCMF_EINVAL, "bad probe arguments");
  if (h->state < 2) return fail(h, HCCMF_ESTATE, "probe needs partition");
  if (h->k % 128 != 0) return fail(h, HCCMF_EINVAL, "probe needs k a multiple of 128");
  if (h->G == 1 && h->Br == 1 && h->Bc > 1) {
    // the Hogwild epoch's column-block phases (one launch each, e.g. C4): the same phases with
    // their own records and warp counts, one after the other; *ms is their sum
    double sum = 0.0;
    for (int64_t cb = 0; cb < h->Bc; ++cb) {
      const int64_t lo = h->block_off[h->blk0 + cb] - h->rec0, hi = h->block_off[h->blk0 + cb + 1] - h->rec0;
      const int64_t items = ceil_div((cb + 1) * h->n, h->Bc) - ceil_div(cb * h->n, h->Bc);
      if (hi <= lo) continue;
      float t = 0.f;
      CU(h, k_probe_roundtrip(mode, h->d_u + lo, h->d_v + lo, h->d_r + lo, hi - lo, h->k, h->n, h->d_P, h->row0,
                              h->d_Q, warps ? warps : auto_warps(h, items), reps, &t, h->stream));
      sum += t;
    }
    *ms = sum;
    return finish(h);
  }
  const int64_t w = warps ? warps : auto_warps(h, h->n);
  float t = 0.f;
  CU(h, k_probe_roundtrip(mode, h->d_u, h->d_v, h->d_r, h->local_nnz, h->k, h->n, h->d_P, h->row0, h->d_Q, w, reps, &t,
                          h->stream));
  *ms = t;
  return finish(h);
}

hccmf_status hccmf_get_info(hccmf_t h, hccmf_info* o) {
  if (!h || !o) return fail(h, HCCMF_EINVAL, "NULL argument");
  memset(o, 0, sizeof(*o));
  o->m = h->m;
  o->n = h->n;
  o->nnz = h->nnz;
  o->k = h->k;
  o->n_shards = h->G;
  o->shard_lo = h->shard_lo;
  o->shard_hi = h->shard_hi;
  o->local_nnz = h->local_nnz;
  o->row0 = h->row0;
  o->rows = h->rows;
  o->n_blocks = (int64_t)h->G * h->Br * h->Bc;
  o->n_tasks = h->n_tasks;
  o->key_bits = h->geom.bb + h->geom.bu + h->geom.bv;
  o->rank = h->rank;
  o->world = h->world;
  o->device_bytes = (int64_t)h->device_bytes;
  o->transposed = h->transposed ? 1 : 0;
  o->det_path = h->det_path;
  return HCCMF_OK;
}

}  // extern "C"
