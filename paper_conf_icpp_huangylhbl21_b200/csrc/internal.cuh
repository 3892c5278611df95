// internal.cuh -- shared declarations of libhccmf (product path; no oracle code).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <atomic>
#include <string>
#include <vector>

#include "comm.cuh"
#include "hccmf.h"

namespace hccmf {

// DET wavefront progress counters: one per 128-byte line (counter i at progress[i * kProgressStride]),
// so the warps polling their successors spread over L2 slices instead of hammering a few lines
constexpr int kProgressStride = 32;

// every <<<...>>> launch site of the library is written (note_launch(), kernel<<<...>>>(...))
// so hccmf_kernel_launches() reports what actually ran (bench.py's gpu_launches)
inline std::atomic<long long> g_kernel_launches{0};
inline void note_launch() { g_kernel_launches.fetch_add(1, std::memory_order_relaxed); }

// ------------------------------------------------------------------ hashing
// DESIGN.md R8: SplitMix64 finaliser (Steele, Lea, Flood 2014) and the
// counter-based hash H(seed, tag, a, b) = sm(sm(sm(seed ^ tag<<56) ^ a) ^ b).
__host__ __device__ __forceinline__ uint64_t splitmix(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__host__ __device__ __forceinline__ uint64_t hash4(uint64_t seed, uint64_t tag, uint64_t a, uint64_t b) {
  return splitmix(splitmix(splitmix(seed ^ (tag << 56)) ^ a) ^ b);
}
// 24-bit uniform in [0,1): exact in fp32.
__host__ __device__ __forceinline__ float uniform24(uint64_t h) {
  return (float)(uint32_t)(h >> 40) * (1.0f / 16777216.0f);
}

// --------------------------------------------------------------- SGD plans
// One kernel launch of the SGD kernel: tasks [t0, t0+nt) of the plan's task
// arrays, against Q replica `qrep` (logical all-reduce) ; `stage` = ring stage.
struct Launch {
  int64_t t0, nt;
  int32_t qrep;
  int32_t stage;
  int32_t phase;  // all-reduce sub-epoch round (R22)
  int64_t items;  // Q rows this launch's blocks may touch (distinct column blocks): the
                  // Hogwild concurrency cap of DESIGN.md R14 is taken from it
};

struct Plan {
  int sched = -1, sync = -1;
  int64_t* d_lo = nullptr;  // record ranges [lo, hi) in local record indices
  int64_t* d_hi = nullptr;
  int64_t n_tasks = 0;
  std::vector<Launch> launches;
  int32_t n_stages = 1;
  int32_t phases = 1;
};

struct SgdArgs {
  const int32_t* __restrict__ ru;
  const int32_t* __restrict__ rv;
  const float* __restrict__ rr;
  float* P;         // local P rows [row0, row0 + rows)
  float* Q;         // n x k (or one replica)
  int64_t row0;
  int32_t k;
  float gamma, lambda;
  const int64_t* __restrict__ task_lo;
  const int64_t* __restrict__ task_hi;
  int64_t n_tasks;
  unsigned long long* counter;
  int32_t atomic_q;  // Hogwild: apply q_v increments with vector atomics
  int32_t vec_pref;  // float4 slots per lane (0 = auto)
  int32_t prefetch;  // L2 bulk prefetch of the next window's p_u / q_v rows (DET blocks)
  int32_t depth;     // q_v prefetch distance in ratings (warp-per-rating Hogwild kernel)
  int32_t qhalf;     // Q is IEEE binary16: 1 round to nearest, 2 stochastic rounding (R26, R27)
  int64_t rec0;      // global index of local record 0 (SR random words)
  unsigned epoch;    // epochs since the factors were set (SR random words)
};

// launch the SGD kernel for a list of tasks; warps = concurrent warps wanted
cudaError_t launch_sgd(const SgdArgs& a, int64_t warps, cudaStream_t st);
// DET as one wavefront kernel (G == 1, square B x B grid, warp-per-rating geometry)
bool wave_supported(int k, int vec_pref, int B);
cudaError_t launch_wave(const SgdArgs& a, const int64_t* off /* local block offsets, B*B+1 */, int B,
                        int* progress /* B ints */, cudaStream_t st);
// the same wavefront with each column block's Q rows staged in shared memory
bool wave_slab_supported(int k, int vec_pref, int B, int64_t n);
cudaError_t launch_wave_slab(const SgdArgs& a, const int64_t* off, int B, int* progress, int64_t n,
                             cudaStream_t st);
// DET as the chain-parallel wavefront (detchain.cu): the per-partition schedule
struct DetChain {
  int32_t* cv = nullptr;       // records reordered group by group inside each segment
  float* cr = nullptr;
  uint32_t* meta = nullptr;    // p slot | dependency (group, index)
  int64_t* blk_seg = nullptr;  // nblk + 1: segments of each block
  int64_t* seg_lo = nullptr;   // nseg + 1: first record of each segment
  int64_t* seg_run = nullptr;  // nseg + 1: first user run of each segment
  uint16_t* seg_gend = nullptr;// 4 per segment: group ends inside the segment
  int32_t* run_user = nullptr; // nrun: the user of each run
  int64_t nseg = 0, nrun = 0, nrec = 0;
  int NG = 0, SU = 0, B = 0;
};
bool det_chain_plan(int k, int B, int64_t n, int* NG, int* SU);
cudaError_t k_det_chain_schedule(const int32_t* ru, const int32_t* rv, const float* rr, const int64_t* off,
                                 int64_t nblk, int Bc, int64_t n, int NG, int SU, DetChain* out, cudaStream_t st);
void det_chain_free(DetChain* d, cudaStream_t st);
cudaError_t launch_wave_chain(const DetChain& d, float* P, float* Q, int64_t row0, int64_t n, int32_t k, float gamma,
                              float lambda, int B, int* progress, cudaStream_t st);
// lane geometry of the SGD kernel: L lanes per rating group, VEC float4 per lane
void sgd_geometry(int k, int vec_pref, int* L, int* VEC);
int sgd_lanes(int k, int vec_pref);
// Hogwild rating groups per warp (1 for the warp-per-rating kernels)
int hogwild_groups_per_warp(int k, int vec_pref);
// lanes per rating of the RMSE kernel (one float4 per lane)
int lanes_per_rating(int k);

// ---------------------------------------------------------------- blocker
struct BlockGeom {  // a4 block geometry for the bit-exact sort key
  int32_t G, Br, Bc;
  int64_t m, n;
  int32_t bu, bv, bb;  // key bits: local row, local col, block id
  uint64_t seed;       // row-dependent column rotation inside a block (R21)
};

cudaError_t k_validate(const int32_t* u, const int32_t* v, const float* r, int64_t nnz, int64_t m,
                       int64_t n, unsigned int* flag, cudaStream_t st);
cudaError_t k_perm(uint64_t seed, uint64_t tag, int64_t count, int32_t* perm, cudaStream_t st);
cudaError_t k_row_prefix(const int32_t* u, int64_t nnz, const int32_t* perm_row, int64_t m,
                         unsigned long long* S /* m+1 */, cudaStream_t st);
cudaError_t k_item_degree(const int32_t* v, int64_t nnz, int64_t n, unsigned long long* deg /* n */, cudaStream_t st);
cudaError_t k_bound_search(const unsigned long long* S, int64_t m, const int64_t* targets, int32_t nt,
                           int64_t* out, cudaStream_t st);
cudaError_t k_block_sort(const BlockGeom& g, const int32_t* bounds, const int32_t* perm_row,
                         const int32_t* perm_col, const int32_t* u, const int32_t* v, const float* r,
                         int64_t nnz, int32_t* ou, int32_t* ov, float* orr, int64_t* block_off,
                         cudaStream_t st);
// sliced ingest: stable split of n ratings by the shard owning perm_row[u] (bounds on the
// device, G + 1); out_* receive them grouped by shard in input order, counts[G] (host)
cudaError_t k_shard_split(const int32_t* u, const int32_t* v, const float* r, int64_t nnz, const int32_t* perm_row,
                          const int32_t* bounds, int32_t G, int32_t* ou, int32_t* ov, float* orr, int64_t* counts,
                          cudaStream_t st);
cudaError_t k_build_tasks(const int32_t* ru, int64_t nrec, const int64_t* blk_off_local /*nb+1, local idx*/,
                          int64_t nb, int64_t target, int64_t heavy, int64_t** task_lo, int64_t** task_hi, int64_t* n_tasks,
                          cudaStream_t st);
// blk_task_off (host, nb + 1): the first task of every block (tasks are grouped by block; a
// block without tasks starts where the next one does), computed on the device
cudaError_t k_task_block_offsets(const int64_t* task_lo, int64_t nt, const int64_t* blk_off_local /*device, nb+1*/,
                                 int64_t nb, int64_t* blk_task_off, cudaStream_t st);
// plan task lists: segment s copies tasks [seg_src[s], +len) to [seg_dst[s], seg_dst[s+1]) (host
// tables, seg_dst ascending, the last segment ends at total)
cudaError_t k_gather_tasks(const int64_t* seg_src, const int64_t* seg_dst, int64_t nseg, int64_t total,
                           const int64_t* lo, const int64_t* hi, int64_t* olo, int64_t* ohi, cudaStream_t st);

// ------------------------------------------------------------ eval/export
cudaError_t k_init_factors(uint64_t seed, uint64_t tag, int64_t rows_total, int32_t k, const int32_t* perm,
                           int64_t row0, int64_t rows, float* X, cudaStream_t st);
cudaError_t k_scatter_rows(const float* src /*orig order*/, int64_t rows_total, int32_t k, const int32_t* perm,
                           int64_t row0, int64_t rows, float* dst, cudaStream_t st);
cudaError_t k_gather_rows(const float* src /*permuted, local*/, int64_t rows_total, int32_t k,
                          const int32_t* perm, int64_t row0, float* dst /*orig order*/, cudaStream_t st);
cudaError_t k_rmse(const int32_t* tu, const int32_t* tv, const float* tr, int64_t nt, const int32_t* perm_row,
                   const int32_t* perm_col, const float* P, int64_t row0, int64_t rows, const float* Q, int32_t k,
                   double* partials /*2*RMSE_BLOCKS*/, double* out2 /*sum, count*/, cudaStream_t st);
cudaError_t k_average(const float* reps, int32_t G, int64_t count, float* out, cudaStream_t st);
// sum of r^2 over n ratings (fp64, one value on the device)
cudaError_t k_sum_sq(const float* r, int64_t n, double* out, cudaStream_t st);
cudaError_t k_round_half(float* x, int64_t count, cudaStream_t st);
cudaError_t k_pack_half(const float* x, void* y /* __half */, int64_t count, cudaStream_t st);
cudaError_t k_unpack_half(const void* y /* __half */, float* x, int64_t count, cudaStream_t st);
cudaError_t k_average_half(const float* reps, int32_t G, int64_t count, float* out, cudaStream_t st);
// W gathered binary16 copies (stride halves apart) -> fp64 mean rounded once to binary16
cudaError_t k_mean_gathered_half(const void* g, int32_t W, int64_t stride, int64_t count, void* out, cudaStream_t st);
constexpr int RMSE_BLOCKS = 592;
// q_v round-trip ceiling probe (probe.cu): mean ms of one pass over the records
cudaError_t k_probe_roundtrip(int mode, const int32_t* ru, const int32_t* rv, const float* rr, int64_t nrec, int32_t k,
                              int64_t n, float* P, int64_t row0, const float* Q, int64_t warps, int reps, float* ms,
                              cudaStream_t st);

}  // namespace hccmf

// ------------------------------------------------------------- the handle
struct hccmf_ctx {
  int64_t m = 0, n = 0;
  int32_t k = 0;
  float gamma = 0.f, lambda = 0.f;
  int device = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int32_t rank = 0, world = 1;
  hccmf::Comm* comm = nullptr;                  // NCCL or loopback (world > 1 / distributed handles)
  int64_t comm_counts[hccmf::N_COMM_SITES] = {};// per-call-site executions (hccmf_comm_counts)
  cudaStream_t comm_stream = nullptr;           // ring transfers overlapped with compute
  std::vector<cudaEvent_t> ev_done, ev_recv;    // per (stage, column block)
  void* d_wire = nullptr;                       // binary16 staging (send | recv) for Strategy 2
  size_t wire_bytes = 0;
  int state = 0;  // 0 created, 1 loaded, 2 partitioned, 3 factors ready
  hccmf_status sticky = HCCMF_OK;
  std::string err;
  int64_t opt_staleness = 60;  // Hogwild staleness budget, units of 1e-4 (R32); 0: no cap
  double r_rms = 0.0;          // sqrt(mean r^2) of the local records (R32)
  int64_t opt_warps = 0, opt_task = 256, opt_atomic = 1, opt_conflict = 0, opt_heavy = 1024, opt_vec = 0, opt_wave = 1, opt_phases = 1, opt_wire16 = 0, opt_l2persist = 0, opt_depth = 0;
  bool sync_stream = true;
  size_t device_bytes = 0;

  // a1 input (global COO, or this rank's slice of it: sliced ingest), device
  int64_t nnz = 0;     // global ratings (after partition; = nnz_in until then unless sliced)
  int64_t nnz_in = 0;  // ratings in d_in_*
  bool sliced = false; // d_in_* is this rank's slice of the global COO (hccmf_load_ratings_slice)
  int32_t* d_in_u = nullptr;
  int32_t* d_in_v = nullptr;
  float* d_in_r = nullptr;

  // a2-a4
  int32_t G = 1, Br = 1, Bc = 1;
  uint64_t seed = 0;
  std::vector<double> x;
  std::vector<int32_t> bounds;     // G+1
  std::vector<int64_t> block_off;  // global, G*Br*Bc+1
  hccmf::BlockGeom geom{};
  int32_t* d_perm_row = nullptr;
  int32_t* d_perm_col = nullptr;
  int32_t shard_lo = 0, shard_hi = 1;
  int64_t rec0 = 0, local_nnz = 0;
  int32_t* d_u = nullptr;  // sorted local records (permuted ids)
  int32_t* d_v = nullptr;
  float* d_r = nullptr;
  int64_t blk0 = 0, nblk_local = 0;   // first local block, count
  std::vector<int64_t> blk_task_off;  // nblk_local+1 into base tasks
  int64_t n_tasks = 0;
  int64_t* d_task_lo = nullptr;
  int64_t* d_task_hi = nullptr;

  // factors
  int64_t row0 = 0, rows = 0;
  float* d_P = nullptr;
  float* d_Q = nullptr;
  float* d_Qrep = nullptr;  // logical all-reduce replicas
  int32_t storage = 0;      // 1: Q held in binary16 while an epoch runs (R26); 2: with stochastic rounding (R27)
  uint32_t epoch = 0;       // train_epoch calls since init_factors / set_factors
  uint16_t* d_Qh = nullptr; // n x k binary16 copy of Q, authoritative inside an epoch (storage = 1)
  unsigned long long* d_counters = nullptr;
  int64_t n_counters = 0;
  double* d_partials = nullptr;
  double* d_scalar = nullptr;
  int64_t* d_blk_off = nullptr;  // local block offsets (DET wavefront), nblk_local + 1
  int* d_progress = nullptr;     // wavefront progress counters, Br
  hccmf::DetChain det_chain;     // chain-parallel DET schedule (built at the first such epoch)

  bool transposed = false;  // column grid: internal rows are the caller's columns
  int det_path = -1;        // kernel of the last DET epoch (hccmf_info.det_path)
  // HCCMF_OPT_TIMELINE: events of the last epoch {kind, stage, block, start, end}
  struct TimelineRow {
    int kind, stage, block;
    cudaEvent_t a, b;
  };
  bool opt_timeline = false;
  std::vector<TimelineRow> timeline;
  int q_ring_sched = -1;  // >= 0: distributed ring left only this rank's Q group valid
  std::vector<hccmf::Plan> plans;
};
