// blocker.cu -- a1-a4 and the Hogwild task builder: validation, seeded ID shuffle,
// row histogram + prefix, shard-boundary search, blocking + stable radix sort.
//
// PAPER.md section 3.1 preprocessing "shuffling, sorting, and data partition"
// (L543-L548), row grid (L881-L895), row-sorted blocks (L1472-L1474).  Every
// step is integer work and bit-exact against the oracle (tests/test_gpu_*).
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include <cub/cub.cuh>
#include <thrust/iterator/counting_iterator.h>

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

__global__ void validate_kernel(const int32_t* __restrict__ u, const int32_t* __restrict__ v,
                                const float* __restrict__ r, int64_t nnz, int64_t m, int64_t n,
                                unsigned int* flag) {
  unsigned bad = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t uu = u[i], vv = v[i];
    const float rr = r[i];
    if (uu < 0 || uu >= m) bad |= 1u;
    if (vv < 0 || vv >= n) bad |= 2u;
    if (!isfinite(rr)) bad |= 4u;
  }
  bad = __reduce_or_sync(0xffffffffu, bad);
  if (bad && (threadIdx.x & 31) == 0) atomicOr(flag, bad);
}

__global__ void perm_keys_kernel(uint64_t seed, uint64_t tag, int64_t count, uint64_t* keys, int32_t* ids) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x) {
    keys[i] = hash4(seed, tag, (uint64_t)i, 0);
    ids[i] = (int32_t)i;
  }
}

__global__ void perm_scatter_kernel(const int32_t* ids_sorted, int64_t count, int32_t* perm) {
  for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < count; r += (int64_t)gridDim.x * blockDim.x)
    perm[ids_sorted[r]] = (int32_t)r;
}

__global__ void iota_kernel(int32_t* perm, int64_t count) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < count; i += (int64_t)gridDim.x * blockDim.x)
    perm[i] = (int32_t)i;
}

__global__ void row_count_kernel(const int32_t* __restrict__ u, int64_t nnz, const int32_t* __restrict__ perm_row,
                                 unsigned long long* cnt) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt + perm_row[u[i]], 1ull);
}

// first r in [0, m] with S[r] >= x  (S non-decreasing, m+1 entries); m+1 if none
__device__ int64_t lower_bound_u64(const unsigned long long* S, int64_t m, unsigned long long x) {
  int64_t lo = 0, hi = m + 1;
  while (lo < hi) {
    const int64_t mid = lo + ((hi - lo) >> 1);
    if (S[mid] < x) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// unrestricted argmin_r |S[r] - T|, ties to the smaller r (R10); the
// host applies b_s = max(b_{s-1}, r*), which equals the restricted argmin.
__global__ void bound_search_kernel(const unsigned long long* S, int64_t m, const int64_t* targets, int32_t nt,
                                    int64_t* out) {
  const int s = blockIdx.x * blockDim.x + threadIdx.x;
  if (s >= nt) return;
  const int64_t T = targets[s];
  if (T <= 0) { out[s] = 0; return; }
  const int64_t a = lower_bound_u64(S, m, (unsigned long long)T);  // S[a] >= T
  int64_t best = -1;
  int64_t dbest = 0;
  if (a <= m) { best = a; dbest = (int64_t)S[a] - T; }
  if (a > 0) {
    const unsigned long long vb = S[a - 1];  // < T
    const int64_t b = lower_bound_u64(S, m, vb);  // first r with S[r] == vb
    const int64_t db = T - (int64_t)vb;
    if (best < 0 || db <= dbest) best = b;
  }
  out[s] = best;
}

__device__ __forceinline__ int32_t shard_of(const int32_t* b, int32_t G, int32_t up) {
  // largest s with b[s] <= up (b non-decreasing, b[0] = 0 <= up < b[G] = m)
  int lo = 0, hi = G;  // answer in [0, G-1]
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (b[mid] <= up) lo = mid; else hi = mid;
  }
  return lo;
}

__device__ __forceinline__ int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

__global__ void block_key_kernel(BlockGeom g, const int32_t* __restrict__ bounds, const int32_t* __restrict__ perm_row,
                                 const int32_t* __restrict__ perm_col, const int32_t* __restrict__ u,
                                 const int32_t* __restrict__ v, int64_t nnz, uint64_t* keys) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t up = perm_row[u[i]], vp = perm_col[v[i]];
    const int32_t s = shard_of(bounds, g.G, up);
    const int64_t rows = (int64_t)bounds[s + 1] - bounds[s];
    const int64_t l = (int64_t)up - bounds[s];
    const int64_t rb = (l * g.Br) / rows;
    const int64_t rstart = ceil_div(rb * rows, g.Br);
    const int64_t cb = ((int64_t)vp * g.Bc) / g.n;
    const int64_t cstart = ceil_div(cb * g.n, g.Bc);
    const int64_t w = ceil_div((cb + 1) * g.n, g.Bc) - cstart;
    // a row's ratings inside a block start at a row-dependent column (R21): Hogwild
    // groups that start together do not sweep the same items in lock step
    const int64_t rot = g.seed ? (int64_t)(hash4(g.seed, 5, (uint64_t)up, 0) % (uint64_t)w) : 0;
    const uint64_t blk = (uint64_t)(((int64_t)s * g.Br + rb) * g.Bc + cb);
    keys[i] = (blk << (g.bu + g.bv)) | ((uint64_t)(l - rstart) << g.bv) | (uint64_t)((vp - cstart + rot) % w);
  }
}

__global__ void block_decode_kernel(BlockGeom g, const int32_t* __restrict__ bounds, const uint64_t* __restrict__ keys,
                                    int64_t nnz, int32_t* ou, int32_t* ov) {
  const uint64_t mu = (g.bu >= 64) ? ~0ull : ((1ull << g.bu) - 1);
  const uint64_t mv = (g.bv >= 64) ? ~0ull : ((1ull << g.bv) - 1);
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t key = keys[i];
    const int sh = g.bu + g.bv;
    const int64_t blk = sh >= 64 ? 0 : (int64_t)(key >> sh);
    const int64_t lu = (int64_t)((key >> g.bv) & mu);
    const int64_t lv = (int64_t)(key & mv);
    const int64_t cb = blk % g.Bc;
    const int64_t srb = blk / g.Bc;
    const int64_t rb = srb % g.Br;
    const int64_t s = srb / g.Br;
    const int64_t rows = (int64_t)bounds[s + 1] - bounds[s];
    const int64_t rstart = ceil_div(rb * rows, g.Br);
    const int64_t cstart = ceil_div(cb * g.n, g.Bc);
    const int64_t w = ceil_div((cb + 1) * g.n, g.Bc) - cstart;
    const int64_t up = bounds[s] + rstart + lu;
    const int64_t rot = g.seed ? (int64_t)(hash4(g.seed, 5, (uint64_t)up, 0) % (uint64_t)w) : 0;
    ou[i] = (int32_t)up;
    ov[i] = (int32_t)(cstart + (lv + w - rot) % w);
  }
}

__global__ void block_off_kernel(const uint64_t* __restrict__ keys, int64_t nnz, int shift, int64_t nblk, int64_t* off) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j <= nblk; j += (int64_t)gridDim.x * blockDim.x) {
    if (j == nblk) { off[j] = nnz; continue; }
    const uint64_t x = shift >= 64 ? 0 : ((uint64_t)j << shift);
    int64_t lo = 0, hi = nnz;
    if (shift >= 64) { off[j] = 0; continue; }
    while (lo < hi) {
      const int64_t mid = lo + ((hi - lo) >> 1);
      if (keys[mid] < x) lo = mid + 1; else hi = mid;
    }
    off[j] = lo;
  }
}

// ---------------------------------------------------------------- tasks
__global__ void run_flag_kernel(const int32_t* __restrict__ ru, int64_t nrec, unsigned char* flag) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nrec; i += (int64_t)gridDim.x * blockDim.x)
    flag[i] = (i == 0 || ru[i] != ru[i - 1]) ? 1 : 0;
}

__global__ void block_start_flag_kernel(const int64_t* off, int64_t nb, int64_t nrec, unsigned char* flag) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < nb; j += (int64_t)gridDim.x * blockDim.x)
    if (off[j] < off[j + 1] && off[j] < nrec) flag[off[j]] = 1;
}

__global__ void cand_count_kernel(const int64_t* off, int64_t nb, int64_t target, int64_t* cnt) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < nb; j += (int64_t)gridDim.x * blockDim.x) {
    const int64_t len = off[j + 1] - off[j];
    cnt[j] = (len + target - 1) / target;
  }
}

__device__ int64_t upper_bound_i64(const int64_t* a, int64_t n, int64_t x) {  // first idx with a[idx] > x
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    const int64_t mid = lo + ((hi - lo) >> 1);
    if (a[mid] <= x) lo = mid + 1; else hi = mid;
  }
  return lo;
}
__device__ int64_t lower_bound_i64(const int64_t* a, int64_t n, int64_t x) {  // first idx with a[idx] >= x
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    const int64_t mid = lo + ((hi - lo) >> 1);
    if (a[mid] < x) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// candidate c (global numbering): block j = upper_bound(cand_off, c)-1, q = c - cand_off[j],
// pos = off[j] + q*target, mapped to the first run start >= pos; kept if < off[j+1]
// and different from the mapping of candidate q-1.
__global__ void cand_map_kernel(const int64_t* cand_off, int64_t nb, int64_t ncand, const int64_t* off,
                                int64_t target, const int64_t* runs, int64_t nruns, int64_t* cand_pos,
                                unsigned char* keep) {
  for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < ncand; c += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = upper_bound_i64(cand_off, nb + 1, c) - 1;
    const int64_t q = c - cand_off[j];
    const int64_t pos = off[j] + q * target;
    const int64_t ri = lower_bound_i64(runs, nruns, pos);
    const int64_t mp = ri < nruns ? runs[ri] : INT64_MAX;
    bool k = mp < off[j + 1];
    if (k && q > 0) {
      const int64_t pp = off[j] + (q - 1) * target;
      const int64_t rp = lower_bound_i64(runs, nruns, pp);
      const int64_t mpp = rp < nruns ? runs[rp] : INT64_MAX;
      k = mpp != mp;
    }
    cand_pos[c] = mp;
    keep[c] = k ? 1 : 0;
  }
}

__global__ void task_hi_kernel(const int64_t* lo, int64_t nt, const int64_t* off, int64_t nb, int64_t heavy,
                               int64_t* hi, uint64_t* sortkey, int64_t* idx) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nt; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = upper_bound_i64(off, nb + 1, lo[t]) - 1;
    int64_t h = off[j + 1];
    if (t + 1 < nt && lo[t + 1] < h) h = lo[t + 1];
    hi[t] = h;
    // inside each block: tasks longer than `heavy` first, longest first (LPT),
    // then the rest in record order (the shuffled user order); heavy < 0: none
    const uint64_t len = (uint64_t)(h - lo[t]);
    const bool is_heavy = heavy >= 0 && (int64_t)len > heavy;
    const uint64_t inv = (len >= (1ull << 38)) ? 0 : ((1ull << 38) - 1 - len);
    sortkey[t] = ((uint64_t)j << 39) | (is_heavy ? inv : ((1ull << 38) | (uint64_t)t));
    idx[t] = t;
  }
}

__global__ void permute_tasks_kernel(const int64_t* idx, int64_t nt, const int64_t* lo, const int64_t* hi,
                                     int64_t* olo, int64_t* ohi) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nt; t += (int64_t)gridDim.x * blockDim.x) {
    olo[t] = lo[idx[t]];
    ohi[t] = hi[idx[t]];
  }
}

__global__ void item_degree_kernel(const int32_t* __restrict__ v, int64_t nnz, unsigned long long* cnt) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt + v[i], 1ull);
}

// sliced ingest: destination shard of every rating (key) and its input index (value)
__global__ void shard_key_kernel(const int32_t* __restrict__ u, int64_t nnz, const int32_t* __restrict__ perm_row,
                                 const int32_t* __restrict__ bounds, int32_t G, uint32_t* key, int64_t* idx,
                                 unsigned long long* cnt) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t s = shard_of(bounds, G, perm_row[u[i]]);
    key[i] = (uint32_t)s;
    idx[i] = i;
    atomicAdd(cnt + s, 1ull);
  }
}

__global__ void gather_ratings_kernel(const int64_t* __restrict__ idx, int64_t nnz, const int32_t* __restrict__ u,
                                      const int32_t* __restrict__ v, const float* __restrict__ r, int32_t* ou,
                                      int32_t* ov, float* orr) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < nnz; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = idx[i];
    ou[i] = u[j];
    ov[i] = v[j];
    orr[i] = r[j];
  }
}

template <typename T>
cudaError_t dalloc(T** p, size_t count, cudaStream_t st) {
  return cudaMallocAsync((void**)p, sizeof(T) * (count ? count : 1), st);
}

#define CKR(x)                            \
  do {                                    \
    cudaError_t e_ = (x);                 \
    if (e_ != cudaSuccess) return e_;     \
  } while (0)

}  // namespace

cudaError_t k_validate(const int32_t* u, const int32_t* v, const float* r, int64_t nnz, int64_t m, int64_t n,
                       unsigned int* flag, cudaStream_t st) {
  if (nnz == 0) return cudaSuccess;
  (note_launch(), validate_kernel<<<grid_for(nnz), kT, 0, st>>>(u, v, r, nnz, m, n, flag));
  return cudaGetLastError();
}

cudaError_t k_perm(uint64_t seed, uint64_t tag, int64_t count, int32_t* perm, cudaStream_t st) {
  if (count == 0) return cudaSuccess;
  if (seed == 0) {
    (note_launch(), iota_kernel<<<grid_for(count), kT, 0, st>>>(perm, count));
    return cudaGetLastError();
  }
  uint64_t *k0 = nullptr, *k1 = nullptr;
  int32_t *i0 = nullptr, *i1 = nullptr;
  CKR(dalloc(&k0, count, st));
  CKR(dalloc(&k1, count, st));
  CKR(dalloc(&i0, count, st));
  CKR(dalloc(&i1, count, st));
  (note_launch(), perm_keys_kernel<<<grid_for(count), kT, 0, st>>>(seed, tag, count, k0, i0));
  CKR(cudaGetLastError());
  size_t tb = 0;
  void* tmp = nullptr;
  CKR(cub::DeviceRadixSort::SortPairs(nullptr, tb, k0, k1, i0, i1, count, 0, 64, st));
  CKR(cudaMallocAsync(&tmp, tb, st));
  CKR(cub::DeviceRadixSort::SortPairs(tmp, tb, k0, k1, i0, i1, count, 0, 64, st));
  (note_launch(), perm_scatter_kernel<<<grid_for(count), kT, 0, st>>>(i1, count, perm));
  CKR(cudaGetLastError());
  cudaFreeAsync(tmp, st);
  cudaFreeAsync(k0, st);
  cudaFreeAsync(k1, st);
  cudaFreeAsync(i0, st);
  cudaFreeAsync(i1, st);
  return cudaGetLastError();
}

cudaError_t k_row_prefix(const int32_t* u, int64_t nnz, const int32_t* perm_row, int64_t m, unsigned long long* S,
                         cudaStream_t st) {
  unsigned long long* cnt = nullptr;
  CKR(dalloc(&cnt, m + 1, st));
  CKR(cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * (m + 1), st));
  if (nnz) {
    (note_launch(), row_count_kernel<<<grid_for(nnz), kT, 0, st>>>(u, nnz, perm_row, cnt));
    CKR(cudaGetLastError());
  }
  size_t tb = 0;
  void* tmp = nullptr;
  CKR(cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, S, m + 1, st));
  CKR(cudaMallocAsync(&tmp, tb, st));
  CKR(cub::DeviceScan::ExclusiveSum(tmp, tb, cnt, S, m + 1, st));
  cudaFreeAsync(tmp, st);
  cudaFreeAsync(cnt, st);
  return cudaGetLastError();
}

cudaError_t k_item_degree(const int32_t* v, int64_t nnz, int64_t n, unsigned long long* deg, cudaStream_t st) {
  CKR(cudaMemsetAsync(deg, 0, sizeof(unsigned long long) * n, st));
  if (nnz) {
    (note_launch(), item_degree_kernel<<<grid_for(nnz), kT, 0, st>>>(v, nnz, deg));
    CKR(cudaGetLastError());
  }
  return cudaSuccess;
}

cudaError_t k_bound_search(const unsigned long long* S, int64_t m, const int64_t* targets, int32_t nt, int64_t* out,
                           cudaStream_t st) {
  if (nt <= 0) return cudaSuccess;
  (note_launch(), bound_search_kernel<<<(nt + 127) / 128, 128, 0, st>>>(S, m, targets, nt, out));
  return cudaGetLastError();
}

static void bs_mark(cudaStream_t st, const char* what) {
  static bool on = getenv("HCCMF_PROFILE") != nullptr;
  if (!on) return;
  static auto t0 = std::chrono::steady_clock::now();
  cudaStreamSynchronize(st);
  auto t1 = std::chrono::steady_clock::now();
  fprintf(stderr, "[hccmf]   %-26s %9.3f ms\n", what, std::chrono::duration<double, std::milli>(t1 - t0).count());
  t0 = t1;
}

cudaError_t k_block_sort(const BlockGeom& g, const int32_t* bounds, const int32_t* perm_row, const int32_t* perm_col,
                         const int32_t* u, const int32_t* v, const float* r, int64_t nnz, int32_t* ou, int32_t* ov,
                         float* orr, int64_t* block_off, cudaStream_t st) {
  bs_mark(st, "bs: enter");
  const int64_t nblk = (int64_t)g.G * g.Br * g.Bc;
  const int bits = g.bb + g.bu + g.bv;
  uint64_t *k0 = nullptr, *k1 = nullptr;
  CKR(dalloc(&k0, nnz, st));
  CKR(dalloc(&k1, nnz, st));
  bs_mark(st, "bs: alloc keys");
  if (nnz) {
    (note_launch(), block_key_kernel<<<grid_for(nnz), kT, 0, st>>>(g, bounds, perm_row, perm_col, u, v, nnz, k0));
    CKR(cudaGetLastError());
  }
  bs_mark(st, "bs: key kernel");
  const uint64_t* ks = k0;
  if (nnz && bits > 0) {
    size_t tb = 0;
    void* tmp = nullptr;
    const int end_bit = bits;
    CKR(cub::DeviceRadixSort::SortPairs(nullptr, tb, k0, k1, r, orr, nnz, 0, end_bit, st));
    CKR(cudaMallocAsync(&tmp, tb, st));
    CKR(cub::DeviceRadixSort::SortPairs(tmp, tb, k0, k1, r, orr, nnz, 0, end_bit, st));
    cudaFreeAsync(tmp, st);
    ks = k1;
  } else if (nnz) {
    CKR(cudaMemcpyAsync(orr, r, sizeof(float) * nnz, cudaMemcpyDeviceToDevice, st));
  }
  bs_mark(st, "bs: radix sort");
  if (nnz) {
    (note_launch(), block_decode_kernel<<<grid_for(nnz), kT, 0, st>>>(g, bounds, ks, nnz, ou, ov));
    CKR(cudaGetLastError());
  }
  bs_mark(st, "bs: decode");
  (note_launch(), block_off_kernel<<<grid_for(nblk + 1), kT, 0, st>>>(ks, nnz, g.bu + g.bv, nblk, block_off));
  CKR(cudaGetLastError());
  cudaFreeAsync(k0, st);
  cudaFreeAsync(k1, st);
  return cudaGetLastError();
}

cudaError_t k_shard_split(const int32_t* u, const int32_t* v, const float* r, int64_t nnz, const int32_t* perm_row,
                          const int32_t* bounds, int32_t G, int32_t* ou, int32_t* ov, float* orr, int64_t* counts,
                          cudaStream_t st) {
  for (int s = 0; s < G; ++s) counts[s] = 0;
  if (nnz == 0) return cudaSuccess;
  uint32_t *k0 = nullptr, *k1 = nullptr;
  int64_t *i0 = nullptr, *i1 = nullptr;
  unsigned long long* cnt = nullptr;
  CKR(dalloc(&k0, nnz, st));
  CKR(dalloc(&k1, nnz, st));
  CKR(dalloc(&i0, nnz, st));
  CKR(dalloc(&i1, nnz, st));
  CKR(dalloc(&cnt, G, st));
  CKR(cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * G, st));
  (note_launch(), shard_key_kernel<<<grid_for(nnz), kT, 0, st>>>(u, nnz, perm_row, bounds, G, k0, i0, cnt));
  CKR(cudaGetLastError());
  int bits = 0;
  while ((1 << bits) < G) ++bits;
  const int64_t* idx = i0;
  if (bits > 0) {  // LSD radix sort: stable, so each shard keeps the input order
    size_t tb = 0;
    void* tmp = nullptr;
    CKR(cub::DeviceRadixSort::SortPairs(nullptr, tb, k0, k1, i0, i1, nnz, 0, bits, st));
    CKR(cudaMallocAsync(&tmp, tb, st));
    CKR(cub::DeviceRadixSort::SortPairs(tmp, tb, k0, k1, i0, i1, nnz, 0, bits, st));
    cudaFreeAsync(tmp, st);
    idx = i1;
  }
  (note_launch(), gather_ratings_kernel<<<grid_for(nnz), kT, 0, st>>>(idx, nnz, u, v, r, ou, ov, orr));
  CKR(cudaGetLastError());
  std::vector<unsigned long long> h(G);
  CKR(cudaMemcpyAsync(h.data(), cnt, sizeof(unsigned long long) * G, cudaMemcpyDeviceToHost, st));
  CKR(cudaStreamSynchronize(st));
  for (int s = 0; s < G; ++s) counts[s] = (int64_t)h[s];
  for (void* p : {(void*)k0, (void*)k1, (void*)i0, (void*)i1, (void*)cnt}) cudaFreeAsync(p, st);
  return cudaGetLastError();
}

cudaError_t k_build_tasks(const int32_t* ru, int64_t nrec, const int64_t* off, int64_t nb, int64_t target,
                          int64_t heavy, int64_t** task_lo, int64_t** task_hi, int64_t* n_tasks, cudaStream_t st) {
  *n_tasks = 0;
  *task_lo = nullptr;
  *task_hi = nullptr;
  if (nrec == 0) {
    CKR(cudaMallocAsync((void**)task_lo, sizeof(int64_t), st));
    CKR(cudaMallocAsync((void**)task_hi, sizeof(int64_t), st));
    return cudaSuccess;
  }
  unsigned char* flag = nullptr;
  int64_t* runs = nullptr;
  int64_t* nsel = nullptr;
  CKR(dalloc(&flag, nrec, st));
  CKR(dalloc(&runs, nrec, st));
  CKR(dalloc(&nsel, 1, st));
  (note_launch(), run_flag_kernel<<<grid_for(nrec), kT, 0, st>>>(ru, nrec, flag));
  (note_launch(), block_start_flag_kernel<<<grid_for(nb), kT, 0, st>>>(off, nb, nrec, flag));
  CKR(cudaGetLastError());
  size_t tb = 0;
  void* tmp = nullptr;
  thrust::counting_iterator<int64_t> it(0);
  CKR(cub::DeviceSelect::Flagged(nullptr, tb, it, flag, runs, nsel, nrec, st));
  CKR(cudaMallocAsync(&tmp, tb, st));
  CKR(cub::DeviceSelect::Flagged(tmp, tb, it, flag, runs, nsel, nrec, st));
  cudaFreeAsync(tmp, st);
  int64_t nruns = 0;
  CKR(cudaMemcpyAsync(&nruns, nsel, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
  CKR(cudaStreamSynchronize(st));

  // candidates per block
  int64_t *ccnt = nullptr, *coff = nullptr;
  CKR(dalloc(&ccnt, nb + 1, st));
  CKR(dalloc(&coff, nb + 1, st));
  CKR(cudaMemsetAsync(ccnt, 0, sizeof(int64_t) * (nb + 1), st));
  (note_launch(), cand_count_kernel<<<grid_for(nb), kT, 0, st>>>(off, nb, target, ccnt));
  CKR(cudaGetLastError());
  tb = 0;
  CKR(cub::DeviceScan::ExclusiveSum(nullptr, tb, ccnt, coff, nb + 1, st));
  CKR(cudaMallocAsync(&tmp, tb, st));
  CKR(cub::DeviceScan::ExclusiveSum(tmp, tb, ccnt, coff, nb + 1, st));
  cudaFreeAsync(tmp, st);
  int64_t ncand = 0;
  CKR(cudaMemcpyAsync(&ncand, coff + nb, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
  CKR(cudaStreamSynchronize(st));

  int64_t* cpos = nullptr;
  unsigned char* keep = nullptr;
  int64_t* lo = nullptr;
  CKR(dalloc(&cpos, ncand, st));
  CKR(dalloc(&keep, ncand, st));
  CKR(dalloc(&lo, ncand, st));
  (note_launch(), cand_map_kernel<<<grid_for(ncand), kT, 0, st>>>(coff, nb, ncand, off, target, runs, nruns, cpos, keep));
  CKR(cudaGetLastError());
  tb = 0;
  CKR(cub::DeviceSelect::Flagged(nullptr, tb, cpos, keep, lo, nsel, ncand, st));
  CKR(cudaMallocAsync(&tmp, tb, st));
  CKR(cub::DeviceSelect::Flagged(tmp, tb, cpos, keep, lo, nsel, ncand, st));
  cudaFreeAsync(tmp, st);
  int64_t nt = 0;
  CKR(cudaMemcpyAsync(&nt, nsel, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
  CKR(cudaStreamSynchronize(st));

  int64_t* hi = nullptr;
  uint64_t *sk0 = nullptr, *sk1 = nullptr;
  int64_t *ix0 = nullptr, *ix1 = nullptr;
  CKR(dalloc(&hi, nt, st));
  CKR(dalloc(&sk0, nt, st));
  CKR(dalloc(&sk1, nt, st));
  CKR(dalloc(&ix0, nt, st));
  CKR(dalloc(&ix1, nt, st));
  (note_launch(), task_hi_kernel<<<grid_for(nt), kT, 0, st>>>(lo, nt, off, nb, heavy, hi, sk0, ix0));
  CKR(cudaGetLastError());
  tb = 0;
  CKR(cub::DeviceRadixSort::SortPairs(nullptr, tb, sk0, sk1, ix0, ix1, nt, 0, 64, st));
  CKR(cudaMallocAsync(&tmp, tb, st));
  CKR(cub::DeviceRadixSort::SortPairs(tmp, tb, sk0, sk1, ix0, ix1, nt, 0, 64, st));
  cudaFreeAsync(tmp, st);
  CKR(cudaMallocAsync((void**)task_lo, sizeof(int64_t) * (nt ? nt : 1), st));
  CKR(cudaMallocAsync((void**)task_hi, sizeof(int64_t) * (nt ? nt : 1), st));
  (note_launch(), permute_tasks_kernel<<<grid_for(nt), kT, 0, st>>>(ix1, nt, lo, hi, *task_lo, *task_hi));
  CKR(cudaGetLastError());
  for (void* p : {(void*)flag, (void*)runs, (void*)nsel, (void*)ccnt, (void*)coff, (void*)cpos, (void*)keep,
                  (void*)lo, (void*)hi, (void*)sk0, (void*)sk1, (void*)ix0, (void*)ix1})
    cudaFreeAsync(p, st);
  CKR(cudaStreamSynchronize(st));
  *n_tasks = nt;
  return cudaSuccess;
}

// ---- task index per block and plan gathering, without a host copy of the tasks
namespace {
__device__ __forceinline__ int64_t block_of(const int64_t* off, int64_t nb, int64_t lo) {
  int64_t a = 0, b = nb;  // largest j in [0, nb) with off[j] <= lo
  while (b - a > 1) {
    const int64_t mid = (a + b) >> 1;
    if (off[mid] <= lo) a = mid; else b = mid;
  }
  return a;
}
__global__ void task_block_start_kernel(const int64_t* __restrict__ task_lo, int64_t nt, const int64_t* __restrict__ off,
                                        int64_t nb, int64_t* __restrict__ start) {
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nt; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = block_of(off, nb, task_lo[t]);
    if (t == 0 || block_of(off, nb, task_lo[t - 1]) != b) start[b] = t;
  }
}
__global__ void gather_tasks_kernel(const int64_t* __restrict__ seg_src, const int64_t* __restrict__ seg_dst,
                                    int64_t nseg, int64_t total, const int64_t* __restrict__ lo,
                                    const int64_t* __restrict__ hi, int64_t* __restrict__ olo, int64_t* __restrict__ ohi) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t a = 0, b = nseg;  // segment s with seg_dst[s] <= i < seg_dst[s + 1]
    while (b - a > 1) {
      const int64_t mid = (a + b) >> 1;
      if (seg_dst[mid] <= i) a = mid; else b = mid;
    }
    const int64_t src = seg_src[a] + (i - seg_dst[a]);
    olo[i] = lo[src];
    ohi[i] = hi[src];
  }
}
}  // namespace

cudaError_t k_task_block_offsets(const int64_t* task_lo, int64_t nt, const int64_t* off, int64_t nb, int64_t* blk_task_off,
                                 cudaStream_t st) {
  int64_t* d = nullptr;
  CKR(dalloc(&d, nb + 1, st));
  CKR(cudaMemsetAsync(d, 0xff, sizeof(int64_t) * (nb + 1), st));  // -1: no task starts there
  if (nt > 0) (note_launch(), task_block_start_kernel<<<grid_for(nt), kT, 0, st>>>(task_lo, nt, off, nb, d));
  CKR(cudaGetLastError());
  CKR(cudaMemcpyAsync(blk_task_off, d, sizeof(int64_t) * (nb + 1), cudaMemcpyDeviceToHost, st));
  CKR(cudaStreamSynchronize(st));
  cudaFreeAsync(d, st);
  blk_task_off[nb] = nt;  // a block without tasks starts where the next one does
  for (int64_t j = nb - 1; j >= 0; --j)
    if (blk_task_off[j] < 0) blk_task_off[j] = blk_task_off[j + 1];
  return cudaSuccess;
}

cudaError_t k_gather_tasks(const int64_t* seg_src, const int64_t* seg_dst, int64_t nseg, int64_t total,
                           const int64_t* lo, const int64_t* hi, int64_t* olo, int64_t* ohi, cudaStream_t st) {
  if (total <= 0 || nseg <= 0) return cudaSuccess;
  int64_t *ds = nullptr, *dd = nullptr;
  CKR(dalloc(&ds, nseg, st));
  CKR(dalloc(&dd, nseg, st));
  CKR(cudaMemcpyAsync(ds, seg_src, sizeof(int64_t) * nseg, cudaMemcpyHostToDevice, st));
  CKR(cudaMemcpyAsync(dd, seg_dst, sizeof(int64_t) * nseg, cudaMemcpyHostToDevice, st));
  (note_launch(), gather_tasks_kernel<<<grid_for(total), kT, 0, st>>>(ds, dd, nseg, total, lo, hi, olo, ohi));
  CKR(cudaGetLastError());
  CKR(cudaStreamSynchronize(st));  // the host segment tables are the caller's
  cudaFreeAsync(ds, st);
  cudaFreeAsync(dd, st);
  return cudaSuccess;
}

}  // namespace hccmf
