/*
 * hccmf.h -- C ABI of libhccmf, the B200-native hot path of HCC-MF
 * (Huang, Yin, Liu, He, Bai, Li: "A Novel Multi-CPU/GPU Collaborative Computing
 * Framework for SGD-based Matrix Factorization", ICPP '21).
 *
 * Citations: L<n> = line n of the paper text.
 * lists every reading taken where the paper is silent or garbled (R1..R33).
 *
 * What the library computes:
 *   a0 factor init, a1 ingest+validate COO, a2 seeded ID shuffle, a3 row-grid
 *   partition (DP0/DP1/DP2), a4 blocking + stable sort, a5 deterministic SGD
 *   epoch, a6 Hogwild SGD epoch, a7 Q synchronisation across shards, a8 RMSE,
 *   a9 export.
 *
 * Conventions (all entry points):
 *  - extern "C", plain pointers and sizes; no C++ types or exceptions cross it.
 *  - Every call returns hccmf_status; details in hccmf_last_error(h).  CUDA and
 *    NCCL failures are sticky: after one, every call on the handle returns the
 *    same code.
 *  - Indices are 0-based.  u in [0, m), v in [0, n).
 *  - Factor layout: P is m x k row-major fp32 (p_u contiguous); Q is n x k
 *    row-major fp32 (q_v contiguous) -- this is the paper's k x n item matrix Q
 *    (Table 1) TRANSPOSED.
 *  - Input pointers may be host or device memory (resolved through unified
 *    virtual addressing, cudaMemcpyDefault).  The library COPIES inputs; the caller keeps
 *    ownership and may free them when the call returns.  Output pointers are
 *    caller-allocated, host or device.  The handle owns all device memory it
 *    allocates; hccmf_destroy frees it.
 *  - Call order: create -> load_ratings -> partition -> (init_factors |
 *    set_factors) -> { train_epoch | rmse | get_factors }*.  Out of order:
 *    HCCMF_ESTATE.
 *  - All work is issued on the handle's CUDA stream (its own, or the one given
 *    to hccmf_set_stream); every call returns after that stream is synchronised
 *    unless stated otherwise, so host timing around a call is meaningful.  The
 *    handle's own stream is a blocking stream (ordered after the legacy default
 *    stream); with hccmf_set_stream the caller orders device inputs itself.
 *  - Not thread-safe per handle; distinct handles are independent.
 *  - There is no CPU fallback: without a CUDA device every call that needs one
 *    returns HCCMF_ECUDA.
 */
#ifndef HCCMF_H_
#define HCCMF_H_

#include <stdint.h>

#if defined(__GNUC__)
#define HCCMF_API __attribute__((visibility("default")))
#else
#define HCCMF_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct hccmf_ctx* hccmf_t;
/* In-process loopback communicator hub: G handles of ONE process on one device,
 * one host thread each, exchange Q through it exactly as G ranks exchange it over
 * NCCL (same call sites, same buffers, same stream ordering). */
typedef struct hccmf_hub* hccmf_hub_t;

typedef enum {
    HCCMF_OK = 0,
    HCCMF_EINVAL = -1, /* bad argument (sizes, k, gamma, grid, NULL)         */
    HCCMF_ERANGE = -2, /* rating index out of range, non-finite r, overflow  */
    HCCMF_ENOMEM = -3, /* device allocation failed                           */
    HCCMF_ESTATE = -4, /* call out of order                                  */
    HCCMF_ECUDA = -5,  /* CUDA runtime error / no device (sticky)            */
    HCCMF_ENCCL = -6   /* NCCL error (sticky)                                */
} hccmf_status;

/* a5 / a6: the SGD schedule inside a shard.
 * DET: FPSGD-style conflict-free strata of independent blocks in a fixed order
 *      (PAPER.md L93-L97, L2269-L2275); the result equals the oracle's serial
 *      run of the same order up to fp32 rounding.
 * HOGWILD: lock-free racing updates over user-aligned tasks (Hogwild!, L216-L219,
 *      L1680-L1691).  Non-deterministic by design. */
typedef enum { HCCMF_SCHED_DET = 0, HCCMF_SCHED_HOGWILD = 1 } hccmf_sched;

/* a7: how shards exchange Q (only Q moves: Strategy 1, L1203-L1233).
 * NONE: one shard.  RING: rotating column groups of Q, stage t shard s updates
 *      group (s+t) mod G and passes it to shard s-1 (hidden synchronisation,
 *      L1143-L1172; async computing-transmission, L1251-L1269).
 * ALLREDUCE_AVG: every shard trains against its own replica of Q, then
 *      Q = mean_s Q_s (the server's multiply-add sync, L549-L557, L783-L784). */
typedef enum { HCCMF_SYNC_NONE = 0, HCCMF_SYNC_RING = 1, HCCMF_SYNC_ALLREDUCE_AVG = 2 } hccmf_sync;

/* a3: data partition strategy (section 3.3).
 * DP0: Eq. 6 (L967-L981) from t_meas if given, else equal shares x_s = 1/G.
 * DP1: Algorithm 1 compensation (L1025-L1142), needs t_meas (R11).
 * DP2: Eq. 7 hidden-synchronisation ramp (L1143-L1172), needs t_meas, t_sync. */
typedef enum { HCCMF_DP0 = 0, HCCMF_DP1 = 1, HCCMF_DP2 = 2 } hccmf_dp;

typedef struct {
    int32_t n_shards;     /* G >= 1.  Distributed handle: must equal world size.
                             Single-process handle: G > 1 runs G LOGICAL shards on
                             the one device (exactly the multi-GPU schedule). */
    int32_t grid_rows;    /* B_r >= 1 row blocks per shard                         */
    int32_t grid_cols;    /* B_c >= 1 column blocks over all n columns.  DET needs
                             B_r == B_c (NONE, ALLREDUCE) or B_c == G*B_r (RING);
                             HOGWILD+RING needs B_c % G == 0.                      */
    int32_t strategy;     /* hccmf_dp                                               */
    const double* x;      /* optional [G] starting fractions of nnz, sum 1 (DP1/2) */
    const double* t_meas; /* optional [G] measured compute time per shard, s       */
    double t_sync;        /* DP2: per-shard sync time, s                            */
    uint64_t seed;        /* a2 ID shuffle seed; 0 = identity permutation          */
    int32_t storage;      /* 0 = fp32 factors; 1 = Q stored as IEEE binary16 while
                             an epoch runs (fp32 arithmetic, P stays fp32): every
                             q_v write keeps the nearest binary16 value (DESIGN.md
                             R26).  Needs one rating per warp
                             (k a multiple of 128): train_epoch returns EINVAL
                             otherwise.  Q read back (rmse, get_factors) holds
                             binary16 values.  2 = as 1 with stochastic rounding
                             of every q_v write (unbiased; random bits from a
                             counter-based hash of (record, epoch, element pair),
                             DESIGN.md R27).                                     */
    int32_t grid_dim;     /* 0 (default): row grid, shards of users, only Q moves;
                             1: column grid, shards of items, only P moves (Strategy 1
                             "transmitting P only", L1216-L1218); 2: the paper's rule
                             (L884-L886): rows if m >= n, else columns.  Under a column
                             grid every caller-facing call keeps its orientation (P is
                             still m x k, rmse takes (u, v)); get_partition, get_records
                             and hccmf_info describe the transposed problem. */
    int32_t col_balance;  /* 0 (default): columns shuffled by the seeded hash (R8);
                             1: degree-balanced column blocks (R30): items
                             in order of (ratings desc, id asc) each take a slot of
                             the least-loaded column block with a free slot (ties to
                             the lowest block), so the heaviest column block -- the
                             DET order's critical path -- carries about the heaviest
                             item alone.  Rows keep the hash shuffle.             */
} hccmf_partition_opts;

typedef struct {
    int64_t m, n, nnz;       /* problem (nnz = ratings loaded, all shards)        */
    int32_t k;
    int32_t n_shards;        /* G                                                 */
    int32_t shard_lo;        /* first shard held by this handle                   */
    int32_t shard_hi;        /* one past the last shard held                      */
    int64_t local_nnz;       /* ratings held by this handle                       */
    int64_t row0, rows;      /* permuted row range [row0, row0+rows) of local P   */
    int64_t n_blocks;        /* G * B_r * B_c                                     */
    int64_t n_tasks;         /* Hogwild tasks (user-aligned runs) held locally    */
    int32_t key_bits;        /* bits of the a4 sort key                           */
    int32_t rank, world;     /* 0, 1 for a single-process handle                  */
    int64_t device_bytes;    /* device memory currently owned by the handle       */
    int32_t transposed;      /* 1: column grid (m, n, rows describe R^T)          */
    int32_t det_path;        /* kernel of the last DET epoch: 0 per-stratum launches,
                                1 slab wavefront, 2 register wavefront, 3 chain-parallel
                                wavefront; -1 none yet                             */
} hccmf_info;

/* Tunables for hccmf_set_option (values are int64). */
typedef enum {
    HCCMF_OPT_HOGWILD_WARPS = 1, /* concurrent warps of the Hogwild kernel; 0 = auto
                                    (R14)                               */
    HCCMF_OPT_TASK_RATINGS = 2,  /* target ratings per Hogwild task (>= 1, default
                                    256); tasks never split a user's run          */
    HCCMF_OPT_SYNC_STREAM = 3,   /* 1 (default): calls return after the stream is
                                    synchronised; 0: return after enqueueing      */
    HCCMF_OPT_HOGWILD_ATOMIC = 5,/* 1 (default): Hogwild applies q_v increments with
                                    vector atomic adds (Hogwild!'s component-wise
                                    atomic model, no lost updates); 0: plain stores
                                    (racing writers may overwrite: the paper's
                                    "coverage", L1680-L1686)                      */
    HCCMF_OPT_CONFLICT_RATIO = 6,/* > 0: auto Hogwild concurrency is at most (items a
                                    launch can touch) / value rating groups (round-1
                                    rule); 0 (default): the staleness budget below  */
    HCCMF_OPT_HEAVY_FIRST = 7,   /* Hogwild task order inside a block: tasks with more
                                    than `value` ratings run first, longest first
                                    (no late heavy user stretches the epoch); the
                                    rest keep the shuffled user order.  Default
                                    1024; -1: shuffled order only; 0: pure LPT.
                                    Takes effect at the next hccmf_partition.     */
    HCCMF_OPT_VEC = 8,           /* float4 slots of p_u / q_v per lane (1, 2, 4; 0 =
                                    auto: k/128 clamped to [1, 4], i.e. one rating
                                    per warp from k = 128); lanes per rating
                                    L = min(32, k / (4 VEC))                      */
    HCCMF_OPT_DET_WAVE = 9,      /* 1 (default): a single-shard DET epoch on a square
                                    grid runs as one wavefront kernel (warp i waits
                                    only for warp i+1's previous stratum) when the
                                    B warps fit on the device, each column block's
                                    Q rows staged in shared memory while a warp
                                    holds it (when ceil(n/B) rows fit); 2: the
                                    wavefront without the shared-memory slab; 0: one
                                    launch per stratum.  Same update order and
                                    bit-identical factors in every case.          */
    HCCMF_OPT_SYNC_PHASES = 10,  /* ALLREDUCE_AVG + HOGWILD: rounds per epoch (>= 1,
                                    default 1; must divide grid_rows).  Round ph runs
                                    every shard's row blocks [ph Br/S, (ph+1) Br/S)
                                    on its Q copy, then averages Q: the paper's
                                    several pull-compute-push pipelines per epoch
                                    (L1251-L1269, Fig. 6; R22).         */
    HCCMF_OPT_WIRE_FP16 = 11,    /* 1: Q travels as IEEE binary16 (Strategy 2,
                                    "Transmitting FP16 Data", L1234-L1249): ring
                                    transfers and the all-reduce pack to half and
                                    unpack to fp32; factors stay fp32 (R25).  The
                                    logical-shard backend applies the same rounding
                                    at every stage boundary.  Default 0.          */
    HCCMF_OPT_L2_PERSIST = 12,   /* 1: during a Hogwild epoch Q is an L2 persisting
                                    access-policy window on the launch stream
                                    (removed afterwards).  Default 0.             */
    HCCMF_OPT_PREFETCH_DEPTH = 13,/* Hogwild, one rating per warp (k = 32, 64 and
                                    k = 128 j): the q_v row of rating j + D is
                                    requested while rating j is updated (1..4;
                                    0 = auto, the default: 1 for k = 128 j, 4 for
                                    k = 32 / 64).  Loads
                                    issued before a warp's own update of the same
                                    item are corrected in registers, so a single
                                    warp stays serial; across warps D widens the
                                    read-to-write window (R14).         */
    HCCMF_OPT_STALENESS = 16,    /* auto Hogwild concurrency (R32): at most
                                    items * kappa / (gamma (r_rms + lambda)) rating
                                    groups in flight per launch, items = the Q rows the
                                    launch can touch, r_rms = sqrt(mean r^2) of the
                                    shard, kappa = value * 1e-4 (default 60 -> 0.006);
                                    0 = no cap (resident warps only)              */
    HCCMF_OPT_TIMELINE = 15,     /* 1: train_epoch records CUDA events around every SGD
                                    launch (compute stream) and every Q transfer (comm
                                    stream) of the epoch; hccmf_timeline reads them.
                                    Default 0 (no events).                        */
    HCCMF_OPT_STORAGE = 14       /* Q storage from the next epoch on: 0 fp32, 1
                                    binary16, 2 binary16 with stochastic rounding
                                    (the partition option `storage`,
                                    changeable without re-partitioning).          */
} hccmf_option;

/* ------------------------------------------------------------------ lifecycle */

/* Create a single-process handle on the current CUDA device.
 * m, n in [1, 2^31); k multiple of 4 in [4, 512]; gamma > 0 finite (learning
 * rate, Table 3); lambda >= 0 finite (L2 weight lambda_1 = lambda_2,
 * Table 3).  *out receives the handle. */
HCCMF_API hccmf_status hccmf_create(int64_t m, int64_t n, int32_t k, float gamma, float lambda, hccmf_t* out);

/* Write an NCCL unique id (128 bytes) into out[128]; rank 0 calls it and
 * broadcasts the bytes with torch.distributed before hccmf_create_dist. */
HCCMF_API hccmf_status hccmf_nccl_unique_id(void* out128);

/* Create a distributed handle: one process per GPU, rank in [0, world), on CUDA
 * device `device`.  Collective: all ranks must call it with the same id. */
HCCMF_API hccmf_status hccmf_create_dist(int64_t m, int64_t n, int32_t k, float gamma, float lambda,
                               const void* nccl_unique_id, int32_t rank, int32_t world,
                               int32_t device, hccmf_t* out);

/* Loopback hub for `world` ranks (no device work; never fails for world >= 1).
 * The hub lives until hccmf_hub_destroy AND every handle created on it is
 * destroyed (reference counted). */
HCCMF_API hccmf_status hccmf_hub_create(int32_t world, hccmf_hub_t* out);
HCCMF_API void hccmf_hub_destroy(hccmf_hub_t hub);

/* A distributed handle whose data plane is the loopback `hub` instead of NCCL:
 * rank in [0, world of the hub), on CUDA device `device`.  Every collective call
 * (partition, train_epoch with sync RING / ALLREDUCE_AVG, rmse, get_factors) must
 * be made by all ranks, each from its own host thread; host waits time out after
 * HCCMF_LOOPBACK_TIMEOUT_S seconds (default 300) with HCCMF_ENCCL.  Used to run
 * the multi-rank data plane on one GPU (tests); production uses hccmf_create_dist. */
HCCMF_API hccmf_status hccmf_create_loopback(int64_t m, int64_t n, int32_t k, float gamma, float lambda,
                                             hccmf_hub_t hub, int32_t rank, int32_t device, hccmf_t* out);

/* Per-call-site counters of the shard data plane (how many times each exchange
 * ran on this handle): counts[i] for i < min(n, HCCMF_COMM_SITES).  Sites, in
 * order: 0 stage-wise ring transfer, 1 pipelined ring block transfer, 2 ring
 * transfer in binary16, 3 ring-group broadcast (materialise Q), 4 fp32 Q average,
 * 5 binary16 Q average, 6 RMSE {sum, count}, 7 P export, 8 sliced-ingest
 * histogram, 9 sliced-ingest rating exchange, 10 sliced-ingest block offsets.
 * Returns the number of sites through *n_sites if non-NULL. */
#define HCCMF_COMM_SITES 11
HCCMF_API hccmf_status hccmf_comm_counts(hccmf_t h, int64_t* counts, int32_t n, int32_t* n_sites);

/* Issue all further work on `stream` (a cudaStream_t, may be the legacy default
 * 0).  The caller keeps ownership of the stream and must keep it alive. */
HCCMF_API hccmf_status hccmf_set_stream(hccmf_t h, void* stream);

HCCMF_API hccmf_status hccmf_set_option(hccmf_t h, int32_t option, int64_t value);

/* Release all device memory and the NCCL communicator.  NULL is a no-op. */
HCCMF_API void hccmf_destroy(hccmf_t h);

/* Last error message of the handle ("" if none); h == NULL -> last global error. */
HCCMF_API const char* hccmf_last_error(hccmf_t h);

/* ---------------------------------------------------------------- the path */

/* a1 (preprocessing, L543-L548): copy nnz >= 0 COO ratings (u[i], v[i], r[i])
 * of R (Table 1).  Duplicated (u, v) are kept, each one update.
 * Validates 0 <= u < m, 0 <= v < n and finite r -> HCCMF_ERANGE otherwise.
 * Distributed handles: every rank passes the same global COO (each keeps only its
 * shard after hccmf_partition; see hccmf_load_ratings_slice to avoid the copies). */
HCCMF_API hccmf_status hccmf_load_ratings(hccmf_t h, const int32_t* u, const int32_t* v, const float* r, int64_t nnz);

/* a1, sharded ingest (each rank loads 1/G of the input, L543-L548 "the server
 * ... partitions the data", without the global COO on any GPU): this rank's slice
 * of the global COO.  The slices of ranks 0, 1, .., world-1 concatenated in rank
 * order ARE the global COO (any split, empty slices allowed), so every result --
 * permutation, boundaries, block offsets, the sorted records of each shard -- is
 * bit-identical to a single-process load of the concatenation.  hccmf_partition
 * then all-reduces the permuted-row histogram (boundaries), sends every rating to
 * the rank that owns its row (one all-to-all), and each rank sorts only its shard.
 * Validation as hccmf_load_ratings (ERANGE is local to the rank that holds the
 * bad rating; partition then fails collectively with ESTATE on that rank only, so
 * callers must check every rank's load status).  Single-process handles: same as
 * hccmf_load_ratings. */
HCCMF_API hccmf_status hccmf_load_ratings_slice(hccmf_t h, const int32_t* u, const int32_t* v, const float* r,
                                                int64_t nnz_local);

/* a2-a4: shuffle (seeded permutation of row and column ids), row-grid partition
 * into G shards of contiguous permuted rows balanced on nnz (DP0/1/2,
 * L881-L1172), blocking into G*B_r*B_c blocks and a stable sort by
 * (shard, row block, column block, u', o) -- the row-sorted blocks of
 * L1472-L1474 -- where o = (v' - c0 + H(seed,5,u',0) mod w) mod w is v' rotated
 * by a row-dependent offset inside the block's w columns [c0, c0+w) (DESIGN.md
 * R21; seed 0: o = v' - c0, plain column order).  Bit-exact with the oracle.
 * Collective for distributed handles. */
HCCMF_API hccmf_status hccmf_partition(hccmf_t h, const hccmf_partition_opts* opts);

/* a0: P[u][j] = U(H(seed,3,u,j)) * sqrtf(1/k), Q[v][j] = U(H(seed,4,v,j)) * sqrtf(1/k)
 * on ORIGINAL ids (R5); H is the SplitMix64-based hash of DESIGN.md R8. */
HCCMF_API hccmf_status hccmf_init_factors(hccmf_t h, uint64_t seed);

/* Set P (m x k) and Q (n x k) in ORIGINAL id order (checkpoint restore, tests).
 * Distributed handles: every rank passes the full matrices. */
HCCMF_API hccmf_status hccmf_set_factors(hccmf_t h, const float* P, const float* Q);

/* a5/a6 + a7: one epoch over every held rating:
 *   e = r - p_u.q_v;  p_u += gamma (e q_v - lambda p_u);  q_v += gamma (e p_u - lambda q_v)
 * (section 2.1; Fig. 1; p_u on the right is the pre-update value, R1),
 * in the given schedule, followed (G > 1) by the given Q synchronisation. */
HCCMF_API hccmf_status hccmf_train_epoch(hccmf_t h, hccmf_sched sched, hccmf_sync sync);

/* a8: sqrt( sum_T (r - p_u.q_v)^2 / |T| ) over nt test ratings in ORIGINAL ids
 * (Fig. 1 caption L405-L407, Fig. 7).  fp32 dot products, fp64 accumulation in a
 * fixed order (deterministic).  Distributed: all-reduced over ranks, collective. */
HCCMF_API hccmf_status hccmf_rmse(hccmf_t h, const int32_t* u, const int32_t* v, const float* r, int64_t nt, double* out);

/* a9 (final push, L1205-L1206): P (m x k) and/or Q (n x k) in ORIGINAL id order;
 * either pointer may be NULL.  Distributed: collective; every rank gets the full
 * matrices. */
HCCMF_API hccmf_status hccmf_get_factors(hccmf_t h, float* P, float* Q);

/* Partition introspection (bit-exact parity tests).  Any pointer may be NULL.
 * bounds[G+1] (int32 permuted-row boundaries b_s), block_off[G*B_r*B_c+1]
 * (int64, first record of each block in the global sorted order), perm_row[m],
 * perm_col[n] (int32, original id -> permuted id). */
HCCMF_API hccmf_status hccmf_get_partition(hccmf_t h, int32_t* bounds, int64_t* block_off, int32_t* perm_row,
                                 int32_t* perm_col);

/* Sorted records held by this handle (local_nnz of them, permuted ids).
 * Any pointer may be NULL. */
HCCMF_API hccmf_status hccmf_get_records(hccmf_t h, int32_t* u, int32_t* v, float* r);

/* Partition fractions x[G] actually used (after DP0/1/2). */
HCCMF_API hccmf_status hccmf_get_fractions(hccmf_t h, double* x);

HCCMF_API hccmf_status hccmf_get_info(hccmf_t h, hccmf_info* out);

/* Host-only (no device needed): the a5-a7 schedule that shard `shard` of a
 * distributed handle executes (shard = -1: all G logical shards of one handle).
 * Launch i runs blocks[launch_off[i] .. launch_off[i+1]) (block index
 * (s*Br + rb)*Bc + cb) concurrently at ring stage launch_stage[i]; blocks of one
 * launch share no P rows and no Q columns (DET) or no users (HOGWILD).  For RING,
 * ring[4t .. 4t+3] = Q rows [send_lo, send_hi) the shard sends to shard-1 after
 * stage t and [recv_lo, recv_hi) it receives from shard+1 (R19).
 * Size query: pass blocks or launch_off NULL (or too small *n_blocks /
 * *n_launches): the required counts are written and HCCMF_OK returned.
 * launch_off needs *n_launches + 1 entries; ring needs 4*G. */
HCCMF_API hccmf_status hccmf_schedule(int32_t G, int32_t Br, int32_t Bc, int64_t n, int32_t sched, int32_t sync,
                                      int32_t shard, int64_t* blocks, int64_t* n_blocks, int64_t* launch_off,
                                      int32_t* launch_stage, int64_t* n_launches, int64_t* ring);

/* Host-only: the time cost model of section 3.2 and the strategy choice of 3.3.
 * Worker i (p of them) has runtime memory bandwidth B[i] and bus bandwidth Bbus[i]
 * (bytes/s); the server B_server.  With D = n (q_only: Strategy 1, L1203-L1233) or
 * m + n, and elem_bytes per parameter (4 fp32, 2 fp16: Strategy 2):
 *   T_i,e = nnz (16k+4) / B_i;  x = DP0 (Eq. 6);
 *   T_i = x_i nnz (16k+4) / B_i + 2 elem k D / Bbus_i        (Eq. 2)
 *   T_sync = 3 t elem k D / B_server                          (Eq. 3)
 *   T = max T_i if max T_i / T_sync >= lambda_sync (the paper's threshold "lambda" = 10,
 *   L855-L859) and *strategy = HCCMF_DP1; else T = max T_i + T_sync, HCCMF_DP2 (Eq. 5).
 * x, T_i: [p] caller-allocated. */
HCCMF_API hccmf_status hccmf_cost_model(int32_t p, int64_t m, int64_t n, int64_t nnz, int32_t k, const double* B,
                                        const double* Bbus, double B_server, int32_t t, int32_t q_only,
                                        int32_t elem_bytes, double lambda_sync, double* x, double* T_i,
                                        double* T_sync, double* T, int32_t* strategy);

/* Diagnostic (bench.py roofline.binding_frac): the ceiling of the
 * Hogwild q_v round trip on this device.  Streams the handle's local sorted records with
 * `warps` warps (0: the Hogwild epoch's automatic count for the whole of Q), one rating
 * ahead, doing per rating only the kernel's q_v traffic into a SCRATCH copy of Q (the
 * model is not touched): mode 0 fp32 vector reductions only (red.v4.f32), 1 binary16
 * load + dependent reduction (red.v2.f16x2), 2 fp32 load + dependent reduction, 3 the
 * q_v stream alone (loads of the model's Q), 4 the p_u stream alone (per user run one load
 * of the row and one store of the same values: the model is left unchanged).  Modes 3-4
 * let ncu report the L2 hit rate of the Q and of the P stream separately.  Modes 5-9 move
 * the row through the TMA bulk-copy engine (profiles/r02_probe_tma.md): 5 bulk reductions
 * only, 7 per-lane load + bulk reduction, 6 / 8 / 9 bulk load 3 / 7 / 1 ratings ahead + a
 * dependent bulk reduction (k = 128 only).
 * *ms = mean duration of one pass over `reps` timed passes (CUDA events on the handle's
 * stream, after one warm-up pass).  On a one-shard grid (1, Bc > 1) -- a Hogwild epoch of Bc
 * column-block phases -- the probe runs phase by phase with each phase's records and warp
 * count and *ms is the sum.  Needs partition; k a multiple of 128. */
HCCMF_API hccmf_status hccmf_probe_roundtrip(hccmf_t h, int32_t mode, int64_t warps, int32_t reps, double* ms);

/* The last train_epoch's timeline (HCCMF_OPT_TIMELINE = 1): up to `cap` rows of 5 doubles
 * {kind, stage, column block, start ms, end ms}, times relative to the epoch's first
 * event, measured with CUDA events on the stream each piece ran on.  kind: 0 SGD launch,
 * 1 pipelined ring transfer of one column block (comm stream), 2 stage-wise ring
 * transfer, 3 Q average (all-reduce).  *n = rows available.  Synchronises the streams. */
HCCMF_API hccmf_status hccmf_timeline(hccmf_t h, double* rows, int64_t cap, int64_t* n);

/* Library version string, e.g. "hccmf 0.1 sm_100a". */
HCCMF_API const char* hccmf_version(void);

/* Process-wide count of the CUDA kernels this library has launched (every handle,
 * every call; CUB's internal sort/scan/select launches in hccmf_partition are not
 * counted).  Read it before and after a region to count that region's launches
 * (bench.py's gpu_launches).  Never fails. */
HCCMF_API int64_t hccmf_kernel_launches(void);

#ifdef __cplusplus
}
#endif
#endif /* HCCMF_H_ */
