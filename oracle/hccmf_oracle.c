/*
 * hccmf_oracle.c -- the plain, slow, serial CPU ORACLE for the HCC-MF hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  The product path
 * (paper_conf_icpp_huangylhbl21_b200/) never links, imports or calls it, and it
 * shares no code, header, table or constant generator with the CUDA path: every
 * function below is written from PAPER.md (Huang et al., ICPP '21) and from the
 * readings recorded in DESIGN.md section 3 ("Readings of the paper").
 *
 * Citation convention: L<n> = /root/reference/PAPER.md line n.
 *
 * Arithmetic: fp64 for every floating-point quantity (the paper fixes no
 * precision for P and Q; L1234-L1249 only mentions FP16 for transmission).
 * Build strictly: -O2 -ffp-contract=off, no -ffast-math, no OpenMP, so each
 * a*b+c is two IEEE roundings, exactly as written.
 *
 * Pins (tests/test_oracle_pins.py, -m "not gpu"): Fig. 1 worked example
 * (L283-L403), finite-difference gradient, monotone loss at small gamma,
 * planted rank-k recovery, full-batch O(gamma^2) limit, dense brute-force
 * objective, Theorem-1 equalisation (L924-L954), Eq. 6 closed form, brute-force
 * partition/sort on tiny inputs, SplitMix64 published test vectors.
 * Parity unpinned: none of the functions below is left without a pin; the
 * all-reduce replica mode is pinned only against its own definition
 * (mean of per-shard replicas) -- see DESIGN.md section 3, reading R13.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------- */
/* Counter-based hash (R8: "shuffling", L546).  SplitMix64 finaliser  */
/* as published by Steele, Lea & Flood (2014); the CUDA side implements the     */
/* same specification independently.                                           */
/* ------------------------------------------------------------------------- */
uint64_t orc_splitmix(uint64_t x)
{
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

/* H(seed, tag, a, b) = sm(sm(sm(seed ^ (tag << 56)) ^ a) ^ b) */
uint64_t orc_hash(uint64_t seed, uint64_t tag, uint64_t a, uint64_t b)
{
    uint64_t h = orc_splitmix(seed ^ (tag << 56));
    h = orc_splitmix(h ^ a);
    return orc_splitmix(h ^ b);
}

/* U[0,1) with 24 random bits: exact in fp32 and fp64. */
double orc_uniform(uint64_t h) { return (double)(h >> 40) * (1.0 / 16777216.0); }

/* ------------------------------------------------------------------------- */
/* Step 1 of the preprocessing (L543-L548): shuffle = seeded ID permutation.   */
/* perm[id] = rank of (H(seed, tag, id, 0), id) among all ids; seed 0 = identity */
/* ------------------------------------------------------------------------- */
typedef struct { uint64_t key; int64_t id; } orc_keyid;

static int cmp_keyid(const void* a, const void* b)
{
    const orc_keyid* x = (const orc_keyid*)a;
    const orc_keyid* y = (const orc_keyid*)b;
    if (x->key != y->key) return x->key < y->key ? -1 : 1;
    if (x->id != y->id) return x->id < y->id ? -1 : 1;
    return 0;
}

int orc_perm(uint64_t seed, uint64_t tag, int64_t count, int32_t* perm)
{
    if (count < 0) return -1;
    if (seed == 0) {
        for (int64_t i = 0; i < count; ++i) perm[i] = (int32_t)i;
        return 0;
    }
    orc_keyid* a = (orc_keyid*)malloc(sizeof(orc_keyid) * (size_t)(count ? count : 1));
    if (!a) return -3;
    for (int64_t i = 0; i < count; ++i) {
        a[i].key = orc_hash(seed, tag, (uint64_t)i, 0);
        a[i].id = i;
    }
    qsort(a, (size_t)count, sizeof(orc_keyid), cmp_keyid);
    for (int64_t r = 0; r < count; ++r) perm[a[r].id] = (int32_t)r;
    free(a);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Degree-balanced column permutation (R30): "shuffling" exists to    */
/* balance the blocks (L546); under the DET order every rating of a column      */
/* block is serialised through the block's owners one row block after another,   */
/* so the heaviest column block is the epoch's critical path.  Items are taken  */
/* in order of (degree descending, id ascending); each goes to the column block  */
/* with the least load (sum of degrees) among those with a free slot, ties to    */
/* the lowest block index, and takes that block's next slot.  Column block c    */
/* holds v' in [ceil(c n / B), ceil((c+1) n / B)) (a4), so it has that many     */
/* slots.  deg[v] = number of ratings of item v (original ids).                 */
/* ------------------------------------------------------------------------- */
typedef struct { int64_t deg; int64_t id; } orc_degid;

static int cmp_degid(const void* a, const void* b)
{
    const orc_degid* x = (const orc_degid*)a;
    const orc_degid* y = (const orc_degid*)b;
    if (x->deg != y->deg) return x->deg > y->deg ? -1 : 1;
    if (x->id != y->id) return x->id < y->id ? -1 : 1;
    return 0;
}

int orc_perm_balanced(int64_t n, int64_t nnz, const int32_t* v, int32_t B, int32_t* perm)
{
    if (n < 1 || B < 1 || nnz < 0) return -1;
    orc_degid* it = (orc_degid*)malloc(sizeof(orc_degid) * (size_t)n);
    int64_t* load = (int64_t*)calloc((size_t)B, sizeof(int64_t));
    int64_t* used = (int64_t*)calloc((size_t)B, sizeof(int64_t));
    if (!it || !load || !used) return -3;
    for (int64_t x = 0; x < n; ++x) { it[x].deg = 0; it[x].id = x; }
    for (int64_t i = 0; i < nnz; ++i) it[v[i]].deg += 1;
    qsort(it, (size_t)n, sizeof(orc_degid), cmp_degid);
    for (int64_t x = 0; x < n; ++x) {
        int32_t best = -1;
        for (int32_t c = 0; c < B; ++c) {
            const int64_t start = ((int64_t)c * n + B - 1) / B, end = ((int64_t)(c + 1) * n + B - 1) / B;
            if (used[c] >= end - start) continue;  /* no free slot */
            if (best < 0 || load[c] < load[best]) best = c;
        }
        const int64_t start = ((int64_t)best * n + B - 1) / B;
        perm[it[x].id] = (int32_t)(start + used[best]);
        used[best] += 1;
        load[best] += it[x].deg;
    }
    free(it);
    free(load);
    free(used);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Data partition strategies (section 3.3).                        */
/* ------------------------------------------------------------------------- */

/* DP0, Eq. 6 (L967-L981): x_i = 1 / sum_j (T_i,e / T_j,e). */
void orc_dp0(int32_t p, const double* t_e, double* x)
{
    for (int32_t i = 0; i < p; ++i) {
        double s = 0.0;
        for (int32_t j = 0; j < p; ++j) s += t_e[i] / t_e[j];
        x[i] = 1.0 / s;
    }
}

/* Theorem 1 (L924-L954) with unequal b_i: the minimiser of max_i(a_i x_i + b_i)
 * s.t. sum x_i = 1, x_i >= 0 equalises a_i x_i + b_i over the workers that get
 * data.  Water-filling: T* = (1 + sum b_j/a_j) / sum (1/a_j) over the active set;
 * workers with b_i >= T* get x_i = 0 and leave the active set. */
void orc_dp0_affine(int32_t p, const double* a, const double* b, double* x)
{
    int32_t* active = (int32_t*)malloc(sizeof(int32_t) * (size_t)(p ? p : 1));
    for (int32_t i = 0; i < p; ++i) active[i] = 1;
    for (;;) {
        double num = 1.0, den = 0.0;
        for (int32_t j = 0; j < p; ++j)
            if (active[j]) { num += b[j] / a[j]; den += 1.0 / a[j]; }
        double T = num / den;
        int changed = 0;
        for (int32_t j = 0; j < p; ++j)
            if (active[j] && b[j] >= T) { active[j] = 0; changed = 1; }
        if (!changed) {
            for (int32_t j = 0; j < p; ++j) x[j] = active[j] ? (T - b[j]) / a[j] : 0.0;
            break;
        }
    }
    free(active);
}

/* DP1, Algorithm 1 (L1025-L1142) generalised to a GPU-only box (R11):
 * per-shard compensation toward the mean time, renormalised, stop when
 * max_s |t_s - Tbar| / min_s t_s <= 0.1, at most 8 rounds.  The re-measurement
 * of line 12 (sgd_update) uses the paper's constant-bandwidth observation
 * (L1013-L1016): t_s scales linearly with x_s.  Returns the number of rounds. */
int32_t orc_dp1(int32_t p, const double* x_in, const double* t_in, double* x_out)
{
    double* x = (double*)malloc(sizeof(double) * (size_t)p);
    double* t = (double*)malloc(sizeof(double) * (size_t)p);
    memcpy(x, x_in, sizeof(double) * (size_t)p);
    memcpy(t, t_in, sizeof(double) * (size_t)p);
    int32_t it = 0;
    for (; it < 8; ++it) {
        double tbar = 0.0, tmin = t[0], dev = 0.0;
        for (int32_t s = 0; s < p; ++s) tbar += t[s];
        tbar /= (double)p;
        for (int32_t s = 0; s < p; ++s) {
            if (t[s] < tmin) tmin = t[s];
            double d = fabs(t[s] - tbar);
            if (d > dev) dev = d;
        }
        if (dev / tmin <= 0.1) break;
        double sum = 0.0;
        for (int32_t s = 0; s < p; ++s) sum += x[s] * tbar / t[s];
        for (int32_t s = 0; s < p; ++s) {
            double xn = (x[s] * tbar / t[s]) / sum;
            t[s] = t[s] * xn / x[s];
            x[s] = xn;
        }
    }
    memcpy(x_out, x, sizeof(double) * (size_t)p);
    free(x);
    free(t);
    return it;
}

/* DP2, Eq. 7 (L1143-L1172) (R12): the shard s_med = (p-1)/2 keeps its
 * DP1 time T_med = t[s_med]; shard s targets T_s = T_med + (s - s_med) * T_sync so
 * that shard s's sync hides under shard s+1's compute; x_s <- x_s * T_s / t_s
 * (line 6 of Algorithm 1, the "similar method"), renormalised. */
void orc_dp2(int32_t p, const double* x_in, const double* t_in, double t_sync, double* x_out)
{
    int32_t smed = (p - 1) / 2;
    double tmed = t_in[smed];
    double sum = 0.0;
    for (int32_t s = 0; s < p; ++s) {
        double Ts = tmed + (double)(s - smed) * t_sync;
        if (Ts < 0.0) Ts = 0.0;
        x_out[s] = x_in[s] * Ts / t_in[s];
        sum += x_out[s];
    }
    for (int32_t s = 0; s < p; ++s) x_out[s] /= sum;
}

/* Row grid (L881-L895): per-row counts in permuted order, exclusive prefix S
 * (S has m+1 entries), and shard boundaries b_0 = 0 <= ... <= b_G = m where b_s
 * is the row r in [b_{s-1}, m] minimising |S[r] - llround(nnz * sum_{j<s} x_j)|,
 * ties to the smaller r (R10).  Brute-force linear scan. */
void orc_row_prefix(int64_t m, int64_t nnz, const int32_t* u, const int32_t* perm_row, int64_t* S)
{
    int64_t* cnt = (int64_t*)calloc((size_t)(m + 1), sizeof(int64_t));
    for (int64_t i = 0; i < nnz; ++i) cnt[perm_row[u[i]]] += 1;
    S[0] = 0;
    for (int64_t r = 0; r < m; ++r) S[r + 1] = S[r] + cnt[r];
    free(cnt);
}

void orc_bounds(int64_t m, int64_t nnz, const int64_t* S, int32_t G, const double* x, int32_t* b)
{
    double cum = 0.0;
    b[0] = 0;
    for (int32_t s = 1; s < G; ++s) {
        cum += x[s - 1];
        int64_t T = llround((double)nnz * cum);
        int64_t best = b[s - 1];
        for (int64_t r = b[s - 1]; r <= m; ++r) {
            int64_t dr = S[r] - T, db = S[best] - T;
            if (dr < 0) dr = -dr;
            if (db < 0) db = -db;
            if (dr < db) best = r;
        }
        b[s] = (int32_t)best;
    }
    b[G] = (int32_t)m;
}

/* ------------------------------------------------------------------------- */
/* Blocking + stable sort (L546 "sorting", L1472-L1474 row-sorted blocks).      */
/* Record i goes to shard s (b_s <= u' < b_{s+1}), row block                     */
/* rb = floor((u'-b_s) * Br / (b_{s+1}-b_s)), column block cb = floor(v' * Bc / n),*/
/* and records are ordered by (s, rb, cb, u', o, i) where o orders a row's       */
/* ratings inside the block: the block's columns [c0, c1), c0 = ceil(cb n / Bc), */
/* rotated by a row-dependent offset (R21):                            */
/*   o = (v' - c0 + rot(u')) mod (c1 - c0),  rot(u') = H(seed, 5, u', 0) mod (c1 - c0) */
/* seed 0: rot = 0, plain column order.                                          */
/* off[((s*Br + rb)*Bc + cb)] = first record of the block; off has G*Br*Bc+1.    */
/* ------------------------------------------------------------------------- */
typedef struct { int64_t blk; int32_t up; int64_t o; int64_t i; } orc_rec;

static int cmp_rec(const void* a, const void* b)
{
    const orc_rec* x = (const orc_rec*)a;
    const orc_rec* y = (const orc_rec*)b;
    if (x->blk != y->blk) return x->blk < y->blk ? -1 : 1;
    if (x->up != y->up) return x->up < y->up ? -1 : 1;
    if (x->o != y->o) return x->o < y->o ? -1 : 1;
    if (x->i != y->i) return x->i < y->i ? -1 : 1;
    return 0;
}

int orc_block_sort(int64_t m, int64_t n, int64_t nnz, const int32_t* u, const int32_t* v,
                   const float* r, int32_t G, int32_t Br, int32_t Bc, const int32_t* b,
                   const int32_t* perm_row, const int32_t* perm_col, uint64_t seed, int32_t* out_u,
                   int32_t* out_v, float* out_r, int64_t* off)
{
    int64_t nblk = (int64_t)G * Br * Bc;
    orc_rec* a = (orc_rec*)malloc(sizeof(orc_rec) * (size_t)(nnz ? nnz : 1));
    if (!a) return -3;
    for (int64_t i = 0; i < nnz; ++i) {
        int32_t up = perm_row[u[i]], vp = perm_col[v[i]];
        int32_t s = 0;
        while (!(b[s] <= up && up < b[s + 1])) ++s;
        int64_t rows = (int64_t)b[s + 1] - b[s];
        int64_t rb = ((int64_t)(up - b[s]) * Br) / rows;
        int64_t cb = ((int64_t)vp * Bc) / n;
        int64_t c0 = (cb * n + Bc - 1) / Bc, c1 = ((cb + 1) * n + Bc - 1) / Bc, w = c1 - c0;
        int64_t rot = seed ? (int64_t)(orc_hash(seed, 5, (uint64_t)up, 0) % (uint64_t)w) : 0;
        a[i].blk = ((int64_t)s * Br + rb) * Bc + cb;
        a[i].up = up;
        a[i].o = (vp - c0 + rot) % w;
        a[i].i = i;
    }
    qsort(a, (size_t)nnz, sizeof(orc_rec), cmp_rec);
    for (int64_t j = 0; j <= nblk; ++j) off[j] = 0;
    for (int64_t j = 0; j < nnz; ++j) off[a[j].blk + 1] += 1;
    for (int64_t j = 0; j < nblk; ++j) off[j + 1] += off[j];
    for (int64_t j = 0; j < nnz; ++j) {
        out_u[j] = a[j].up;
        out_v[j] = perm_col[v[a[j].i]];
        out_r[j] = r[a[j].i];
    }
    free(a);
    (void)m;
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Factor initialisation (R5; the paper is silent): on ORIGINAL ids, */
/* P[u][j] = U(H(seed,3,u,j)) * sqrt(1/k), Q[v][j] = U(H(seed,4,v,j)) * sqrt(1/k).*/
/* Stored in permuted order: P'[perm_row[u]] = P[u].                           */
/* ------------------------------------------------------------------------- */
void orc_init(uint64_t seed, int64_t m, int64_t n, int32_t k, const int32_t* perm_row,
              const int32_t* perm_col, double* P, double* Q)
{
    double sc = sqrt(1.0 / (double)k);
    for (int64_t u = 0; u < m; ++u)
        for (int32_t j = 0; j < k; ++j)
            P[(int64_t)perm_row[u] * k + j] = orc_uniform(orc_hash(seed, 3, (uint64_t)u, (uint64_t)j)) * sc;
    for (int64_t v = 0; v < n; ++v)
        for (int32_t j = 0; j < k; ++j)
            Q[(int64_t)perm_col[v] * k + j] = orc_uniform(orc_hash(seed, 4, (uint64_t)v, (uint64_t)j)) * sc;
}

/* ------------------------------------------------------------------------- */
/* The per-rating SGD update (section 2.1, Fig. 1,          */
/* north_star; R1 old-p reading, R2 gamma absorbs the factor 2):      */
/*   e  = r - p.q                                                              */
/*   p' = p + gamma (e q - lambda p)                                           */
/*   q' = q + gamma (e p - lambda q)      (p = value before this update)       */
/* Returns e.                                                                  */
/* ------------------------------------------------------------------------- */
double orc_round_half(double x);

/* Storage of Q (R26).  0: Q as computed (fp64 here).   */
/* 1: Q is stored in IEEE binary16: every write of q_v keeps the binary16 value   */
/* nearest to the update's result (orc_round_half), and an epoch starts from Q    */
/* rounded to binary16.  2: as 1, but the write is a binary16 ADD of the          */
/* increment: q <- rn16(q + rn16(gamma (e p - lambda q))) (Hogwild's component-   */
/* wise atomic add on binary16 words).  P is never rounded.  Set per call by      */
/* orc_epoch_q16.                                                                 */
static int g_q16 = 0;
static uint32_t g_sr_epoch = 0; /* mode 3 (stochastic rounding): epoch t of the random words */
static int64_t g_sr_rec = 0;    /* mode 3: global index of the record being updated          */

/* Stochastic rounding to binary16 (storage = 2, R27), from its definition:
 * y = sign(x) * floor((|x| + R13 * ulp / 2^13) / ulp) * ulp, with ulp the binary16 spacing
 * at |x| (2^(e-10) for |x| in [2^e, 2^(e+1)), e >= -14; 2^-24 below 2^-14) and R13 in
 * [0, 2^13) random: the result is one of the two binary16 neighbours of x, the upper
 * one with probability (fraction of x past the lower one) quantised to 2^-13 ulp. */
double orc_round_half_sr(double x, uint32_t r13)
{
    if (x != x) return x;
    double a = fabs(x);
    if (a == 0.0) return x;
    int e;
    frexp(a, &e);
    int lead = e - 1;
    if (lead < -14) lead = -14;
    double ulp = ldexp(1.0, lead - 10);
    double y = floor((a + (double)(r13 & 0x1FFFu) * ulp / 8192.0) / ulp) * ulp;
    if (y >= 65536.0) y = INFINITY;
    return x < 0 ? -y : y;
}

/* The random word of element pair c (elements 2c, 2c+1) for the q write of record i in
 * epoch t (R27): for even c, lowbias32(i*0x9E3779B1 + t*0x85EBCA77 + c*0xC2B2AE3D mod 2^32),
 * with lowbias32 the 32-bit finaliser of C. Wellons (xorshift-multiply, 2 rounds); for odd
 * c, the word of pair c-1 times 0x9E3779B1 mod 2^32.  Element 2c takes bits 12:0, element
 * 2c+1 bits 28:16. */
uint32_t orc_sr_word(int64_t i, uint32_t t, uint32_t c)
{
    if (c & 1u) return orc_sr_word(i, t, c - 1u) * 0x9E3779B1u;
    uint32_t x = (uint32_t)i * 0x9E3779B1u + t * 0x85EBCA77u + c * 0xC2B2AE3Du;
    x ^= x >> 16;
    x *= 0x7FEB352Du;
    x ^= x >> 15;
    x *= 0x846CA68Bu;
    x ^= x >> 16;
    return x;
}

double orc_sgd_update(int32_t k, double gamma, double lambda, double* p, double* q, double r)
{
    double d = 0.0;
    for (int32_t j = 0; j < k; ++j) d += p[j] * q[j];
    double e = r - d;
    for (int32_t j = 0; j < k; ++j) {
        double pj = p[j], qj = q[j];
        p[j] = pj + gamma * (e * qj - lambda * pj);
        if (g_q16 == 3) {
            uint32_t w = orc_sr_word(g_sr_rec, g_sr_epoch, (uint32_t)(j / 2));
            q[j] = orc_round_half_sr(qj + gamma * (e * pj - lambda * qj), (j % 2 == 0) ? (w & 0x1FFFu) : ((w >> 16) & 0x1FFFu));
        } else if (g_q16 == 2)
            q[j] = orc_round_half(qj + orc_round_half(gamma * (e * pj - lambda * qj)));
        else if (g_q16 == 1)
            q[j] = orc_round_half(qj + gamma * (e * pj - lambda * qj));
        else
            q[j] = qj + gamma * (e * pj - lambda * qj);
    }
    return e;
}

/* Serial pass over records [lo, hi) in stored order. */
void orc_run(int64_t lo, int64_t hi, int32_t k, double gamma, double lambda, const int32_t* ru,
             const int32_t* rv, const float* rr, double* P, double* Q)
{
    for (int64_t i = lo; i < hi; ++i) {
        g_sr_rec = i;
        orc_sgd_update(k, gamma, lambda, P + (int64_t)ru[i] * k, Q + (int64_t)rv[i] * k, (double)rr[i]);
    }
}

/* One epoch in the canonical serialisation of a schedule (R19).
 *   sched 0 = DET (conflict-free strata, L2269-L2275), 1 = SERIAL (the record
 *   order the Hogwild mode races through, L216-L219).
 *   sync  0 = NONE (G == 1), 1 = RING (rotating Q column groups, L1143-L1172,
 *   L1251-L1269), 2 = ALLREDUCE_AVG (per-shard Q replica, then the server's
 *   multiply-add sync Q = sum_s Q_s / G, L549-L557, L783-L784).
 * DET needs Br == Bc (NONE, ALLREDUCE) or Bc == G*Br (RING).
 * Returns 0, or -1 for an invalid grid. */
static void det_square(int32_t s, int32_t c, int32_t Br, int32_t Bc, int32_t col0, const int64_t* off,
                       int32_t k, double gamma, double lambda, const int32_t* ru, const int32_t* rv,
                       const float* rr, double* P, double* Q)
{
    for (int32_t t = 0; t < c; ++t)
        for (int32_t i = 0; i < c; ++i) {
            int64_t blk = ((int64_t)s * Br + i) * Bc + col0 + (i + t) % c;
            orc_run(off[blk], off[blk + 1], k, gamma, lambda, ru, rv, rr, P, Q);
        }
}

int orc_epoch(int32_t sched, int32_t sync, int32_t G, int32_t Br, int32_t Bc, const int64_t* off,
              int64_t n, int32_t k, double gamma, double lambda, const int32_t* ru, const int32_t* rv,
              const float* rr, double* P, double* Q)
{
    if (sync == 0) {
        if (G != 1) return -1;
        if (sched == 0) {
            if (Br != Bc) return -1;
            det_square(0, Br, Br, Bc, 0, off, k, gamma, lambda, ru, rv, rr, P, Q);
        } else {
            orc_run(0, off[(int64_t)Br * Bc], k, gamma, lambda, ru, rv, rr, P, Q);
        }
        return 0;
    }
    if (sync == 1) {
        if (Bc % G != 0) return -1;
        int32_t c = Bc / G;
        if (sched == 0 && c != Br) return -1;
        for (int32_t t = 0; t < G; ++t)
            for (int32_t s = 0; s < G; ++s) {
                int32_t g = (s + t) % G;
                if (sched == 0) {
                    det_square(s, c, Br, Bc, g * c, off, k, gamma, lambda, ru, rv, rr, P, Q);
                } else {
                    for (int32_t j = 0; j < c; ++j)
                        for (int32_t rb = 0; rb < Br; ++rb) {
                            int64_t blk = ((int64_t)s * Br + rb) * Bc + g * c + j;
                            orc_run(off[blk], off[blk + 1], k, gamma, lambda, ru, rv, rr, P, Q);
                        }
                }
            }
        return 0;
    }
    if (sync == 2) {
        if (sched == 0 && Br != Bc) return -1;
        size_t qn = (size_t)n * (size_t)k;
        double* Qs = (double*)malloc(sizeof(double) * qn);
        double* Qsum = (double*)calloc(qn, sizeof(double));
        for (int32_t s = 0; s < G; ++s) {
            memcpy(Qs, Q, sizeof(double) * qn);
            if (sched == 0) {
                det_square(s, Br, Br, Bc, 0, off, k, gamma, lambda, ru, rv, rr, P, Qs);
            } else {
                int64_t lo = off[(int64_t)s * Br * Bc], hi = off[(int64_t)(s + 1) * Br * Bc];
                orc_run(lo, hi, k, gamma, lambda, ru, rv, rr, P, Qs);
            }
            for (size_t i = 0; i < qn; ++i) Qsum[i] += Qs[i];
        }
        for (size_t i = 0; i < qn; ++i) Q[i] = Qsum[i] / (double)G;
        free(Qs);
        free(Qsum);
        return 0;
    }
    return -1;
}

/* ------------------------------------------------------------------------- */
/* Evaluation (Fig. 1 caption L405-L407; Fig. 7).                              */
/* RMSE over a set T given in ORIGINAL ids: sqrt(sum (r - p_u.q_v)^2 / |T|).   */
/* ------------------------------------------------------------------------- */
double orc_rmse(int64_t nt, const int32_t* tu, const int32_t* tv, const float* tr, int32_t k,
                const int32_t* perm_row, const int32_t* perm_col, const double* P, const double* Q)
{
    if (nt == 0) return 0.0;
    double sse = 0.0;
    for (int64_t i = 0; i < nt; ++i) {
        const double* p = P + (int64_t)perm_row[tu[i]] * k;
        const double* q = Q + (int64_t)perm_col[tv[i]] * k;
        double d = 0.0;
        for (int32_t j = 0; j < k; ++j) d += p[j] * q[j];
        double e = (double)tr[i] - d;
        sse += e * e;
    }
    return sqrt(sse / (double)nt);
}

/* Objective over the training set in ORIGINAL ids (R2, R4):
 * L = sum_Omega [ (r - p_u.q_v)^2 + lambda (|p_u|^2 + |q_v|^2) ]. */
double orc_objective(int64_t nnz, const int32_t* u, const int32_t* v, const float* r, int32_t k,
                     double lambda, const int32_t* perm_row, const int32_t* perm_col, const double* P,
                     const double* Q)
{
    double L = 0.0;
    for (int64_t i = 0; i < nnz; ++i) {
        const double* p = P + (int64_t)perm_row[u[i]] * k;
        const double* q = Q + (int64_t)perm_col[v[i]] * k;
        double d = 0.0, pp = 0.0, qq = 0.0;
        for (int32_t j = 0; j < k; ++j) {
            d += p[j] * q[j];
            pp += p[j] * p[j];
            qq += q[j] * q[j];
        }
        double e = (double)r[i] - d;
        L += e * e + lambda * (pp + qq);
    }
    return L;
}

/* Export (final push, L1205-L1206): un-permute to original ids. */
void orc_unpermute(int64_t rows, int32_t k, const int32_t* perm, const double* Xp, double* X)
{
    for (int64_t i = 0; i < rows; ++i)
        memcpy(X + i * k, Xp + (int64_t)perm[i] * k, sizeof(double) * (size_t)k);
}

/* ------------------------------------------------------------------------- */
/* Time cost model (section 3.2, Eq. 1-5) and the strategy choice    */
/* (section 3.3): per worker i with runtime memory bandwidth B_i and bus        */
/* bandwidth Bbus_i, elem bytes per parameter (R18):                           */
/*   T_i,e   = nnz (16k + 4) / B_i                       (whole data, Eq. 2)   */
/*   x       = DP0 (Eq. 6 on T_i,e)                                            */
/*   T_i     = x_i nnz (16k + 4) / B_i + 2 elem k D / Bbus_i   (Eq. 2)          */
/*   T_sync  = 3 t elem k D / B_server                        (Eq. 3)          */
/*   D = n (Strategy 1, only Q moves, L1203-L1233) or m + n                     */
/*   T = max T_i           if max T_i / T_sync >= lambda_sync  (Eq. 5)         */
/*     = max T_i + T_sync  otherwise                                           */
/* Returns 1 when the sync term is negligible (DP1 applies), 2 otherwise (DP2). */
/* ------------------------------------------------------------------------- */
int32_t orc_cost_model(int32_t p, int64_t m, int64_t n, int64_t nnz, int32_t k, const double* B,
                       const double* Bbus, double B_server, int32_t t, int32_t q_only, int32_t elem,
                       double lambda_sync, double* x, double* T_i, double* T_sync, double* T)
{
    double D = q_only ? (double)n : (double)(m + n);
    double* Te = (double*)malloc(sizeof(double) * (size_t)p);
    for (int32_t i = 0; i < p; ++i) Te[i] = (double)nnz * (16.0 * k + 4.0) / B[i];
    orc_dp0(p, Te, x);
    double Tmax = 0.0;
    for (int32_t i = 0; i < p; ++i) {
        T_i[i] = x[i] * (double)nnz * (16.0 * k + 4.0) / B[i] + 2.0 * elem * k * D / Bbus[i];
        if (T_i[i] > Tmax) Tmax = T_i[i];
    }
    *T_sync = 3.0 * t * elem * k * D / B_server;
    free(Te);
    if (Tmax / *T_sync >= lambda_sync) {
        *T = Tmax;
        return 1;
    }
    *T = Tmax + *T_sync;
    return 2;
}

/* Sub-epoch synchronisation (Strategy 3's several pull-compute-push
 * pipelines per epoch, L1251-L1269, Fig. 6; R22): the all-reduce mode in
 * `phases` rounds.  Round phi runs, on every shard's own copy of Q, the shard's row
 * blocks [phi*Br/phases, (phi+1)*Br/phases) -- every column block of each, records
 * in stored order -- and then Q = (sum_s Q_s) / G.  phases = 1 is
 * orc_epoch(serial, allreduce).  Needs Br % phases == 0; returns -1 otherwise. */
int orc_epoch_phased(int32_t G, int32_t Br, int32_t Bc, int32_t phases, const int64_t* off, int64_t n,
                     int32_t k, double gamma, double lambda, const int32_t* ru, const int32_t* rv,
                     const float* rr, double* P, double* Q)
{
    if (phases < 1 || Br % phases != 0) return -1;
    int32_t per = Br / phases;
    size_t qn = (size_t)n * (size_t)k;
    double* Qs = (double*)malloc(sizeof(double) * qn);
    double* Qsum = (double*)malloc(sizeof(double) * qn);
    for (int32_t ph = 0; ph < phases; ++ph) {
        memset(Qsum, 0, sizeof(double) * qn);
        for (int32_t s = 0; s < G; ++s) {
            memcpy(Qs, Q, sizeof(double) * qn);
            for (int32_t rb = ph * per; rb < (ph + 1) * per; ++rb)
                for (int32_t cb = 0; cb < Bc; ++cb) {
                    int64_t blk = ((int64_t)s * Br + rb) * Bc + cb;
                    orc_run(off[blk], off[blk + 1], k, gamma, lambda, ru, rv, rr, P, Qs);
                }
            for (size_t i = 0; i < qn; ++i) Qsum[i] += Qs[i];
        }
        for (size_t i = 0; i < qn; ++i) Q[i] = Qsum[i] / (double)G;
    }
    free(Qs);
    free(Qsum);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Strategy 2, "Transmitting FP16 Data" (L1234-L1249): Q travels as IEEE-754     */
/* binary16.  orc_round_half returns the binary16 value nearest to x (ties to    */
/* even), as a double: the pack -> unpack a transfer applies.  Written from the */
/* format's definition (1 sign, 5 exponent bits with bias 15, 10 fraction bits, */
/* subnormals below 2^-14, largest finite 65504); overflow gives +-inf.          */
/* ------------------------------------------------------------------------- */
double orc_round_half(double x)
{
    if (x != x) return x;
    double a = fabs(x);
    if (a == 0.0) return x;
    if (a >= 65520.0) return x > 0 ? INFINITY : -INFINITY; /* 65504 + half an ulp (16) rounds up */
    int e;
    frexp(a, &e);                        /* a = f * 2^e, f in [0.5, 1) -> leading bit 2^(e-1) */
    int lead = e - 1;
    if (lead < -14) lead = -14;          /* subnormal range: fixed spacing 2^-24 */
    double ulp = ldexp(1.0, lead - 10);
    double q = a / ulp;                  /* exact: ulp is a power of two */
    double fl = floor(q), rem = q - fl;
    double r = fl;
    if (rem > 0.5 || (rem == 0.5 && fmod(fl, 2.0) != 0.0)) r = fl + 1.0;
    double y = r * ulp;
    if (y >= 65520.0) y = INFINITY;
    return x < 0 ? -y : y;
}

/* Ring / all-reduce epoch with FP16 transmission (R25).  RING: after
 * stage t, the column group each shard held, (s+t) mod G, has been shipped as
 * binary16 -> its Q rows are rounded.  ALLREDUCE: every shard's copy is rounded
 * before the mean and the mean is rounded again (it comes back as binary16).
 * Same grid rules as orc_epoch. */
int orc_epoch_wire16(int32_t sched, int32_t sync, int32_t G, int32_t Br, int32_t Bc, const int64_t* off,
                     int64_t n, int32_t k, double gamma, double lambda, const int32_t* ru, const int32_t* rv,
                     const float* rr, double* P, double* Q)
{
    if (sync == 1) {
        if (Bc % G != 0) return -1;
        int32_t c = Bc / G;
        if (sched == 0 && c != Br) return -1;
        for (int32_t t = 0; t < G; ++t) {
            for (int32_t s = 0; s < G; ++s) {
                int32_t g = (s + t) % G;
                if (sched == 0) {
                    det_square(s, c, Br, Bc, g * c, off, k, gamma, lambda, ru, rv, rr, P, Q);
                } else {
                    for (int32_t j = 0; j < c; ++j)
                        for (int32_t rb = 0; rb < Br; ++rb) {
                            int64_t blk = ((int64_t)s * Br + rb) * Bc + g * c + j;
                            orc_run(off[blk], off[blk + 1], k, gamma, lambda, ru, rv, rr, P, Q);
                        }
                }
            }
            for (int32_t g = 0; g < G; ++g) { /* every group moved once at the end of stage t */
                int64_t a = ((int64_t)g * c * n + Bc - 1) / Bc, b = ((int64_t)(g + 1) * c * n + Bc - 1) / Bc;
                for (int64_t i = a * k; i < b * k; ++i) Q[i] = orc_round_half(Q[i]);
            }
        }
        return 0;
    }
    if (sync == 2) {
        if (sched == 0 && Br != Bc) return -1;
        size_t qn = (size_t)n * (size_t)k;
        double* Qs = (double*)malloc(sizeof(double) * qn);
        double* Qsum = (double*)calloc(qn, sizeof(double));
        for (int32_t s = 0; s < G; ++s) {
            memcpy(Qs, Q, sizeof(double) * qn);
            if (sched == 0) {
                det_square(s, Br, Br, Bc, 0, off, k, gamma, lambda, ru, rv, rr, P, Qs);
            } else {
                int64_t lo = off[(int64_t)s * Br * Bc], hi = off[(int64_t)(s + 1) * Br * Bc];
                orc_run(lo, hi, k, gamma, lambda, ru, rv, rr, P, Qs);
            }
            for (size_t i = 0; i < qn; ++i) Qsum[i] += orc_round_half(Qs[i]);
        }
        for (size_t i = 0; i < qn; ++i) Q[i] = orc_round_half(Qsum[i] / (double)G);
        free(Qs);
        free(Qsum);
        return 0;
    }
    return -1;
}

/* orc_epoch with Q stored in binary16 (storage = 1, R26): Q is rounded
 * to binary16 first (the epoch starts from stored values), then every q_v write
 * is rounded (orc_sgd_update; add16 = 1: as a binary16 add of the rounded
 * increment; sr = 1: stochastically rounded with the random words of epoch t,
 * storage = 2, R27).  Same schedules, grids and return codes.  Record indices are
 * positions in the sorted record array (global order). */
int orc_epoch_q16(int32_t sched, int32_t sync, int32_t G, int32_t Br, int32_t Bc, const int64_t* off,
                  int64_t n, int32_t k, double gamma, double lambda, const int32_t* ru, const int32_t* rv,
                  const float* rr, double* P, double* Q, int32_t add16, int32_t sr, uint32_t t)
{
    size_t qn = (size_t)n * (size_t)k;
    for (size_t i = 0; i < qn; ++i) Q[i] = orc_round_half(Q[i]);
    g_q16 = sr ? 3 : (add16 ? 2 : 1);
    g_sr_epoch = t;
    int rc = orc_epoch(sched, sync, G, Br, Bc, off, n, k, gamma, lambda, ru, rv, rr, P, Q);
    g_q16 = 0;
    return rc;
}
