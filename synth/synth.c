/*
 * synth.c — seeded synthetic sparse-matrix and vector generators.
 *
 * This module is INPUT GENERATION ONLY.  It holds none of the DASP method's
 * arithmetic (no classification, packing or SpMV).  It is the one piece of
 * code shared by the oracle tests (oracle/), the GPU parity tests (tests/) and
 * bench.py; the recipes are stated in DESIGN.md §"Input recipe".
 *
 * Every random number is a pure function of (seed, row, k) through a
 * counter-based splitmix64 hash, so any row range can be regenerated
 * independently (each rank of the multi-GPU mode builds only its slab).
 *
 * Matrices are produced in two passes:
 *   synth_row_lengths(kind, p, row0, nrows, len)        -> len[nrows]
 *   synth_fill(kind, p, row0, nrows, row_ptr, col, val)  -> CSR slice
 * where row_ptr is the caller's LOCAL prefix sum of len (row_ptr[0] = 0).
 * Columns within a row are distinct and ascending.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum {
    SYN_UNIFORM = 0,   /* C1a: len ~ Poisson(mean), uniform columns            */
    SYN_MIX = 1,       /* C1b: class-coverage mix (empty/1/2/3/4/medium/long)  */
    SYN_STENCIL27 = 2, /* C2 : 3-D 27-point stencil on nx*ny*nz                */
    SYN_POWERLAW = 3,  /* C3 : power-law row lengths, local + Zipf columns     */
    SYN_MIXED64 = 4,   /* C5 : mixed-class, mean row length ~64, |row|_1 <= 1  */
    SYN_SHORT = 5,     /* C6 : short rows only, len U{1..4}                    */
    SYN_LENLIST = 6    /* lengths given by the caller (edge-case tests)        */
};

enum { VAL_UNIFORM = 0, VAL_INT = 1, VAL_ONES = 2, VAL_SPD = 3 };

typedef struct {
    int64_t m, n;
    uint64_t seed;
    int32_t val_mode;   /* VAL_* */
    int32_t nx, ny, nz; /* stencil */
    double mean;        /* UNIFORM: Poisson mean */
    double gamma;       /* POWERLAW exponent */
    int64_t kmax;       /* POWERLAW max row length */
    int64_t n_forced;   /* POWERLAW rows forced to kmax */
    double local_frac;  /* POWERLAW fraction of local columns */
    int64_t local_w;    /* POWERLAW local half-width */
    double zipf_s;      /* POWERLAW Zipf exponent of hub columns */
    const int64_t* lenlist; /* LENLIST: lengths of rows [0, m) */
} synth_params;

/* ---- counter-based RNG (splitmix64 finaliser) ---- */
static inline uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
static inline uint64_t rng3(uint64_t seed, uint64_t row, uint64_t k) {
    return mix64(mix64(seed * 0xD1B54A32D192ED03ull ^ row) ^ (k * 0xA24BAED4963EE407ull + 0x5851F42D4C957F2Dull));
}
static inline double u01(uint64_t r) { return (double)(r >> 11) * 0x1.0p-53; }

/* streams: k values reserved for row-level draws */
#define K_LEN   0xFFFFFFFF00000001ull
#define K_LEN2  0xFFFFFFFF00000002ull
#define K_COL(k) (2ull * (uint64_t)(k))
#define K_VAL(k) (2ull * (uint64_t)(k) + 1ull)

/* ---- power-law length table (discrete P(k) ∝ k^-gamma on [1,kmax]) ---- */
static double* pl_cdf = 0;
static double pl_gamma = -1.0;
static int64_t pl_kmax = -1;
static void pl_table(double gamma, int64_t kmax) {
    if (pl_cdf && pl_gamma == gamma && pl_kmax == kmax) return;
    free(pl_cdf);
    pl_cdf = (double*)malloc(sizeof(double) * (size_t)kmax);
    double s = 0.0;
    for (int64_t k = 1; k <= kmax; ++k) { s += pow((double)k, -gamma); pl_cdf[k - 1] = s; }
    for (int64_t k = 0; k < kmax; ++k) pl_cdf[k] /= s;
    pl_cdf[kmax - 1] = 1.0;
    pl_gamma = gamma; pl_kmax = kmax;
}
static int64_t pl_sample(double u) { /* smallest k with cdf[k-1] > u */
    int64_t lo = 0, hi = pl_kmax - 1;
    while (lo < hi) { int64_t mid = (lo + hi) >> 1; if (pl_cdf[mid] > u) hi = mid; else lo = mid + 1; }
    return lo + 1;
}
/* mean of the (untruncated-by-forcing) power-law length distribution */
double synth_powerlaw_mean(double gamma, int64_t kmax) {
    pl_table(gamma, kmax);
    double mean = 0.0, prev = 0.0;
    for (int64_t k = 1; k <= kmax; ++k) { mean += (double)k * (pl_cdf[k - 1] - prev); prev = pl_cdf[k - 1]; }
    return mean;
}

static int64_t poisson(double mean, double u) {
    double p = exp(-mean), c = p; int64_t k = 0;
    while (u > c && k < 100000) { ++k; p *= mean / (double)k; c += p; }
    return k;
}

static int is_forced(const synth_params* p, int64_t row) {
    if (p->n_forced <= 0) return 0;
    /* forced rows: floor((j + 0.5) * m / n_forced) */
    for (int64_t j = 0; j < p->n_forced; ++j)
        if ((int64_t)(((double)j + 0.5) * (double)p->m / (double)p->n_forced) == row) return 1;
    return 0;
}

static int64_t row_len(int kind, const synth_params* p, int64_t row) {
    uint64_t s = p->seed;
    int64_t L = 0;
    switch (kind) {
    case SYN_UNIFORM: L = poisson(p->mean, u01(rng3(s, row, K_LEN))); break;
    case SYN_MIX: {
        static const int64_t longs[5] = {257, 300, 1000, 2048, 4096};
        for (int j = 0; j < 5; ++j) if (row == (int64_t)(j + 1) * p->m / 6) return longs[j] > p->n ? p->n : longs[j];
        double u = u01(rng3(s, row, K_LEN));
        if (u < 0.10) L = 0;
        else if (u < 0.25) L = 1;
        else if (u < 0.35) L = 2;
        else if (u < 0.45) L = 3;
        else if (u < 0.50) L = 4;
        else L = 5 + (int64_t)(u01(rng3(s, row, K_LEN2)) * 52.0); /* U[5,56] */
        break;
    }
    case SYN_STENCIL27: {
        int64_t nx = p->nx, ny = p->ny, nz = p->nz;
        int64_t x = row % nx, y = (row / nx) % ny, z = row / (nx * ny);
        int64_t cx = 1 + (x > 0) + (x < nx - 1), cy = 1 + (y > 0) + (y < ny - 1), cz = 1 + (z > 0) + (z < nz - 1);
        L = cx * cy * cz;
        break;
    }
    case SYN_POWERLAW:
        if (is_forced(p, row)) L = p->kmax;
        else { pl_table(p->gamma, p->kmax); L = pl_sample(u01(rng3(s, row, K_LEN))); }
        break;
    case SYN_MIXED64: {
        double u = u01(rng3(s, row, K_LEN)), v = u01(rng3(s, row, K_LEN2));
        if (u < 0.50) L = 1 + (int64_t)(v * 4.0);              /* short  U{1..4}      */
        else if (u < 0.995) L = 5 + (int64_t)(v * 152.0);       /* medium U[5,156]     */
        else if (u < 0.99995) L = (int64_t)exp(log(257.0) + v * (log(20000.0) - log(257.0))); /* long */
        else L = 100000;
        break;
    }
    case SYN_SHORT: L = 1 + (int64_t)(u01(rng3(s, row, K_LEN)) * 4.0); break;
    case SYN_LENLIST: L = p->lenlist[row]; break;
    default: L = 0;
    }
    if (L > p->n) L = p->n;
    if (L < 0) L = 0;
    return L;
}

int synth_row_lengths(int kind, const synth_params* p, int64_t row0, int64_t nrows, int64_t* len) {
    if (kind == SYN_POWERLAW) pl_table(p->gamma, p->kmax); /* build the table before threads start */
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < nrows; ++i) len[i] = row_len(kind, p, row0 + i);
    return 0;
}

static int cmp_i64(const void* a, const void* b) {
    int64_t x = *(const int64_t*)a, y = *(const int64_t*)b;
    return (x > y) - (x < y);
}

/* sort, then make strictly increasing inside [0, n) (needs L <= n) */
static void make_distinct(int64_t* c, int64_t L, int64_t n) {
    if (L <= 0) return;
    int sorted = 1;
    for (int64_t k = 1; k < L; ++k) if (c[k] <= c[k - 1]) { sorted = 0; break; }
    if (sorted && c[0] >= 0 && c[L - 1] < n) return;
    qsort(c, (size_t)L, sizeof(int64_t), cmp_i64);
    if (c[0] < 0) c[0] = 0;
    for (int64_t k = 1; k < L; ++k) if (c[k] <= c[k - 1]) c[k] = c[k - 1] + 1;
    if (c[L - 1] >= n) {
        c[L - 1] = n - 1;
        for (int64_t k = L - 2; k >= 0; --k) if (c[k] >= c[k + 1]) c[k] = c[k + 1] - 1;
    }
}

static double gen_val(int kind, const synth_params* p, int64_t row, int64_t k, int64_t L) {
    uint64_t r = rng3(p->seed, (uint64_t)row, K_VAL(k));
    switch (p->val_mode) {
    case VAL_INT: return (double)((int64_t)(r % 7ull) - 3);   /* {-3..3} */
    case VAL_ONES: return 1.0;
    default: {
        double v = 2.0 * u01(r) - 1.0;                        /* U(-1, 1) */
        if (kind == SYN_MIXED64 && L > 0) v /= (double)L;     /* sum_j |a_ij| <= 1 */
        return v;
    }
    }
}

static int64_t wrap(int64_t c, int64_t n) { c %= n; return c < 0 ? c + n : c; }

static void row_cols(int kind, const synth_params* p, int64_t row, int64_t L, int64_t* c) {
    uint64_t s = p->seed;
    int64_t n = p->n;
    switch (kind) {
    case SYN_STENCIL27: {
        int64_t nx = p->nx, ny = p->ny, nz = p->nz;
        int64_t x = row % nx, y = (row / nx) % ny, z = row / (nx * ny), q = 0;
        for (int dz = -1; dz <= 1; ++dz) for (int dy = -1; dy <= 1; ++dy) for (int dx = -1; dx <= 1; ++dx) {
            int64_t xx = x + dx, yy = y + dy, zz = z + dz;
            if (xx < 0 || xx >= nx || yy < 0 || yy >= ny || zz < 0 || zz >= nz) continue;
            c[q++] = xx + nx * (yy + ny * zz);
        }
        return; /* already ascending and distinct */
    }
    case SYN_LENLIST:
        if (p->local_frac <= 0.0) goto uniform;
        /* fall through: local + Zipf columns */
    case SYN_POWERLAW:
    case SYN_MIXED64: {
        double one_minus_s = 1.0 - p->zipf_s;
        double nz1 = pow((double)n, one_minus_s);
        for (int64_t k = 0; k < L; ++k) {
            uint64_t r = rng3(s, (uint64_t)row, K_COL(k));
            double u = u01(r), v = u01(mix64(r));
            if (u < p->local_frac) {
                int64_t off = (int64_t)floor((2.0 * v - 1.0) * (double)p->local_w + 0.5);
                c[k] = wrap(row + off, n);
            } else {   /* continuous Zipf(s) rank in [1, n], scattered by a bijection */
                double rk = pow(1.0 - v * (1.0 - nz1), 1.0 / one_minus_s);
                int64_t rank = (int64_t)rk - 1;
                if (rank < 0) rank = 0;
                if (rank >= n) rank = n - 1;
                c[k] = (int64_t)(((unsigned __int128)rank * 1000003ull + 7919ull) % (unsigned __int128)n);
            }
        }
        break;
    }
    default:
    uniform: /* uniform columns */
        for (int64_t k = 0; k < L; ++k) c[k] = (int64_t)(u01(rng3(s, (uint64_t)row, K_COL(k))) * (double)n);
    }
    make_distinct(c, L, n);
}

int synth_fill(int kind, const synth_params* p, int64_t row0, int64_t nrows, const int64_t* row_ptr,
               int32_t* col, double* val) {
    if (kind == SYN_POWERLAW) pl_table(p->gamma, p->kmax);
    int64_t maxL = 0;
    for (int64_t i = 0; i < nrows; ++i) { int64_t L = row_ptr[i + 1] - row_ptr[i]; if (L > maxL) maxL = L; }
    int err = 0;
#pragma omp parallel
    {
        int64_t* buf = (int64_t*)malloc(sizeof(int64_t) * (size_t)(maxL > 0 ? maxL : 1));
        if (!buf) {
#pragma omp atomic write
            err = 1;
        }
#pragma omp for schedule(dynamic, 256)
        for (int64_t i = 0; i < nrows; ++i) {
            if (!buf) continue;
            int64_t row = row0 + i, b = row_ptr[i], L = row_ptr[i + 1] - b;
            row_cols(kind, p, row, L, buf);
            for (int64_t k = 0; k < L; ++k) {
                col[b + k] = (int32_t)buf[k];
                /* VAL_SPD: -1 off the diagonal, L + 0.5 on it: symmetric patterns (stencils) give a
                   strictly diagonally dominant symmetric, hence SPD, matrix (solver consumer, f4) */
                if (p->val_mode == VAL_SPD) val[b + k] = buf[k] == row ? (double)L + 0.5 : -1.0;
                else val[b + k] = gen_val(kind, p, row, k, L);
            }
        }
        free(buf);
    }
    return err;
}

/* dense vector entries i0 .. i0+cnt-1 of a seeded vector (mode as val_mode) */
int synth_vector(uint64_t seed, int32_t mode, int64_t i0, int64_t cnt, double* out) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < cnt; ++i) {
        uint64_t r = rng3(seed ^ 0x5EEDF00Dull, (uint64_t)(i0 + i), 0x7777ull);
        if (mode == VAL_INT) out[i] = (double)((int64_t)(r % 7ull) - 3);
        else if (mode == VAL_ONES) out[i] = 1.0;
        else out[i] = 2.0 * u01(r) - 1.0;
    }
    return 0;
}
