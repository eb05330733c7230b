// builder.cpp — production host builder of the DASP format (§3.2), multithreaded.
//
// Steps: row scan + classification, long-row grouping
// with zero padding, stable descending medium sort + 8-row row-blocks + regular /
// irregular split with tau = 0.75, short-row piecing 1&3 / 4 / 2&2 / 1
// (P:L164), and the output map (R9).  The layout is DESIGN.md §4; oracle/oracle.c builds the
// same bytes independently (tests/test_builder.py compares them).
#include <omp.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "format.hpp"

namespace dasp {

void HostFormat::release() {
    for (auto& b : arr) {
        std::free(b.ptr);
        b.ptr = nullptr;
        b.bytes = 0;
    }
}

namespace {

enum Cls : uint8_t { C_EMPTY = 0, C_S1, C_S2, C_S3, C_S4, C_MED, C_LONG, C_NUM };

bool alloc(HostBuf& b, int64_t bytes) {
    b.bytes = bytes;
    b.ptr = std::malloc(static_cast<size_t>(bytes > 0 ? bytes : 1));
    return b.ptr != nullptr;
}

template <typename T>
T* as(HostBuf& b) { return static_cast<T*>(b.ptr); }

// parallel fill of (val = +0, col = PAD) over [0, count)
template <typename V>
void fill_pads(V* v, int32_t* c, int64_t count) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < count; ++i) { v[i] = V(0); c[i] = PAD_COL; }
}

// position of slot s (0 <= s < K*nreg) of row g of a row-block, inside the row-block's
// regular region: lane-interleaved chunks of CW blocks (R18).
inline int64_t reg_pos(const Geometry& geo, int64_t nreg, int g, int64_t s) {
    int64_t b = s / geo.K;
    int k = static_cast<int>(s % geo.K);
    int t, e;
    if (geo.EPL == 1) { t = k; e = 0; }                       // m8n8k4: A[g][t]
    else if (k < 8) { t = k >> 1; e = k & 1; }               // m16n8k16: a0,a1 = A[g][2t..2t+1]
    else { t = (k - 8) >> 1; e = 2 + (k & 1); }               //           a4,a5 = A[g][2t+8..2t+9]
    int lane = 4 * g + t;
    int64_t c = b / geo.CW, jb = b % geo.CW;
    int64_t w = std::min<int64_t>(geo.CW, nreg - c * geo.CW);
    return c * geo.CW * geo.BE + lane * w * geo.EPL + jb * geo.EPL + e;
}

// position of (4-slot row r in [0,32), inner slot c in [0,4)) inside a short tile
inline int short_pos(int sv, int r, int c) {
    if (sv == 8) return 4 * (4 * (r & 7) + c) + (r >> 3);      // lane (g=r&7, t=c), j = r>>3
    int q = r >> 3, g = r & 7;
    int t = ((q & 1) << 1) | (c >> 1);
    int j = ((q >> 1) << 1) | (c & 1);
    return 4 * (4 * g + t) + j;
}

template <typename V>
int build_impl(HostFormat& f, int64_t m, const int64_t* rp, const int32_t* col, const V* val) {
    const Geometry geo = f.geo;
    const int T = omp_get_max_threads();

    // ---- a1: lengths and classes (R1) ----
    std::vector<uint8_t> cls(static_cast<size_t>(m));
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; ++i) {
        int64_t L = rp[i + 1] - rp[i];
        cls[i] = L > MAX_LEN ? uint8_t{C_LONG} : (L > 4 ? uint8_t{C_MED} : static_cast<uint8_t>(L));
    }
    // stable parallel partition into per-class ascending row lists
    std::vector<int64_t> cnt(static_cast<size_t>(T) * C_NUM, 0);
    auto chunk = [&](int tid, int64_t& lo, int64_t& hi) {
        lo = m * tid / T;
        hi = m * (tid + 1) / T;
    };
#pragma omp parallel num_threads(T)
    {
        int tid = omp_get_thread_num();
        int64_t lo, hi;
        chunk(tid, lo, hi);
        int64_t* c = &cnt[static_cast<size_t>(tid) * C_NUM];
        for (int64_t i = lo; i < hi; ++i) c[cls[i]]++;
    }
    int64_t total[C_NUM] = {0};
    std::vector<int64_t> off(static_cast<size_t>(T) * C_NUM);
    for (int k = 0; k < C_NUM; ++k)
        for (int t = 0; t < T; ++t) {
            off[static_cast<size_t>(t) * C_NUM + k] = total[k];
            total[k] += cnt[static_cast<size_t>(t) * C_NUM + k];
        }
    std::vector<std::vector<int64_t>> rows(C_NUM);
    for (int k = 0; k < C_NUM; ++k) rows[k].resize(static_cast<size_t>(total[k]));
#pragma omp parallel num_threads(T)
    {
        int tid = omp_get_thread_num();
        int64_t lo, hi;
        chunk(tid, lo, hi);
        int64_t o[C_NUM];
        for (int k = 0; k < C_NUM; ++k) o[k] = off[static_cast<size_t>(tid) * C_NUM + k];
        for (int64_t i = lo; i < hi; ++i) rows[cls[i]][o[cls[i]]++] = i;
    }
    f.n0 = total[C_EMPTY]; f.n1 = total[C_S1]; f.n2 = total[C_S2]; f.n3 = total[C_S3]; f.n4 = total[C_S4];
    f.row_medium = total[C_MED];
    f.row_long = total[C_LONG];

    if (!alloc(f.arr[DASP_ARR_EMPTY_ROWS], f.n0 * 4)) return DASP_ERR_OUT_OF_MEMORY;
    {
        int32_t* e = as<int32_t>(f.arr[DASP_ARR_EMPTY_ROWS]);
        const auto& r0 = rows[C_EMPTY];
#pragma omp parallel for schedule(static)
        for (int64_t k = 0; k < f.n0; ++k) e[k] = static_cast<int32_t>(r0[k]);
    }

    // ---- a2: long rows, groups of G, zero padded ----
    {
        const auto& LR = rows[C_LONG];
        const int64_t nl = f.row_long;
        if (!alloc(f.arr[DASP_ARR_GROUP_PTR], (nl + 1) * 8) || !alloc(f.arr[DASP_ARR_LONG_OUT], nl * 4))
            return DASP_ERR_OUT_OF_MEMORY;
        int64_t* gp = as<int64_t>(f.arr[DASP_ARR_GROUP_PTR]);
        int32_t* lo = as<int32_t>(f.arr[DASP_ARR_LONG_OUT]);
        gp[0] = 0;
        int64_t nnz_long = 0;
        for (int64_t r = 0; r < nl; ++r) {
            int64_t L = rp[LR[r] + 1] - rp[LR[r]];
            nnz_long += L;
            gp[r + 1] = gp[r] + (L + geo.G - 1) / geo.G;
            lo[r] = static_cast<int32_t>(LR[r]);
        }
        f.nnz_long = nnz_long;
        f.n_groups = gp[nl];
        f.n_groups_padded = (f.n_groups + geo.UG - 1) / geo.UG * geo.UG;
        f.nnz_long_new = f.n_groups * geo.G;
        const int64_t ne = f.n_groups_padded * geo.G;
        if (!alloc(f.arr[DASP_ARR_LONG_VAL], ne * geo.sv) || !alloc(f.arr[DASP_ARR_LONG_COL], ne * 4))
            return DASP_ERR_OUT_OF_MEMORY;
        V* lv = as<V>(f.arr[DASP_ARR_LONG_VAL]);
        int32_t* lc = as<int32_t>(f.arr[DASP_ARR_LONG_COL]);
#pragma omp parallel for schedule(dynamic, 16)
        for (int64_t r = 0; r < nl; ++r) {
            const int64_t i = LR[r], b = rp[i], L = rp[i + 1] - b, at = gp[r] * geo.G;
            std::memcpy(lv + at, val + b, static_cast<size_t>(L) * sizeof(V));
            std::memcpy(lc + at, col + b, static_cast<size_t>(L) * 4);
            const int64_t end = gp[r + 1] * geo.G;
            for (int64_t k = at + L; k < end; ++k) { lv[k] = V(0); lc[k] = PAD_COL; }
        }
        fill_pads(lv + f.nnz_long_new, lc + f.nnz_long_new, ne - f.nnz_long_new);
    }

    // ---- a3: medium rows ----
    {
        const auto& MR = rows[C_MED];
        const int64_t nm = f.row_medium;
        // stable descending sort by length: counting sort on key MAX_LEN - len (R26)
        constexpr int NB = MAX_LEN + 1;
        std::vector<int64_t> h(static_cast<size_t>(T) * NB, 0);
#pragma omp parallel num_threads(T)
        {
            int tid = omp_get_thread_num();
            int64_t lo = nm * tid / T, hi = nm * (tid + 1) / T;
            int64_t* hh = &h[static_cast<size_t>(tid) * NB];
            for (int64_t k = lo; k < hi; ++k) hh[MAX_LEN - (rp[MR[k] + 1] - rp[MR[k]])]++;
        }
        std::vector<int64_t> ho(static_cast<size_t>(T) * NB);
        int64_t run = 0;
        for (int key = 0; key < NB; ++key)
            for (int t = 0; t < T; ++t) {
                ho[static_cast<size_t>(t) * NB + key] = run;
                run += h[static_cast<size_t>(t) * NB + key];
            }
        f.nrb = (nm + MMA_M - 1) / MMA_M;  // R7
        const int64_t nmp = f.nrb * MMA_M;
        std::vector<int64_t> sorted(static_cast<size_t>(nmp), -1);
#pragma omp parallel num_threads(T)
        {
            int tid = omp_get_thread_num();
            int64_t lo = nm * tid / T, hi = nm * (tid + 1) / T;
            int64_t* o = &ho[static_cast<size_t>(tid) * NB];
            for (int64_t k = lo; k < hi; ++k) sorted[o[MAX_LEN - (rp[MR[k] + 1] - rp[MR[k]])]++] = MR[k];
        }
        if (!alloc(f.arr[DASP_ARR_MED_OUT], nmp * 4) || !alloc(f.arr[DASP_ARR_RB_PTR], (f.nrb + 1) * 8) ||
            !alloc(f.arr[DASP_ARR_IRR_PTR], (nmp + 1) * 8))
            return DASP_ERR_OUT_OF_MEMORY;
        int32_t* mo = as<int32_t>(f.arr[DASP_ARR_MED_OUT]);
        int64_t* rbp = as<int64_t>(f.arr[DASP_ARR_RB_PTR]);
        int64_t* ip = as<int64_t>(f.arr[DASP_ARR_IRR_PTR]);
        auto slen = [&](int64_t i) -> int64_t { return sorted[i] < 0 ? 0 : rp[sorted[i] + 1] - rp[sorted[i]]; };
        std::vector<int64_t> nreg(static_cast<size_t>(f.nrb));
        int64_t nnz_med = 0;
#pragma omp parallel for schedule(static) reduction(+ : nnz_med)
        for (int64_t rb = 0; rb < f.nrb; ++rb) {
            int64_t L[MMA_M];
            for (int g = 0; g < MMA_M; ++g) {
                L[g] = slen(rb * MMA_M + g);
                nnz_med += L[g];
                mo[rb * MMA_M + g] = sorted[rb * MMA_M + g] < 0 ? -1 : static_cast<int32_t>(sorted[rb * MMA_M + g]);
            }
            // regular iff the 8 x K block holds more than tau * 8K real slots, tau = 0.75,
            // strict (R4); prefix of blocks (R6)
            int64_t b = 0;
            for (;;) {
                int64_t c = 0;
                for (int g = 0; g < MMA_M; ++g) c += std::clamp<int64_t>(L[g] - geo.K * b, 0, geo.K);
                if (4 * c > 3 * static_cast<int64_t>(geo.BE)) ++b; else break;
            }
            nreg[rb] = b;
        }
        f.nnz_medium = nnz_med;
        rbp[0] = 0;
        for (int64_t rb = 0; rb < f.nrb; ++rb) rbp[rb + 1] = rbp[rb] + nreg[rb] * geo.BE;
        ip[0] = 0;
        for (int64_t i = 0; i < nmp; ++i) ip[i + 1] = ip[i] + std::max<int64_t>(0, slen(i) - geo.K * nreg[i / MMA_M]);
        f.nnz_reg_new = rbp[f.nrb];
        f.nnz_irreg = ip[nmp];
        if (!alloc(f.arr[DASP_ARR_REG_VAL], f.nnz_reg_new * geo.sv) || !alloc(f.arr[DASP_ARR_REG_COL], f.nnz_reg_new * 4) ||
            !alloc(f.arr[DASP_ARR_IRR_VAL], f.nnz_irreg * geo.sv) || !alloc(f.arr[DASP_ARR_IRR_COL], f.nnz_irreg * 4))
            return DASP_ERR_OUT_OF_MEMORY;
        V* rv = as<V>(f.arr[DASP_ARR_REG_VAL]);
        int32_t* rc = as<int32_t>(f.arr[DASP_ARR_REG_COL]);
        V* iv = as<V>(f.arr[DASP_ARR_IRR_VAL]);
        int32_t* ic = as<int32_t>(f.arr[DASP_ARR_IRR_COL]);
#pragma omp parallel for schedule(dynamic, 64)
        for (int64_t rb = 0; rb < f.nrb; ++rb) {
            const int64_t nr = nreg[rb], base = rbp[rb], nslot = geo.K * nr;
            for (int g = 0; g < MMA_M; ++g) {
                const int64_t i = rb * MMA_M + g, L = slen(i);
                const int64_t src = sorted[i] < 0 ? 0 : rp[sorted[i]];
                for (int64_t s = 0; s < nslot; ++s) {
                    const int64_t at = base + reg_pos(geo, nr, g, s);
                    if (s < L) { rv[at] = val[src + s]; rc[at] = col[src + s]; }
                    else { rv[at] = V(0); rc[at] = PAD_COL; }
                }
                for (int64_t s = nslot; s < L; ++s) {
                    iv[ip[i] + s - nslot] = val[src + s];
                    ic[ip[i] + s - nslot] = col[src + s];
                }
            }
        }
    }

    // ---- a4: short rows, piecing (R13) ----
    {
        const auto &S1 = rows[C_S1], &S2 = rows[C_S2], &S3 = rows[C_S3], &S4 = rows[C_S4];
        const int64_t p13 = std::min(f.n1, f.n3), p22 = f.n2 / 2;
        const int64_t n3l = f.n3 - p13, n2l = f.n2 % 2, n4cat = f.n4 + n3l + n2l, ns = f.n1 - p13;
        f.t13 = (p13 + 31) / 32; f.t4 = (n4cat + 31) / 32; f.t22 = (p22 + 31) / 32; f.ts = (ns + SHORT_TILE - 1) / SHORT_TILE;
        f.nnz_short = f.n1 + 2 * f.n2 + 3 * f.n3 + 4 * f.n4;
        const int64_t ntiles = f.t13 + f.t4 + f.t22 + f.ts;
        f.nnz_short_new = ntiles * SHORT_TILE;
        const int64_t nout = 64 * f.t13 + 32 * f.t4 + 64 * f.t22 + SHORT_TILE * f.ts;
        if (!alloc(f.arr[DASP_ARR_SHORT_VAL], f.nnz_short_new * geo.sv) || !alloc(f.arr[DASP_ARR_SHORT_COL], f.nnz_short_new * 4) ||
            !alloc(f.arr[DASP_ARR_SHORT_OUT], nout * 4))
            return DASP_ERR_OUT_OF_MEMORY;
        V* sv = as<V>(f.arr[DASP_ARR_SHORT_VAL]);
        int32_t* sc = as<int32_t>(f.arr[DASP_ARR_SHORT_COL]);
        int32_t* so = as<int32_t>(f.arr[DASP_ARR_SHORT_OUT]);
        fill_pads(sv, sc, f.nnz_short_new);
#pragma omp parallel for schedule(static)
        for (int64_t o = 0; o < nout; ++o) so[o] = -1;

        auto put_row4 = [&](int64_t tile, int r, int64_t ra, int la, int64_t rb_, int lb) {
            V* tv = sv + tile * SHORT_TILE;
            int32_t* tc = sc + tile * SHORT_TILE;
            for (int k = 0; k < la; ++k) { int p = short_pos(geo.sv, r, k); tv[p] = val[rp[ra] + k]; tc[p] = col[rp[ra] + k]; }
            if (rb_ >= 0)
                for (int k = 0; k < lb; ++k) { int p = short_pos(geo.sv, r, la + k); tv[p] = val[rp[rb_] + k]; tc[p] = col[rp[rb_] + k]; }
        };
        // 1&3: slot 0 = len-1 row, slots 1-3 = len-3 row (Alg. 4 masks)
        const int64_t o13 = 0, tile13 = 0;
#pragma omp parallel for schedule(static)
        for (int64_t q = 0; q < p13; ++q) {
            int64_t tile = tile13 + q / 32;
            int r = static_cast<int>(q % 32);
            put_row4(tile, r, S1[q], 1, S3[q], 3);
            int64_t o = o13 + (q / 32) * 64 + 16 * (r >> 3) + (r & 7);
            so[o] = static_cast<int32_t>(S1[q]);
            so[o + 8] = static_cast<int32_t>(S3[q]);
        }
        // len-4 category: true len-4 rows, then leftover len-3 rows, then the odd len-2 row
        const int64_t tile4 = f.t13, o4 = 64 * f.t13;
#pragma omp parallel for schedule(static)
        for (int64_t q = 0; q < n4cat; ++q) {
            int64_t row;
            int len;
            if (q < f.n4) { row = S4[q]; len = 4; }
            else if (q < f.n4 + n3l) { row = S3[p13 + q - f.n4]; len = 3; }
            else { row = S2[f.n2 - 1]; len = 2; }
            put_row4(tile4 + q / 32, static_cast<int>(q % 32), row, len, -1, 0);
            so[o4 + q] = static_cast<int32_t>(row);   // tile q/32, o = r: 32*(q/32) + q%32 = q
        }
        // 2&2: slots 0-1 = S2[2q], slots 2-3 = S2[2q+1]
        const int64_t tile22 = f.t13 + f.t4, o22 = 64 * f.t13 + 32 * f.t4;
#pragma omp parallel for schedule(static)
        for (int64_t q = 0; q < p22; ++q) {
            int r = static_cast<int>(q % 32);
            put_row4(tile22 + q / 32, r, S2[2 * q], 2, S2[2 * q + 1], 2);
            int64_t o = o22 + (q / 32) * 64 + 16 * (r >> 3) + (r & 7);
            so[o] = static_cast<int32_t>(S2[2 * q]);
            so[o + 8] = static_cast<int32_t>(S2[2 * q + 1]);
        }
        // singles: leftover len-1 rows (Alg. 5)
        const int64_t tiles = f.t13 + f.t4 + f.t22, os = 64 * f.t13 + 32 * f.t4 + 64 * f.t22;
#pragma omp parallel for schedule(static)
        for (int64_t q = 0; q < ns; ++q) {
            const int64_t i = S1[p13 + q];
            sv[tiles * SHORT_TILE + q] = val[rp[i]];
            sc[tiles * SHORT_TILE + q] = col[rp[i]];
            so[os + q] = static_cast<int32_t>(i);
        }
    }
    return DASP_OK;
}

}  // namespace

int build_format(HostFormat& f, int dtype, int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col,
                 const void* val, int nthreads, bool validate) {
    f = HostFormat{};
    f.geo = geometry(dtype);
    f.dtype = dtype;
    f.m = m;
    f.n = n;
    f.nnz = m > 0 ? row_ptr[m] : 0;
    if (nthreads > 0) omp_set_num_threads(nthreads);
    if (validate) {
        if (row_ptr[0] != 0) return DASP_ERR_INVALID_CSR;
        int bad = 0;
#pragma omp parallel for schedule(static) reduction(| : bad)
        for (int64_t i = 0; i < m; ++i)
            if (row_ptr[i + 1] < row_ptr[i]) bad |= 1;
        if (bad) return DASP_ERR_INVALID_CSR;
        const int64_t nnz = f.nnz;
#pragma omp parallel for schedule(static) reduction(| : bad)
        for (int64_t k = 0; k < nnz; ++k)
            if (col[k] < 0 || col[k] >= n) bad |= 1;
        if (bad) return DASP_ERR_INVALID_CSR;
    }
    int st;
    if (dtype == DASP_R_64F) st = build_impl<uint64_t>(f, m, row_ptr, col, static_cast<const uint64_t*>(val));
    else st = build_impl<uint16_t>(f, m, row_ptr, col, static_cast<const uint16_t*>(val));
    if (st != DASP_OK) f.release();
    return st;
}

}  // namespace dasp
