// builder.cpp — production host builder of the DASP format (§3.2), multithreaded.
//
// Steps: row scan + classification, long-row grouping
// with zero padding, stable descending medium sort + 8-row row-blocks + regular /
// irregular split with tau = 0.75, short-row piecing 1&3 / 4 / 2&2 / 1
// (P:L164), and the output map (R9).  Rows are cut into panels (R28); every panel is
// classified, sorted and pieced on its own, and the panels' arrays are concatenated.
//
// Two passes: pass 1 computes each panel's class lists, medium order and counts; pass 2
// writes every panel straight into the final arrays at its offsets.  The layout is
// DESIGN.md §4; oracle/oracle.c builds the same bytes independently (tests/test_builder.py).
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

// position of slot s (0 <= s < K*nreg) of row g of a row-block, inside the row-block's
// regular region: lane-interleaved chunks of CW blocks, the ragged last chunk block by block (R18).
inline int64_t reg_pos(const Geometry& geo, int64_t nreg, int g, int64_t s) {
    int64_t b = s / geo.K;
    int k = static_cast<int>(s % geo.K);
    int t, e;
    if (geo.EPL == 1) { t = k; e = 0; }                       // m8n8k4 f64: A[g][t]
    else { t = k >> 1; e = k & 1; }                           // m16n8k8 f16: a0,a1 = A[g][2t..2t+1]
    int lane = 4 * g + t;
    int64_t c = b / geo.CW, jb = b % geo.CW;
    int64_t w = std::min<int64_t>(geo.CW, nreg - c * geo.CW);
    if (w == geo.CW) return c * geo.CW * geo.BE + lane * w * geo.EPL + jb * geo.EPL + e;   // full chunk
    return c * geo.CW * geo.BE + jb * geo.BE + lane * geo.EPL + e;                          // ragged tail
}

// position of (4-slot row r in [0,32), inner slot c in [0,4)) inside a short tile
inline int short_pos(int K, int r, int c) {
    if (K == 4) return 4 * (4 * (r & 7) + c) + (r >> 3);       // m8n8k4: lane (g=r&7, t=c), j = r>>3
    int q = r >> 3, g = r & 7;
    int t = ((q & 1) << 1) | (c >> 1);
    int j = ((q >> 1) << 1) | (c & 1);
    return 4 * (4 * g + t) + j;
}

// Pass-1 result for one panel (rows [r0, r1)).
struct Panel {
    int64_t r0 = 0, r1 = 0;
    std::vector<int64_t> rows[C_NUM];   // class lists, ascending original order (global row ids)
    std::vector<int64_t> sorted;        // medium rows, stable by length desc, padded to 8 with -1
    std::vector<int64_t> nreg;          // regular blocks per row-block
    int64_t nrb = 0, n_groups = 0, nnz_long = 0, nnz_med = 0, sq_med = 0, reg = 0, irr = 0;
    int64_t p13 = 0, p22 = 0, n3l = 0, n2l = 0, n4cat = 0, ns = 0, t13 = 0, t4 = 0, t22 = 0, ts = 0;
    // offsets into the concatenated arrays (set between the passes)
    int64_t o_long_row = 0, o_group = 0, o_rb = 0, o_reg = 0, o_irr = 0, o_tile = 0, o_out = 0, o_empty = 0;
    int64_t nout() const { return 64 * t13 + 32 * t4 + 64 * t22 + SHORT_TILE * ts; }
};

inline int class_of(int64_t L, int64_t max_len) { return L > max_len ? C_LONG : (L > 4 ? C_MED : static_cast<int>(L)); }

// ---- pass 1: classification, medium order, counts ----
void plan_panel(Panel& P, const Geometry& geo, const int64_t* rp, bool par, int64_t max_len, double tau) {
    const int64_t n = P.r1 - P.r0;
    // a1: classes (R1: empty rows are their own class), lists in ascending row order
    if (!par) {
        for (int64_t i = P.r0; i < P.r1; ++i) P.rows[class_of(rp[i + 1] - rp[i], max_len)].push_back(i);
    } else {  // stable parallel partition
        const int T = omp_get_max_threads();
        std::vector<int64_t> cnt(static_cast<size_t>(T) * C_NUM, 0), off(static_cast<size_t>(T) * C_NUM);
#pragma omp parallel num_threads(T)
        {
            const int tid = omp_get_thread_num();
            const int64_t lo = P.r0 + n * tid / T, hi = P.r0 + n * (tid + 1) / T;
            for (int64_t i = lo; i < hi; ++i) cnt[static_cast<size_t>(tid) * C_NUM + class_of(rp[i + 1] - rp[i], max_len)]++;
        }
        int64_t total[C_NUM] = {0};
        for (int k = 0; k < C_NUM; ++k)
            for (int t = 0; t < T; ++t) {
                off[static_cast<size_t>(t) * C_NUM + k] = total[k];
                total[k] += cnt[static_cast<size_t>(t) * C_NUM + k];
            }
        for (int k = 0; k < C_NUM; ++k) P.rows[k].resize(static_cast<size_t>(total[k]));
#pragma omp parallel num_threads(T)
        {
            const int tid = omp_get_thread_num();
            const int64_t lo = P.r0 + n * tid / T, hi = P.r0 + n * (tid + 1) / T;
            int64_t o[C_NUM];
            for (int k = 0; k < C_NUM; ++k) o[k] = off[static_cast<size_t>(tid) * C_NUM + k];
            for (int64_t i = lo; i < hi; ++i) { const int c = class_of(rp[i + 1] - rp[i], max_len); P.rows[c][o[c]++] = i; }
        }
    }
    // a2: long groups
    for (int64_t r : P.rows[C_LONG]) {
        const int64_t L = rp[r + 1] - rp[r];
        P.nnz_long += L;
        P.n_groups += (L + geo.G - 1) / geo.G;
    }
    // a3: stable descending sort by length (R26): counting sort on max_len - len
    const auto& MR = P.rows[C_MED];
    const int64_t nm = static_cast<int64_t>(MR.size());
    P.nrb = (nm + MMA_M - 1) / MMA_M;  // R7
    P.sorted.assign(static_cast<size_t>(P.nrb * MMA_M), -1);
    {
        const int64_t NB = max_len + 1;
        std::vector<int64_t> h(static_cast<size_t>(NB + 1), 0);
        for (int64_t r : MR) h[max_len - (rp[r + 1] - rp[r]) + 1]++;
        for (int64_t b = 0; b < NB; ++b) h[b + 1] += h[b];
        for (int64_t r : MR) P.sorted[h[max_len - (rp[r + 1] - rp[r])]++] = r;
    }
    P.nreg.assign(static_cast<size_t>(P.nrb), 0);
    int64_t reg = 0, irr = 0, nnz_med = 0, sq_med = 0;
#pragma omp parallel for schedule(static) reduction(+ : reg, irr, nnz_med, sq_med) if (par)
    for (int64_t rb = 0; rb < P.nrb; ++rb) {
        int64_t L[MMA_M];
        for (int g = 0; g < MMA_M; ++g) {
            const int64_t r = P.sorted[rb * MMA_M + g];
            L[g] = r < 0 ? 0 : rp[r + 1] - rp[r];
            nnz_med += L[g];
            sq_med += L[g] * L[g];
        }
        // regular iff the 8 x K block holds more than tau * 8K real slots (default tau = 0.75,
        // strict R4); the regular blocks form a prefix (R6)
        const double thr = static_cast<double>(geo.BE) * tau;
        int64_t b = 0;
        for (;;) {
            int64_t c = 0;
            for (int g = 0; g < MMA_M; ++g) c += std::clamp<int64_t>(L[g] - geo.K * b, 0, geo.K);
            if (static_cast<double>(c) > thr) ++b; else break;
        }
        P.nreg[rb] = b;
        reg += b * geo.BE;
        for (int g = 0; g < MMA_M; ++g) irr += std::max<int64_t>(0, L[g] - geo.K * b);
    }
    P.reg = reg; P.irr = irr; P.nnz_med = nnz_med; P.sq_med = sq_med;
    // a4: short piecing counts (R13)
    const int64_t n1 = P.rows[C_S1].size(), n2 = P.rows[C_S2].size(), n3 = P.rows[C_S3].size(), n4 = P.rows[C_S4].size();
    P.p13 = std::min(n1, n3); P.p22 = n2 / 2; P.n3l = n3 - P.p13; P.n2l = n2 % 2;
    P.n4cat = n4 + P.n3l + P.n2l; P.ns = n1 - P.p13;
    P.t13 = (P.p13 + 31) / 32; P.t4 = (P.n4cat + 31) / 32; P.t22 = (P.p22 + 31) / 32;
    P.ts = (P.ns + SHORT_TILE - 1) / SHORT_TILE;
}

// ---- pass 2: write one panel into the final arrays ----
template <typename V>
void fill_panel(HostFormat& f, const Panel& P, const int64_t* rp, const int32_t* col, const V* val, bool par) {
    const Geometry geo = f.geo;
    // empty rows
    int32_t* er = as<int32_t>(f.arr[DASP_ARR_EMPTY_ROWS]) + P.o_empty;
    for (size_t k = 0; k < P.rows[C_EMPTY].size(); ++k) er[k] = static_cast<int32_t>(P.rows[C_EMPTY][k]);

    // long rows: CSR order, pads appended to a multiple of G
    {
        const auto& LR = P.rows[C_LONG];
        const int64_t nl = static_cast<int64_t>(LR.size());
        int64_t* gp = as<int64_t>(f.arr[DASP_ARR_GROUP_PTR]) + P.o_long_row;
        int32_t* lo = as<int32_t>(f.arr[DASP_ARR_LONG_OUT]) + P.o_long_row;
        int64_t g = P.o_group;
        for (int64_t r = 0; r < nl; ++r) {
            gp[r] = g;
            g += (rp[LR[r] + 1] - rp[LR[r]] + geo.G - 1) / geo.G;
            lo[r] = static_cast<int32_t>(LR[r]);
        }
        gp[nl] = g;   // == the next panel's first entry
        V* lv = as<V>(f.arr[DASP_ARR_LONG_VAL]);
        int32_t* lc = as<int32_t>(f.arr[DASP_ARR_LONG_COL]);
#pragma omp parallel for schedule(dynamic, 16) if (par)
        for (int64_t r = 0; r < nl; ++r) {
            const int64_t i = LR[r], b = rp[i], L = rp[i + 1] - b, at = gp[r] * geo.G;
            std::memcpy(lv + at, val + b, static_cast<size_t>(L) * sizeof(V));
            std::memcpy(lc + at, col + b, static_cast<size_t>(L) * 4);
            const int64_t end = gp[r + 1] * geo.G;
            for (int64_t k = at + L; k < end; ++k) { lv[k] = V(0); lc[k] = PAD_COL; }
        }
    }

    // medium rows: regular chunks (R18) + irregular tails
    {
        int32_t* mo = as<int32_t>(f.arr[DASP_ARR_MED_OUT]) + P.o_rb * MMA_M;
        int64_t* rbp = as<int64_t>(f.arr[DASP_ARR_RB_PTR]) + P.o_rb;
        int64_t* ip = as<int64_t>(f.arr[DASP_ARR_IRR_PTR]) + P.o_rb * MMA_M;
        const int64_t nmp = P.nrb * MMA_M;
        auto slen = [&](int64_t i) -> int64_t { const int64_t r = P.sorted[i]; return r < 0 ? 0 : rp[r + 1] - rp[r]; };
        int64_t acc = P.o_reg;
        for (int64_t rb = 0; rb < P.nrb; ++rb) { rbp[rb] = acc; acc += P.nreg[rb] * geo.BE; }
        rbp[P.nrb] = acc;
        acc = P.o_irr;
        for (int64_t i = 0; i < nmp; ++i) { ip[i] = acc; acc += std::max<int64_t>(0, slen(i) - geo.K * P.nreg[i / MMA_M]); }
        ip[nmp] = acc;
        V* rv = as<V>(f.arr[DASP_ARR_REG_VAL]);
        int32_t* rc = as<int32_t>(f.arr[DASP_ARR_REG_COL]);
        V* iv = as<V>(f.arr[DASP_ARR_IRR_VAL]);
        int32_t* ic = as<int32_t>(f.arr[DASP_ARR_IRR_COL]);
#pragma omp parallel for schedule(dynamic, 64) if (par)
        for (int64_t rb = 0; rb < P.nrb; ++rb) {
            const int64_t nr = P.nreg[rb], base = rbp[rb], nslot = geo.K * nr;
            for (int g = 0; g < MMA_M; ++g) {
                const int64_t i = rb * MMA_M + g, L = slen(i), row = P.sorted[i];
                mo[i] = row < 0 ? -1 : static_cast<int32_t>(row);
                const int64_t src = row < 0 ? 0 : rp[row];
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

    // short rows: [1&3][len4][2&2][singles] tiles of this panel
    {
        const auto &S1 = P.rows[C_S1], &S2 = P.rows[C_S2], &S3 = P.rows[C_S3], &S4 = P.rows[C_S4];
        V* sv = as<V>(f.arr[DASP_ARR_SHORT_VAL]) + P.o_tile * SHORT_TILE;
        int32_t* sc = as<int32_t>(f.arr[DASP_ARR_SHORT_COL]) + P.o_tile * SHORT_TILE;
        int32_t* so = as<int32_t>(f.arr[DASP_ARR_SHORT_OUT]) + P.o_out;
        const int64_t ntiles = P.t13 + P.t4 + P.t22 + P.ts, nout = P.nout();
#pragma omp parallel for schedule(static) if (par)
        for (int64_t e = 0; e < ntiles * SHORT_TILE; ++e) { sv[e] = V(0); sc[e] = PAD_COL; }
#pragma omp parallel for schedule(static) if (par)
        for (int64_t o = 0; o < nout; ++o) so[o] = -1;
        auto put_row4 = [&](int64_t tile, int r, int64_t ra, int la, int64_t rb_, int lb) {
            V* tv = sv + tile * SHORT_TILE;
            int32_t* tc = sc + tile * SHORT_TILE;
            for (int k = 0; k < la; ++k) { const int p = short_pos(geo.K, r, k); tv[p] = val[rp[ra] + k]; tc[p] = col[rp[ra] + k]; }
            if (rb_ >= 0)
                for (int k = 0; k < lb; ++k) { const int p = short_pos(geo.K, r, la + k); tv[p] = val[rp[rb_] + k]; tc[p] = col[rp[rb_] + k]; }
        };
        // 1&3: slot 0 = len-1 row, slots 1-3 = len-3 row (Alg. 4 masks)
#pragma omp parallel for schedule(static) if (par)
        for (int64_t q = 0; q < P.p13; ++q) {
            const int r = static_cast<int>(q % 32);
            put_row4(q / 32, r, S1[q], 1, S3[q], 3);
            const int64_t o = (q / 32) * 64 + 16 * (r >> 3) + (r & 7);
            so[o] = static_cast<int32_t>(S1[q]);
            so[o + 8] = static_cast<int32_t>(S3[q]);
        }
        // len-4 category: true len-4 rows, then leftover len-3 rows, then the odd len-2 row (R13)
        const int64_t n4 = static_cast<int64_t>(S4.size());
#pragma omp parallel for schedule(static) if (par)
        for (int64_t q = 0; q < P.n4cat; ++q) {
            int64_t row;
            int len;
            if (q < n4) { row = S4[q]; len = 4; }
            else if (q < n4 + P.n3l) { row = S3[P.p13 + q - n4]; len = 3; }
            else { row = S2.back(); len = 2; }
            put_row4(P.t13 + q / 32, static_cast<int>(q % 32), row, len, -1, 0);
            so[64 * P.t13 + q] = static_cast<int32_t>(row);
        }
        // 2&2: slots 0-1 = S2[2q], slots 2-3 = S2[2q+1]
#pragma omp parallel for schedule(static) if (par)
        for (int64_t q = 0; q < P.p22; ++q) {
            const int r = static_cast<int>(q % 32);
            put_row4(P.t13 + P.t4 + q / 32, r, S2[2 * q], 2, S2[2 * q + 1], 2);
            const int64_t o = 64 * P.t13 + 32 * P.t4 + (q / 32) * 64 + 16 * (r >> 3) + (r & 7);
            so[o] = static_cast<int32_t>(S2[2 * q]);
            so[o + 8] = static_cast<int32_t>(S2[2 * q + 1]);
        }
        // singles: leftover len-1 rows (Alg. 5)
        const int64_t t0 = (P.t13 + P.t4 + P.t22) * SHORT_TILE, os = 64 * P.t13 + 32 * P.t4 + 64 * P.t22;
#pragma omp parallel for schedule(static) if (par)
        for (int64_t q = 0; q < P.ns; ++q) {
            const int64_t i = S1[P.p13 + q];
            sv[t0 + q] = val[rp[i]];
            sc[t0 + q] = col[rp[i]];
            so[os + q] = static_cast<int32_t>(i);
        }
    }
}

template <typename V>
int build_impl(HostFormat& f, int64_t m, const int64_t* rp, const int32_t* col, const V* val) {
    const Geometry geo = f.geo;
    const int T = omp_get_max_threads();
    const int64_t R = f.panel_rows;
    const int64_t np = m > 0 ? (m + R - 1) / R : 1;
    std::vector<Panel> panels(static_cast<size_t>(np));
    for (int64_t q = 0; q < np; ++q) {
        panels[q].r0 = std::min(m, q * R);
        panels[q].r1 = std::min(m, (q + 1) * R);
    }
    // many panels: one thread per panel; few panels: threads inside each panel
    const bool outer = np >= 2 * T;
#pragma omp parallel for schedule(dynamic, 1) if (outer)
    for (int64_t q = 0; q < np; ++q) plan_panel(panels[q], geo, rp, !outer, f.max_len, f.tau);

    // offsets of every panel in the concatenated arrays
    int64_t lr = 0, grp = 0, rb = 0, reg = 0, irr = 0, tile = 0, out = 0, emp = 0;
    for (auto& P : panels) {
        P.o_long_row = lr; P.o_group = grp; P.o_rb = rb; P.o_reg = reg; P.o_irr = irr;
        P.o_tile = tile; P.o_out = out; P.o_empty = emp;
        lr += P.rows[C_LONG].size(); grp += P.n_groups; rb += P.nrb; reg += P.reg; irr += P.irr;
        tile += P.t13 + P.t4 + P.t22 + P.ts; out += P.nout(); emp += P.rows[C_EMPTY].size();
        f.n1 += P.rows[C_S1].size(); f.n2 += P.rows[C_S2].size();
        f.n3 += P.rows[C_S3].size(); f.n4 += P.rows[C_S4].size();
        f.row_medium += P.rows[C_MED].size();
        f.t13 += P.t13; f.t4 += P.t4; f.t22 += P.t22; f.ts += P.ts;
        f.nnz_long += P.nnz_long; f.nnz_medium += P.nnz_med; f.sumsq_medium += P.sq_med;
    }
    f.n0 = emp;
    f.row_long = lr;
    f.n_panels = np;
    f.nrb = rb;
    f.n_groups = grp;
    f.n_groups_padded = (grp + geo.UG - 1) / geo.UG * geo.UG;   // one pad at the very end
    f.nnz_long_new = grp * geo.G;
    f.nnz_reg_new = reg;
    f.nnz_irreg = irr;
    f.nnz_short_new = tile * SHORT_TILE;
    f.nnz_short = f.n1 + 2 * f.n2 + 3 * f.n3 + 4 * f.n4;
    const int64_t ne = f.n_groups_padded * geo.G;
    if (!alloc(f.arr[DASP_ARR_EMPTY_ROWS], f.n0 * 4) || !alloc(f.arr[DASP_ARR_GROUP_PTR], (f.row_long + 1) * 8) ||
        !alloc(f.arr[DASP_ARR_LONG_OUT], f.row_long * 4) || !alloc(f.arr[DASP_ARR_LONG_VAL], ne * geo.sv) ||
        !alloc(f.arr[DASP_ARR_LONG_COL], ne * 4) || !alloc(f.arr[DASP_ARR_MED_OUT], rb * MMA_M * 4) ||
        !alloc(f.arr[DASP_ARR_RB_PTR], (rb + 1) * 8) || !alloc(f.arr[DASP_ARR_IRR_PTR], (rb * MMA_M + 1) * 8) ||
        !alloc(f.arr[DASP_ARR_REG_VAL], reg * geo.sv) || !alloc(f.arr[DASP_ARR_REG_COL], reg * 4) ||
        !alloc(f.arr[DASP_ARR_IRR_VAL], irr * geo.sv) || !alloc(f.arr[DASP_ARR_IRR_COL], irr * 4) ||
        !alloc(f.arr[DASP_ARR_SHORT_VAL], tile * SHORT_TILE * geo.sv) ||
        !alloc(f.arr[DASP_ARR_SHORT_COL], tile * SHORT_TILE * 4) || !alloc(f.arr[DASP_ARR_SHORT_OUT], out * 4) ||
        !alloc(f.arr[DASP_ARR_PANELS], np * PANEL_FIELDS * 8))
        return DASP_ERR_OUT_OF_MEMORY;
    as<int64_t>(f.arr[DASP_ARR_GROUP_PTR])[0] = 0;
    as<int64_t>(f.arr[DASP_ARR_RB_PTR])[0] = 0;
    as<int64_t>(f.arr[DASP_ARR_IRR_PTR])[0] = 0;
#pragma omp parallel for schedule(dynamic, 1) if (outer)
    for (int64_t q = 0; q < np; ++q) fill_panel<V>(f, panels[q], rp, col, val, !outer);
    // trailing long pad groups
    {
        V* lv = as<V>(f.arr[DASP_ARR_LONG_VAL]);
        int32_t* lc = as<int32_t>(f.arr[DASP_ARR_LONG_COL]);
        for (int64_t e = f.nnz_long_new; e < ne; ++e) { lv[e] = V(0); lc[e] = PAD_COL; }
    }
    // panel table: row0, rows, unit0, nunits, rb0, nrb, tile0, t13, t4, t22, ts, out0
    int64_t* pt = as<int64_t>(f.arr[DASP_ARR_PANELS]);
    for (int64_t q = 0; q < np; ++q) {
        const Panel& P = panels[q];
        int64_t* e = pt + q * PANEL_FIELDS;
        const int64_t u0 = (P.o_group + geo.UG - 1) / geo.UG;          // units whose first group is here
        const int64_t u1 = (P.o_group + P.n_groups + geo.UG - 1) / geo.UG;
        e[0] = P.r0; e[1] = P.r1 - P.r0; e[2] = u0; e[3] = u1 - u0; e[4] = P.o_rb; e[5] = P.nrb;
        e[6] = P.o_tile; e[7] = P.t13; e[8] = P.t4; e[9] = P.t22; e[10] = P.ts; e[11] = P.o_out;
    }
    return DASP_OK;
}

}  // namespace

int build_format(HostFormat& f, int dtype, int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col,
                 const void* val, int nthreads, bool validate, int64_t panel_rows, int64_t max_len, double tau) {
    f = HostFormat{};
    f.max_len = max_len > 0 ? max_len : MAX_LEN;
    f.tau = tau > 0.0 ? tau : 0.75;
    if (f.max_len < 4 || f.tau > 1.0) return DASP_ERR_INVALID_ARG;
    f.geo = geometry(dtype);
    f.dtype = dtype;
    f.m = m;
    f.n = n;
    f.nnz = m > 0 ? row_ptr[m] : 0;
    f.panel_rows = (panel_rows <= 0 || panel_rows >= m) ? std::max<int64_t>(m, 1) : panel_rows;
    const int prev_threads = omp_get_max_threads();
    if (nthreads > 0) omp_set_num_threads(nthreads);
    struct Restore { int n; ~Restore() { omp_set_num_threads(n); } } restore{prev_threads};
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
    else if (dtype == DASP_R_32F) st = build_impl<uint32_t>(f, m, row_ptr, col, static_cast<const uint32_t*>(val));
    else st = build_impl<uint16_t>(f, m, row_ptr, col, static_cast<const uint16_t*>(val));
    if (st != DASP_OK) f.release();
    return st;
}

}  // namespace dasp
