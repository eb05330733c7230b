// gpu_builder.cu — the DASP format built on the GPU from a device-resident CSR (SURVEY.md §8(f)
// f2: "histogram -> counting sort by len -> prefix-sum piecing -> scatter").
//
// Produces exactly the bytes of the host builder (builder.cpp) and of the oracle's literal
// builder (tests/test_gpu_builder.py compares all three).  Steps, all panels at once:
//   1. class of every row, stable radix sort of rows by (panel, class) -> per-panel
//      class lists in ascending row order (the host builder's stable partition);
//   2. long rows: groups of G by an exclusive scan -> group_ptr, one warp per row copies
//      the row and its pads;
//   3. medium rows: stable radix sort by (panel, MAX_LEN - len), row-blocks of 8, the
//      regular prefix per row-block (tau, R4/R6), exclusive scans -> rb_ptr / irr_ptr, scatter of
//      regular chunks (R18) and irregular tails;
//   4. short rows: per-panel piecing counts on the host (a few integers per panel), scatter of the
//      1&3 / len-4 / 2&2 / single tiles (R13);
//   5. empty rows and the panel table.
// CUB (part of the CUDA toolkit) provides the radix sorts and scans.
#include <cub/cub.cuh>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "gpu_builder.cuh"

namespace dasp {
namespace {

#define GB_CHECK(x)                                      \
    do {                                                 \
        cudaError_t e_ = (x);                            \
        if (e_ != cudaSuccess) return DASP_ERR_CUDA;     \
    } while (0)

enum { C_EMPTY = 0, C_S1, C_S2, C_S3, C_S4, C_MED, C_LONG, C_NUM };
constexpr int CLS_STRIDE = 8;   // key = panel * 8 + class

struct Buf {
    void* p = nullptr;
    ~Buf() { if (p) cudaFree(p); }
    cudaError_t alloc(size_t bytes) { return cudaMalloc(&p, bytes > 0 ? bytes : 16); }
    template <typename T> T* as() const { return static_cast<T*>(p); }
};

// host <-> device copies ordered on the build stream (D2H waits for it)
cudaError_t h2d(void* dst, const void* src, size_t bytes, cudaStream_t s) {
    return bytes ? cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, s) : cudaSuccess;
}
cudaError_t d2h(void* dst, const void* src, size_t bytes, cudaStream_t s) {
    if (!bytes) return cudaSuccess;
    cudaError_t e = cudaMemcpyAsync(dst, src, bytes, cudaMemcpyDeviceToHost, s);
    return e != cudaSuccess ? e : cudaStreamSynchronize(s);
}

inline unsigned nblk(int64_t n, int t = 256) { return static_cast<unsigned>(std::max<int64_t>(1, (n + t - 1) / t)); }

__device__ __forceinline__ int class_of(int64_t L, int64_t max_len) {
    return L > max_len ? C_LONG : (L > 4 ? C_MED : static_cast<int>(L));
}

__global__ void k_validate(const int64_t* rp, const int32_t* col, int64_t m, int64_t n, int64_t nnz, int* bad) {
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    for (int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; i < m; i += stride)
        if (rp[i + 1] < rp[i]) atomicOr(bad, 1);
    for (int64_t k = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; k < nnz; k += stride)
        if (col[k] < 0 || col[k] >= n) atomicOr(bad, 1);
}

__global__ void k_classify(const int64_t* rp, int64_t m, int64_t R, int64_t max_len, int32_t* key, int32_t* row) {
    const int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (i >= m) return;
    key[i] = static_cast<int32_t>((i / R) * CLS_STRIDE + class_of(rp[i + 1] - rp[i], max_len));
    row[i] = static_cast<int32_t>(i);
}

// start[k] = first position of key k in the sorted keys (k = 0 .. nkeys)
__global__ void k_bounds(const int32_t* keys, int64_t m, int64_t nkeys, int64_t* start) {
    const int64_t k = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (k > nkeys) return;
    int64_t lo = 0, hi = m;
    while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if (keys[mid] < k) lo = mid + 1; else hi = mid;
    }
    start[k] = lo;
}

// gather the class-`cls` segment of every panel, back to back in panel order
__global__ void k_gather_class(const int32_t* order, const int64_t* start, int64_t np, int cls, const int64_t* dst0,
                               int64_t total, int32_t* out) {
    const int64_t j = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (j >= total) return;
    int64_t lo = 0, hi = np;   // panel: last p with dst0[p] <= j
    while (hi - lo > 1) {
        const int64_t mid = (lo + hi) >> 1;
        if (dst0[mid] <= j) lo = mid; else hi = mid;
    }
    out[j] = order[start[lo * CLS_STRIDE + cls] + (j - dst0[lo])];
}

// ---- long rows ----
__global__ void k_long_groups(const int64_t* rp, const int32_t* lrow, int64_t nl, int G, int64_t* groups,
                              unsigned long long* nnz_long) {
    const int64_t r = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (r >= nl) return;
    const int64_t L = rp[lrow[r] + 1] - rp[lrow[r]];
    groups[r] = (L + G - 1) / G;
    atomicAdd(nnz_long, static_cast<unsigned long long>(L));
}

template <typename V>
__global__ void k_long_fill(const int64_t* rp, const int32_t* col, const V* val, const int32_t* lrow,
                            const int64_t* gp, int64_t nl, int G, V* lv, int32_t* lc) {
    const int64_t r = (static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (r >= nl) return;
    const int64_t i = lrow[r], b = rp[i], L = rp[i + 1] - b, at = gp[r] * G, end = gp[r + 1] * G;
    for (int64_t k = lane; k < end - at; k += 32) {
        if (k < L) { lv[at + k] = val[b + k]; lc[at + k] = col[b + k]; }
        else { lv[at + k] = V(0); lc[at + k] = PAD_COL; }
    }
}

template <typename V>
__global__ void k_pad(V* v, int32_t* c, int64_t from, int64_t to) {
    const int64_t e = from + static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (e < to) { v[e] = V(0); c[e] = PAD_COL; }
}

// ---- medium rows ----
__global__ void k_med_keys(const int64_t* rp, const int32_t* mrow, int64_t nm, int64_t R, int64_t max_len,
                           uint64_t* key) {
    const int64_t j = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (j >= nm) return;
    const int64_t i = mrow[j];
    key[j] = static_cast<uint64_t>(i / R) * static_cast<uint64_t>(max_len + 1) +
             static_cast<uint64_t>(max_len - (rp[i + 1] - rp[i]));
}

// padded sorted slots: panel p owns rb [rb0[p], rb0[p+1]); slot k < nm_p is a row, else -1
__global__ void k_med_pad(const int32_t* msorted, const int64_t* rb0, const int64_t* m0, int64_t np, int64_t nslots,
                          int32_t* slot_row) {
    const int64_t j = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (j >= nslots) return;
    const int64_t rb = j >> 3;
    int64_t lo = 0, hi = np;
    while (hi - lo > 1) {
        const int64_t mid = (lo + hi) >> 1;
        if (rb0[mid] <= rb) lo = mid; else hi = mid;
    }
    const int64_t k = j - rb0[lo] * 8, nm = m0[lo + 1] - m0[lo];
    slot_row[j] = k < nm ? msorted[m0[lo] + k] : -1;
}

__global__ void k_med_nreg(const int64_t* rp, const int32_t* slot_row, int64_t nrb, int K, int BE, double tau,
                           int64_t* reg_elems, int32_t* nreg, int64_t* irr_len, unsigned long long* stats) {
    const int64_t rb = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (rb >= nrb) return;
    int64_t L[8];
    unsigned long long s1 = 0, s2 = 0;
    for (int g = 0; g < 8; ++g) {
        const int32_t r = slot_row[rb * 8 + g];
        L[g] = r < 0 ? 0 : rp[r + 1] - rp[r];
        s1 += static_cast<unsigned long long>(L[g]);
        s2 += static_cast<unsigned long long>(L[g] * L[g]);
    }
    const double thr = static_cast<double>(BE) * tau;   // regular iff count > BE * tau (R4)
    int64_t b = 0;
    for (;;) {
        int64_t c = 0;
        for (int g = 0; g < 8; ++g) c += min(max(L[g] - K * b, int64_t(0)), int64_t(K));
        if (static_cast<double>(c) > thr) ++b; else break;
    }
    nreg[rb] = static_cast<int32_t>(b);
    reg_elems[rb] = b * BE;
    for (int g = 0; g < 8; ++g) irr_len[rb * 8 + g] = max(int64_t(0), L[g] - K * b);
    atomicAdd(&stats[0], s1);
    atomicAdd(&stats[1], s2);
}

// one thread per (row-block, row g): its regular slots (lane-interleaved chunks, R18) and tail
template <typename V>
__global__ void k_med_fill(const int64_t* rp, const int32_t* col, const V* val, const int32_t* slot_row,
                           const int32_t* nreg, const int64_t* rbp, const int64_t* ip, int64_t nrb, int K, int BE,
                           int EPL, int CW, V* rv, int32_t* rc, V* iv, int32_t* ic, int32_t* mo) {
    const int64_t j = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (j >= nrb * 8) return;
    const int64_t rb = j >> 3;
    const int g = static_cast<int>(j & 7);
    const int32_t row = slot_row[j];
    mo[j] = row;
    const int64_t L = row < 0 ? 0 : rp[row + 1] - rp[row], src = row < 0 ? 0 : rp[row];
    const int64_t nr = nreg[rb], base = rbp[rb], nslot = K * nr;
    for (int64_t s = 0; s < nslot; ++s) {
        const int64_t b = s / K;
        const int k = static_cast<int>(s % K);
        const int t = EPL == 1 ? k : (k >> 1), e = EPL == 1 ? 0 : (k & 1);
        const int lane = 4 * g + t;
        const int64_t c = b / CW, jb = b % CW;
        const int64_t w = min(static_cast<int64_t>(CW), nr - c * CW);
        const int64_t at = w == CW ? base + c * CW * BE + lane * w * EPL + jb * EPL + e    // full chunk (R18)
                                   : base + c * CW * BE + jb * BE + lane * EPL + e;        // ragged tail
        if (s < L) { rv[at] = val[src + s]; rc[at] = col[src + s]; }
        else { rv[at] = V(0); rc[at] = PAD_COL; }
    }
    for (int64_t s = nslot; s < L; ++s) {
        iv[ip[j] + s - nslot] = val[src + s];
        ic[ip[j] + s - nslot] = col[src + s];
    }
}

// ---- short rows ----
struct ShortPanel {      // per panel, built on the host from the class counts
    int64_t s[5];        // start of the class-c segment of `order` (c = 1..4)
    int64_t n[5];        // class sizes
    int64_t p13, p22, n3l, n4cat, ns;
    int64_t tile0, t13, t4, t22, out0;
    int64_t q13, q4, q22, qs;   // prefix offsets of the flattened per-category index spaces
};

__device__ __forceinline__ int short_pos(int K, int r, int c) {
    if (K == 4) return 4 * (4 * (r & 7) + c) + (r >> 3);
    const int q = r >> 3, g = r & 7;
    const int t = ((q & 1) << 1) | (c >> 1);
    const int j = ((q >> 1) << 1) | (c & 1);
    return 4 * (4 * g + t) + j;
}

__device__ __forceinline__ int64_t panel_of(const ShortPanel* sp, int64_t np, int64_t j, int field) {
    int64_t lo = 0, hi = np;   // last p with prefix[p] <= j
    while (hi - lo > 1) {
        const int64_t mid = (lo + hi) >> 1;
        const int64_t v = field == 0 ? sp[mid].q13 : field == 1 ? sp[mid].q4 : field == 2 ? sp[mid].q22 : sp[mid].qs;
        if (v <= j) lo = mid; else hi = mid;
    }
    return lo;
}

template <typename V>
__device__ __forceinline__ void put_row4(const int64_t* rp, const int32_t* col, const V* val, V* tv, int32_t* tc, int K,
                                         int r, int64_t ra, int la, int64_t rb_, int lb) {
    for (int k = 0; k < la; ++k) { const int p = short_pos(K, r, k); tv[p] = val[rp[ra] + k]; tc[p] = col[rp[ra] + k]; }
    if (rb_ >= 0)
        for (int k = 0; k < lb; ++k) { const int p = short_pos(K, r, la + k); tv[p] = val[rp[rb_] + k]; tc[p] = col[rp[rb_] + k]; }
}

template <typename V>
__global__ void k_short(const int64_t* rp, const int32_t* col, const V* val, const int32_t* order, const ShortPanel* sp,
                        int64_t np, int cat, int64_t total, int K, V* sval, int32_t* scol, int32_t* sout) {
    const int64_t j = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (j >= total) return;
    const int64_t p = panel_of(sp, np, j, cat);
    const ShortPanel& P = sp[p];
    if (cat == 0) {                                   // 1&3: slot 0 = len-1 row, slots 1-3 = len-3 row
        const int64_t q = j - P.q13;
        const int r = static_cast<int>(q % 32);
        const int64_t a = order[P.s[1] + q], b = order[P.s[3] + q];
        const int64_t tile = P.tile0 + q / 32;
        put_row4(rp, col, val, sval + tile * 128, scol + tile * 128, K, r, a, 1, b, 3);
        const int64_t o = P.out0 + (q / 32) * 64 + 16 * (r >> 3) + (r & 7);
        sout[o] = static_cast<int32_t>(a);
        sout[o + 8] = static_cast<int32_t>(b);
    } else if (cat == 1) {                            // len-4: true 4s, leftover 3s, the odd 2 (R13)
        const int64_t q = j - P.q4;
        int64_t row;
        int len;
        if (q < P.n[4]) { row = order[P.s[4] + q]; len = 4; }
        else if (q < P.n[4] + P.n3l) { row = order[P.s[3] + P.p13 + q - P.n[4]]; len = 3; }
        else { row = order[P.s[2] + P.n[2] - 1]; len = 2; }
        const int64_t tile = P.tile0 + P.t13 + q / 32;
        put_row4(rp, col, val, sval + tile * 128, scol + tile * 128, K, static_cast<int>(q % 32), row, len, -1, 0);
        sout[P.out0 + 64 * P.t13 + q] = static_cast<int32_t>(row);
    } else if (cat == 2) {                            // 2&2
        const int64_t q = j - P.q22;
        const int r = static_cast<int>(q % 32);
        const int64_t a = order[P.s[2] + 2 * q], b = order[P.s[2] + 2 * q + 1];
        const int64_t tile = P.tile0 + P.t13 + P.t4 + q / 32;
        put_row4(rp, col, val, sval + tile * 128, scol + tile * 128, K, r, a, 2, b, 2);
        const int64_t o = P.out0 + 64 * P.t13 + 32 * P.t4 + (q / 32) * 64 + 16 * (r >> 3) + (r & 7);
        sout[o] = static_cast<int32_t>(a);
        sout[o + 8] = static_cast<int32_t>(b);
    } else {                                          // singles (Alg. 5)
        const int64_t q = j - P.qs;
        const int64_t i = order[P.s[1] + P.p13 + q];
        const int64_t t0 = (P.tile0 + P.t13 + P.t4 + P.t22) * 128;
        sval[t0 + q] = val[rp[i]];
        scol[t0 + q] = col[rp[i]];
        sout[P.out0 + 64 * P.t13 + 32 * P.t4 + 64 * P.t22 + q] = static_cast<int32_t>(i);
    }
}

template <typename V>
__global__ void k_short_init(V* v, int32_t* c, int64_t ne, int32_t* o, int64_t no) {
    const int64_t e = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (e < ne) { v[e] = V(0); c[e] = PAD_COL; }
    if (e < no) o[e] = -1;
}

template <typename KT>
cudaError_t radix_sort(const KT* kin, KT* kout, const int32_t* vin, int32_t* vout, int64_t n, int end_bit, cudaStream_t s) {
    size_t tb = 0;
    cudaError_t e = cub::DeviceRadixSort::SortPairs(nullptr, tb, kin, kout, vin, vout, n, 0, end_bit, s);
    if (e != cudaSuccess) return e;
    Buf tmp;
    if ((e = tmp.alloc(tb)) != cudaSuccess) return e;
    e = cub::DeviceRadixSort::SortPairs(tmp.p, tb, kin, kout, vin, vout, n, 0, end_bit, s);
    if (e != cudaSuccess) return e;
    return cudaStreamSynchronize(s);
}

cudaError_t exclusive_scan(const int64_t* in, int64_t* out, int64_t n, cudaStream_t s) {
    size_t tb = 0;
    cudaError_t e = cub::DeviceScan::ExclusiveSum(nullptr, tb, in, out, n, s);
    if (e != cudaSuccess) return e;
    Buf tmp;
    if ((e = tmp.alloc(tb)) != cudaSuccess) return e;
    e = cub::DeviceScan::ExclusiveSum(tmp.p, tb, in, out, n, s);
    if (e != cudaSuccess) return e;
    return cudaStreamSynchronize(s);
}

int bits_for(uint64_t maxkey) {
    int b = 1;
    while (b < 64 && (maxkey >> b)) ++b;
    return b;
}

// build knob DASP_GB_TRACE=1 prints the time of every builder phase (stderr)
#ifndef DASP_GB_TRACE
#define DASP_GB_TRACE 0
#endif
struct Trace {
    bool on = DASP_GB_TRACE != 0;
    cudaStream_t s;
    std::chrono::steady_clock::time_point t = std::chrono::steady_clock::now();
    void operator()(const char* what) {
        if (!on) return;
        cudaStreamSynchronize(s);
        auto now = std::chrono::steady_clock::now();
        std::fprintf(stderr, "[gpu_builder] %-22s %8.3f ms\n", what, std::chrono::duration<double, std::milli>(now - t).count());
        t = now;
    }
};

template <typename V>
int build_impl(HostFormat& f, void** d, const int64_t* rp, const int32_t* col, const V* val, cudaStream_t s) {
    Trace tr{};
    tr.s = s;
    const Geometry geo = f.geo;
    const int64_t m = f.m, R = f.panel_rows;
    const int64_t np = m > 0 ? (m + R - 1) / R : 1;
    const int64_t nkeys = np * CLS_STRIDE;
    // ---- 1. classes, stable partition by (panel, class) ----
    Buf key, key2, row, order, start;
    GB_CHECK(key.alloc(m * 4)); GB_CHECK(key2.alloc(m * 4)); GB_CHECK(row.alloc(m * 4)); GB_CHECK(order.alloc(m * 4));
    GB_CHECK(start.alloc((nkeys + 1) * 8));
    if (m > 0) {
        k_classify<<<nblk(m), 256, 0, s>>>(rp, m, R, f.max_len, key.as<int32_t>(), row.as<int32_t>());
        GB_CHECK(radix_sort<int32_t>(key.as<int32_t>(), key2.as<int32_t>(), row.as<int32_t>(), order.as<int32_t>(), m,
                                     bits_for(static_cast<uint64_t>(nkeys)), s));
    }
    k_bounds<<<nblk(nkeys + 1), 256, 0, s>>>(key2.as<int32_t>(), m, nkeys, start.as<int64_t>());
    std::vector<int64_t> st(static_cast<size_t>(nkeys + 1));
    GB_CHECK(d2h(st.data(), start.p, (nkeys + 1) * 8, s));
    auto cnt = [&](int64_t p, int c) { return st[p * CLS_STRIDE + c + 1] - st[p * CLS_STRIDE + c]; };
    tr("classify+partition");

    // per-panel prefix offsets of every class
    std::vector<int64_t> off[C_NUM];
    for (int c = 0; c < C_NUM; ++c) {
        off[c].assign(static_cast<size_t>(np + 1), 0);
        for (int64_t p = 0; p < np; ++p) off[c][p + 1] = off[c][p] + cnt(p, c);
    }
    f.n0 = off[C_EMPTY][np]; f.n1 = off[C_S1][np]; f.n2 = off[C_S2][np]; f.n3 = off[C_S3][np]; f.n4 = off[C_S4][np];
    f.row_medium = off[C_MED][np];
    f.row_long = off[C_LONG][np];
    f.n_panels = np;
    Buf doff;
    GB_CHECK(doff.alloc((np + 1) * 8));
    auto gather_class = [&](int c, int32_t* out) -> cudaError_t {
        const int64_t total = off[c][np];
        if (total == 0) return cudaSuccess;
        cudaError_t e = h2d(doff.p, off[c].data(), (np + 1) * 8, s);
        if (e != cudaSuccess) return e;
        k_gather_class<<<nblk(total), 256, 0, s>>>(order.as<int32_t>(), start.as<int64_t>(), np, c, doff.as<int64_t>(),
                                                   total, out);
        return cudaGetLastError();
    };

    auto alloc_out = [&](int a, int64_t bytes) -> cudaError_t {
        f.arr[a].bytes = bytes;
        return cudaMalloc(&d[a], static_cast<size_t>(bytes + kDeviceArrayPad));
    };
    // ---- 5a. empty rows ----
    GB_CHECK(alloc_out(DASP_ARR_EMPTY_ROWS, f.n0 * 4));
    GB_CHECK(gather_class(C_EMPTY, static_cast<int32_t*>(d[DASP_ARR_EMPTY_ROWS])));

    // ---- 2. long rows ----
    const int64_t nl = f.row_long;
    GB_CHECK(alloc_out(DASP_ARR_LONG_OUT, nl * 4));
    GB_CHECK(alloc_out(DASP_ARR_GROUP_PTR, (nl + 1) * 8));
    GB_CHECK(gather_class(C_LONG, static_cast<int32_t*>(d[DASP_ARR_LONG_OUT])));
    Buf groups, stats;
    GB_CHECK(groups.alloc((nl + 1) * 8));
    GB_CHECK(stats.alloc(3 * 8));
    GB_CHECK(cudaMemsetAsync(stats.p, 0, 3 * 8, s));
    GB_CHECK(cudaMemsetAsync(groups.p, 0, (nl + 1) * 8, s));
    if (nl > 0)
        k_long_groups<<<nblk(nl), 256, 0, s>>>(rp, static_cast<int32_t*>(d[DASP_ARR_LONG_OUT]), nl, geo.G,
                                               groups.as<int64_t>(), stats.as<unsigned long long>() + 2);
    GB_CHECK(exclusive_scan(groups.as<int64_t>(), static_cast<int64_t*>(d[DASP_ARR_GROUP_PTR]), nl + 1, s));
    std::vector<int64_t> gp_host(static_cast<size_t>(nl + 1));
    GB_CHECK(d2h(gp_host.data(), d[DASP_ARR_GROUP_PTR], (nl + 1) * 8, s));
    f.n_groups = gp_host[nl];
    f.n_groups_padded = (f.n_groups + geo.UG - 1) / geo.UG * geo.UG;
    f.nnz_long_new = f.n_groups * geo.G;
    const int64_t ne = f.n_groups_padded * geo.G;
    GB_CHECK(alloc_out(DASP_ARR_LONG_VAL, ne * geo.sv));
    GB_CHECK(alloc_out(DASP_ARR_LONG_COL, ne * 4));
    if (nl > 0)
        k_long_fill<V><<<nblk(nl * 32), 256, 0, s>>>(rp, col, val, static_cast<int32_t*>(d[DASP_ARR_LONG_OUT]),
                                                     static_cast<int64_t*>(d[DASP_ARR_GROUP_PTR]), nl, geo.G,
                                                     static_cast<V*>(d[DASP_ARR_LONG_VAL]),
                                                     static_cast<int32_t*>(d[DASP_ARR_LONG_COL]));
    if (ne > f.nnz_long_new)
        k_pad<V><<<nblk(ne - f.nnz_long_new), 256, 0, s>>>(static_cast<V*>(d[DASP_ARR_LONG_VAL]),
                                                           static_cast<int32_t*>(d[DASP_ARR_LONG_COL]), f.nnz_long_new, ne);

    tr("long rows");
    // ---- 3. medium rows ----
    const int64_t nm = f.row_medium;
    std::vector<int64_t> rb0(static_cast<size_t>(np + 1), 0);
    for (int64_t p = 0; p < np; ++p) rb0[p + 1] = rb0[p] + (cnt(p, C_MED) + 7) / 8;
    const int64_t nrb = rb0[np];
    f.nrb = nrb;
    Buf mrow, mkey, mkey2, msorted, slot_row, nreg, reg_elems, irr_len, drb0;
    GB_CHECK(mrow.alloc(nm * 4)); GB_CHECK(mkey.alloc(nm * 8)); GB_CHECK(mkey2.alloc(nm * 8)); GB_CHECK(msorted.alloc(nm * 4));
    GB_CHECK(slot_row.alloc(nrb * 8 * 4)); GB_CHECK(nreg.alloc(nrb * 4)); GB_CHECK(reg_elems.alloc((nrb + 1) * 8));
    GB_CHECK(irr_len.alloc((nrb * 8 + 1) * 8)); GB_CHECK(drb0.alloc((np + 1) * 8));
    GB_CHECK(gather_class(C_MED, mrow.as<int32_t>()));
    if (nm > 0) {
        k_med_keys<<<nblk(nm), 256, 0, s>>>(rp, mrow.as<int32_t>(), nm, R, f.max_len, mkey.as<uint64_t>());
        GB_CHECK(radix_sort<uint64_t>(mkey.as<uint64_t>(), mkey2.as<uint64_t>(), mrow.as<int32_t>(), msorted.as<int32_t>(),
                                      nm, bits_for(static_cast<uint64_t>(np) * static_cast<uint64_t>(f.max_len + 1)), s));
    }
    GB_CHECK(h2d(drb0.p, rb0.data(), (np + 1) * 8, s));
    GB_CHECK(h2d(doff.p, off[C_MED].data(), (np + 1) * 8, s));
    GB_CHECK(cudaMemsetAsync(reg_elems.p, 0, (nrb + 1) * 8, s));
    GB_CHECK(cudaMemsetAsync(irr_len.p, 0, (nrb * 8 + 1) * 8, s));
    if (nrb > 0) {
        k_med_pad<<<nblk(nrb * 8), 256, 0, s>>>(msorted.as<int32_t>(), drb0.as<int64_t>(), doff.as<int64_t>(), np, nrb * 8,
                                                slot_row.as<int32_t>());
        k_med_nreg<<<nblk(nrb), 256, 0, s>>>(rp, slot_row.as<int32_t>(), nrb, geo.K, geo.BE, f.tau, reg_elems.as<int64_t>(),
                                             nreg.as<int32_t>(), irr_len.as<int64_t>(), stats.as<unsigned long long>());
    }
    GB_CHECK(alloc_out(DASP_ARR_RB_PTR, (nrb + 1) * 8));
    GB_CHECK(alloc_out(DASP_ARR_IRR_PTR, (nrb * 8 + 1) * 8));
    GB_CHECK(alloc_out(DASP_ARR_MED_OUT, nrb * 8 * 4));
    GB_CHECK(exclusive_scan(reg_elems.as<int64_t>(), static_cast<int64_t*>(d[DASP_ARR_RB_PTR]), nrb + 1, s));
    GB_CHECK(exclusive_scan(irr_len.as<int64_t>(), static_cast<int64_t*>(d[DASP_ARR_IRR_PTR]), nrb * 8 + 1, s));
    GB_CHECK(d2h(&f.nnz_reg_new, static_cast<int64_t*>(d[DASP_ARR_RB_PTR]) + nrb, 8, s));
    GB_CHECK(d2h(&f.nnz_irreg, static_cast<int64_t*>(d[DASP_ARR_IRR_PTR]) + nrb * 8, 8, s));
    GB_CHECK(alloc_out(DASP_ARR_REG_VAL, f.nnz_reg_new * geo.sv));
    GB_CHECK(alloc_out(DASP_ARR_REG_COL, f.nnz_reg_new * 4));
    GB_CHECK(alloc_out(DASP_ARR_IRR_VAL, f.nnz_irreg * geo.sv));
    GB_CHECK(alloc_out(DASP_ARR_IRR_COL, f.nnz_irreg * 4));
    if (nrb > 0)
        k_med_fill<V><<<nblk(nrb * 8), 256, 0, s>>>(rp, col, val, slot_row.as<int32_t>(), nreg.as<int32_t>(),
                                                    static_cast<int64_t*>(d[DASP_ARR_RB_PTR]),
                                                    static_cast<int64_t*>(d[DASP_ARR_IRR_PTR]), nrb, geo.K, geo.BE,
                                                    geo.EPL, geo.CW, static_cast<V*>(d[DASP_ARR_REG_VAL]),
                                                    static_cast<int32_t*>(d[DASP_ARR_REG_COL]),
                                                    static_cast<V*>(d[DASP_ARR_IRR_VAL]),
                                                    static_cast<int32_t*>(d[DASP_ARR_IRR_COL]),
                                                    static_cast<int32_t*>(d[DASP_ARR_MED_OUT]));
    unsigned long long hs[3];
    GB_CHECK(d2h(hs, stats.p, 3 * 8, s));
    f.nnz_medium = static_cast<int64_t>(hs[0]);
    f.sumsq_medium = static_cast<int64_t>(hs[1]);
    f.nnz_long = static_cast<int64_t>(hs[2]);

    tr("medium rows");
    // ---- 4. short rows: piecing counts per panel on the host ----
    std::vector<ShortPanel> sp(static_cast<size_t>(np));
    int64_t tile = 0, out = 0, q13 = 0, q4 = 0, q22 = 0, qs = 0;
    for (int64_t p = 0; p < np; ++p) {
        ShortPanel& P = sp[p];
        for (int c = 1; c <= 4; ++c) { P.s[c] = st[p * CLS_STRIDE + c]; P.n[c] = cnt(p, c); }
        P.s[0] = P.n[0] = 0;
        P.p13 = std::min(P.n[1], P.n[3]); P.p22 = P.n[2] / 2; P.n3l = P.n[3] - P.p13;
        P.n4cat = P.n[4] + P.n3l + P.n[2] % 2; P.ns = P.n[1] - P.p13;
        P.t13 = (P.p13 + 31) / 32; P.t4 = (P.n4cat + 31) / 32; P.t22 = (P.p22 + 31) / 32;
        const int64_t ts = (P.ns + SHORT_TILE - 1) / SHORT_TILE;
        P.tile0 = tile; P.out0 = out;
        P.q13 = q13; P.q4 = q4; P.q22 = q22; P.qs = qs;
        q13 += P.p13; q4 += P.n4cat; q22 += P.p22; qs += P.ns;
        tile += P.t13 + P.t4 + P.t22 + ts;
        out += 64 * P.t13 + 32 * P.t4 + 64 * P.t22 + SHORT_TILE * ts;
        f.t13 += P.t13; f.t4 += P.t4; f.t22 += P.t22; f.ts += ts;
    }
    f.nnz_short_new = tile * SHORT_TILE;
    f.nnz_short = f.n1 + 2 * f.n2 + 3 * f.n3 + 4 * f.n4;
    GB_CHECK(alloc_out(DASP_ARR_SHORT_VAL, tile * SHORT_TILE * geo.sv));
    GB_CHECK(alloc_out(DASP_ARR_SHORT_COL, tile * SHORT_TILE * 4));
    GB_CHECK(alloc_out(DASP_ARR_SHORT_OUT, out * 4));
    Buf dsp;
    GB_CHECK(dsp.alloc(np * sizeof(ShortPanel)));
    GB_CHECK(h2d(dsp.p, sp.data(), np * sizeof(ShortPanel), s));
    const int64_t ninit = std::max(tile * SHORT_TILE, out);
    if (ninit > 0)
        k_short_init<V><<<nblk(ninit), 256, 0, s>>>(static_cast<V*>(d[DASP_ARR_SHORT_VAL]),
                                                    static_cast<int32_t*>(d[DASP_ARR_SHORT_COL]), tile * SHORT_TILE,
                                                    static_cast<int32_t*>(d[DASP_ARR_SHORT_OUT]), out);
    const int64_t tot[4] = {q13, q4, q22, qs};
    for (int c = 0; c < 4; ++c)
        if (tot[c] > 0)
            k_short<V><<<nblk(tot[c]), 256, 0, s>>>(rp, col, val, order.as<int32_t>(), dsp.as<ShortPanel>(), np, c, tot[c],
                                                    geo.K, static_cast<V*>(d[DASP_ARR_SHORT_VAL]),
                                                    static_cast<int32_t*>(d[DASP_ARR_SHORT_COL]),
                                                    static_cast<int32_t*>(d[DASP_ARR_SHORT_OUT]));

    tr("short rows");
    // ---- 5b. panel table (host) ----
    f.panel_table.assign(static_cast<size_t>(np * PANEL_FIELDS), 0);
    for (int64_t p = 0; p < np; ++p) {
        int64_t* e = f.panel_table.data() + p * PANEL_FIELDS;
        const int64_t g0 = gp_host[off[C_LONG][p]], g1 = gp_host[off[C_LONG][p + 1]];
        const int64_t u0 = (g0 + geo.UG - 1) / geo.UG, u1 = (g1 + geo.UG - 1) / geo.UG;
        const int64_t ts = (sp[p].ns + SHORT_TILE - 1) / SHORT_TILE;
        e[0] = std::min(m, p * R); e[1] = std::min(m, (p + 1) * R) - e[0]; e[2] = u0; e[3] = u1 - u0;
        e[4] = rb0[p]; e[5] = rb0[p + 1] - rb0[p];
        e[6] = sp[p].tile0; e[7] = sp[p].t13; e[8] = sp[p].t4; e[9] = sp[p].t22; e[10] = ts; e[11] = sp[p].out0;
    }
    GB_CHECK(alloc_out(DASP_ARR_PANELS, np * PANEL_FIELDS * 8));
    GB_CHECK(h2d(d[DASP_ARR_PANELS], f.panel_table.data(), np * PANEL_FIELDS * 8, s));
    GB_CHECK(cudaStreamSynchronize(s));
    GB_CHECK(cudaGetLastError());
    tr("panel table");
    return DASP_OK;
}

__global__ void k_first_col(const int32_t* lc, int64_t ue, int64_t nu, int32_t* out) {
    const int64_t u = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x;
    if (u < nu) out[u] = lc[u * ue];
}

}  // namespace

namespace {
// medium-class length statistics (count, sum, sum of squares) of rows with lo <= len <= hi
__global__ void k_medium_stats(const int64_t* __restrict__ rp, int64_t m, int64_t lo, int64_t hi,
                               unsigned long long* __restrict__ out) {
    unsigned long long c = 0, s1 = 0, s2 = 0;
    for (int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; i < m;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        const int64_t L = rp[i + 1] - rp[i];
        if (L >= lo && L <= hi) { ++c; s1 += L; s2 += static_cast<unsigned long long>(L * L); }
    }
    for (int o = 16; o > 0; o >>= 1) {
        c += __shfl_xor_sync(0xffffffffu, c, o);
        s1 += __shfl_xor_sync(0xffffffffu, s1, o);
        s2 += __shfl_xor_sync(0xffffffffu, s2, o);
    }
    if ((threadIdx.x & 31) == 0) { atomicAdd(out, c); atomicAdd(out + 1, s1); atomicAdd(out + 2, s2); }
}
}  // namespace

cudaError_t medium_length_stats(const int64_t* d_row_ptr, int64_t m, int64_t max_len, int64_t* count, int64_t* sum,
                                int64_t* sumsq, cudaStream_t s) {
    *count = *sum = *sumsq = 0;
    if (m <= 0) return cudaSuccess;
    Buf acc;
    cudaError_t e = acc.alloc(3 * 8);
    if (e != cudaSuccess || (e = cudaMemsetAsync(acc.p, 0, 24, s)) != cudaSuccess) return e;
    k_medium_stats<<<148 * 4, 256, 0, s>>>(d_row_ptr, m, MIN_MEDIUM_LEN, max_len, acc.as<unsigned long long>());
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    int64_t h[3];
    if ((e = d2h(h, acc.p, 24, s)) != cudaSuccess) return e;
    *count = h[0]; *sum = h[1]; *sumsq = h[2];
    return cudaSuccess;
}

cudaError_t gather_unit_first_col(const int32_t* d_long_col, int64_t unit_elems, int64_t n_units, int32_t* host_out,
                                  cudaStream_t s) {
    Buf tmp;
    cudaError_t e = tmp.alloc(n_units * 4);
    if (e != cudaSuccess) return e;
    k_first_col<<<nblk(n_units), 256, 0, s>>>(d_long_col, unit_elems, n_units, tmp.as<int32_t>());
    if ((e = cudaGetLastError()) != cudaSuccess) return e;
    return d2h(host_out, tmp.p, n_units * 4, s);
}

int build_format_device(HostFormat& f, void** d_arrays, int dtype, int64_t m, int64_t n, int64_t nnz,
                        const int64_t* d_row_ptr, const int32_t* d_col, const void* d_val, bool validate,
                        int64_t panel_rows, int64_t max_len, double tau, cudaStream_t s) {
    f = HostFormat{};
    f.geo = geometry(dtype);
    f.dtype = dtype;
    f.m = m;
    f.n = n;
    f.max_len = max_len > 0 ? max_len : MAX_LEN;
    f.tau = tau > 0.0 ? tau : 0.75;
    if (f.max_len < 4 || f.tau > 1.0) return DASP_ERR_INVALID_ARG;
    f.panel_rows = (panel_rows <= 0 || panel_rows >= m) ? std::max<int64_t>(m, 1) : panel_rows;
    if (d2h(&f.nnz, d_row_ptr + m, 8, s) != cudaSuccess) return DASP_ERR_CUDA;
    // every kernel below reads col / val up to row_ptr[m]: it must be the caller's array length
    if (f.nnz != nnz) return DASP_ERR_INVALID_CSR;
    if (validate) {
        int64_t r0 = 0;
        if (d2h(&r0, d_row_ptr, 8, s) != cudaSuccess) return DASP_ERR_CUDA;
        if (r0 != 0) return DASP_ERR_INVALID_CSR;
        Buf bad;
        if (bad.alloc(4) != cudaSuccess || cudaMemsetAsync(bad.p, 0, 4, s) != cudaSuccess) return DASP_ERR_CUDA;
        k_validate<<<148 * 8, 256, 0, s>>>(d_row_ptr, d_col, m, n, f.nnz, bad.as<int>());
        int hb = 0;
        if (d2h(&hb, bad.p, 4, s) != cudaSuccess) return DASP_ERR_CUDA;
        if (hb) return DASP_ERR_INVALID_CSR;
    }
    for (int a = 0; a < DASP_ARR_COUNT; ++a) d_arrays[a] = nullptr;
    int st = dtype == DASP_R_64F   ? build_impl<uint64_t>(f, d_arrays, d_row_ptr, d_col, static_cast<const uint64_t*>(d_val), s)
             : dtype == DASP_R_32F ? build_impl<uint32_t>(f, d_arrays, d_row_ptr, d_col, static_cast<const uint32_t*>(d_val), s)
                                   : build_impl<uint16_t>(f, d_arrays, d_row_ptr, d_col, static_cast<const uint16_t*>(d_val), s);
    if (st != DASP_OK) {
        for (int a = 0; a < DASP_ARR_COUNT; ++a) {
            if (d_arrays[a]) cudaFree(d_arrays[a]);
            d_arrays[a] = nullptr;
        }
    }
    return st;
}

}  // namespace dasp
