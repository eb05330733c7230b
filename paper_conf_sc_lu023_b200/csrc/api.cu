// api.cu — the C-ABI of libdasp.so (include/dasp.h): plan creation (host build + upload),
// the SpMV launch sequence, host-buffer end-to-end call, introspection, multi-GPU helpers
// and per-kernel event timing.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <memory>
#include <new>
#include <utility>
#include <vector>

#include "format.hpp"
#include "gpu_builder.cuh"
#include "kernels.cuh"

using dasp::HostFormat;

struct TimingRec {
    int kernel;
    cudaEvent_t a, b;
};

struct dasp_plan_s {
    int dtype = 0, device = -1, variant = DASP_VARIANT_CUDACORE, rbw = 1;
    int wide_il = 0;                      // interleaved wide medium warps (setup_launch)
    int narrow_il = 0;                    // interleaved narrow / mid medium warps (measured neutral / slower: off)
    int nrw = 0;                          // row-blocks per narrow / mid warp (0: no narrow path)
    bool occ5 = false;                    // FP16: CUDA-core main kernel at 5 blocks / SM (setup_launch)
    int tpw = 0;                          // short tiles per short warp of the layout
    int64_t rb_mid = 0, rb_narrow = 0;    // row-blocks on mid / narrow warps (all panels)
    bool keep_host = false;
    HostFormat host;                      // counts always valid; arrays freed after upload unless keep_host
    void* d[DASP_ARR_COUNT] = {};
    int64_t bytes[DASP_ARR_COUNT] = {};
    void* d_partial = nullptr;
    void* d_xh = nullptr;                 // dasp_spmv_host staging
    void* d_yh = nullptr;
    // dasp_spmv_host_stream: double-buffered device x/y, two copy streams, per-slot events
    void* d_xs[2] = {};
    void* d_ys[2] = {};
    cudaStream_t s_h2d = nullptr, s_d2h = nullptr;
    cudaEvent_t ev_x[2] = {}, ev_done[2] = {}, ev_yout[2] = {};
    int64_t device_bytes = 0;
    double build_ms = 0, upload_ms = 0;
    int64_t blocks = 0;                   // grid of the medium/short kernel
    int64_t n_units = 0;                  // long units (long kernel)
    void* d_panels = nullptr;             // dasp::PanelDesc[n_panels]
    void* d_warp_word = nullptr;          // uint64 panel / warp of every main-kernel warp (kernels.cuh)
    int64_t n_mwarps = 0;
    void* d_unit_order = nullptr;         // int32 long-unit execution order (column buckets)
    void* d_stage = nullptr;              // dasp::StageEnt per main block (x-window staging), or null
    void* d_stage_map = nullptr;          // the staged blocks' tile maps
    int stage_smem = 0;                   // dynamic shared memory of the staged instantiation
    int stage_map_bytes = 0;              // tile-map bytes in front of the staged tiles
    int64_t stage_blocks = 0;             // staged main blocks
    // timing
    int32_t timing_cap = 0, timing_calls = 0;
    std::vector<TimingRec> recs;
    std::vector<cudaEvent_t> pool;
    size_t pool_used = 0;
};

namespace {

int sx(int dtype) { return dtype == DASP_R_64F ? 8 : (dtype == DASP_R_32F ? 4 : 2); }
int sy(int dtype) { return dtype == DASP_R_64F ? 8 : 4; }
int sa(int dtype) { return dtype == DASP_R_16F ? 4 : 8; }   // long-group partials: f32 (FP16) / f64

// automatic panel: ~1M rows keeps a panel's x window and y (8 B each per row) well inside the
// ~50 MB of L2 that data shared by all SMs gets on B200 (profiles/r01 L2 probe)
constexpr int64_t kAutoPanelRows = int64_t(1) << 20;
#ifndef DASP_COL_BUCKETS
#define DASP_COL_BUCKETS 256   // long-unit column buckets: C3 FP16 long -2.6 %, C5 -1.1 %, C7 -1.7 %, C3 FP64 -0.5 % vs 16 (profiles/r02b/long_col_buckets.jsonl)
#endif
#ifndef DASP_LONG_ORDER
#define DASP_LONG_ORDER 2   // long-unit schedule: 0 memory order, 1 column buckets per panel, 2 global buckets (C3 long -6 %, profiles/r02/long_order.jsonl)
#endif
constexpr int kColBuckets = DASP_COL_BUCKETS;
constexpr int64_t kAllocPad = dasp::kDeviceArrayPad;   // vector loads may read up to 16 B past an array's end
// build knobs (experiments only; the product reads no environment): DASP_CLASS_MASK restricts the
// main kernel to medium (2) or short (4) warps for per-class timings -- the other rows are then
// NOT computed; DASP_NARROW_IL interleaves narrow warps (measured neutral / slower)
#ifndef DASP_CLASS_MASK
#define DASP_CLASS_MASK 7
#endif
#ifndef DASP_NARROW_IL
#define DASP_NARROW_IL 0
#endif
#ifndef DASP_PACK_WARPS
#define DASP_PACK_WARPS 1   // 1: panels' warps packed back to back in the main grid; 0: each panel padded to whole blocks
#endif
#ifndef DASP_HEAVY_FIRST_F16
#define DASP_HEAVY_FIRST_F16 8   // FP16: C3 main -3.2 % (3 reps), C5 +-0 vs 16 (profiles/r02b/heavy_first_f16.jsonl)
#endif
#ifndef DASP_HEAVY_FIRST
#define DASP_HEAVY_FIRST 16  // leading blocks of every panel dispatched at the start of the main grid (C3 FP16 -2.7 %, FP64 -0.1..-0.8 %, others +-0.8 %: profiles/r02/heavy_first_ab.jsonl, chunk_units_removed_and_heavy_first.jsonl)
#endif

// LOOP_NUM (row-blocks per warp, R11) re-tuned on B200 (profiles/r01/rbw_sweep.jsonl,
// profiles/r02/loop_num_recheck.jsonl): small matrices keep the paper's 1 / 2; for large ones, uniform
// medium rows (coefficient of variation of the length < 0.5, e.g. stencils) run best with 8 row-blocks
// per warp, ragged ones with 4, heavy-tailed ones (cv >= 1, power law) with 2 -- more would leave
// warps with very unequal work.
int auto_rbw(int64_t row_medium, int64_t nnz_medium, int64_t sumsq_medium) {
    if (row_medium < 59990) return 1;
    if (row_medium < 400000) return 2;
    const double mean = static_cast<double>(nnz_medium) / static_cast<double>(row_medium);
    const double var = static_cast<double>(sumsq_medium) / static_cast<double>(row_medium) - mean * mean;
    const double cv = var > 0 ? std::sqrt(var) / mean : 0.0;
    // heavy-tailed lengths (power law, cv >= 1) leave a few warps with far more chunks than the rest:
    // 2 row-blocks per warp (C3 main -4.3 %, FP16 -1.4 %; C5, cv 0.55, keeps 4: +2 % at 2;
    // profiles/r02/loop_num_recheck.jsonl)
    return cv < 0.5 ? 8 : (cv < 1.0 ? 4 : 2);
}

struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
        if (prev != dev) cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};

void free_device(dasp_plan_s* p) {
    for (auto& ptr : p->d) {
        if (ptr) cudaFree(ptr);
        ptr = nullptr;
    }
    if (p->d_partial) cudaFree(p->d_partial);
    if (p->d_panels) cudaFree(p->d_panels);
    if (p->d_warp_word) cudaFree(p->d_warp_word);
    if (p->d_unit_order) cudaFree(p->d_unit_order);
    if (p->d_stage) cudaFree(p->d_stage);
    if (p->d_stage_map) cudaFree(p->d_stage_map);
    p->d_panels = p->d_warp_word = p->d_unit_order = p->d_stage = p->d_stage_map = nullptr;

    if (p->d_xh) cudaFree(p->d_xh);
    if (p->d_yh) cudaFree(p->d_yh);
    p->d_partial = p->d_xh = p->d_yh = nullptr;
    for (int b = 0; b < 2; ++b) {
        if (p->d_xs[b]) cudaFree(p->d_xs[b]);
        if (p->d_ys[b]) cudaFree(p->d_ys[b]);
        p->d_xs[b] = p->d_ys[b] = nullptr;
        for (cudaEvent_t* e : {&p->ev_x[b], &p->ev_done[b], &p->ev_yout[b]}) {
            if (*e) cudaEventDestroy(*e);
            *e = nullptr;
        }
    }
    if (p->s_h2d) cudaStreamDestroy(p->s_h2d);
    if (p->s_d2h) cudaStreamDestroy(p->s_d2h);
    p->s_h2d = p->s_d2h = nullptr;
    for (auto& r : p->recs) { (void)r; }
    for (auto e : p->pool) cudaEventDestroy(e);
    p->pool.clear();
    p->recs.clear();
}

cudaEvent_t take_event(dasp_plan_s* p) {
    if (p->pool_used == p->pool.size()) {
        cudaEvent_t e;
        if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
        p->pool.push_back(e);
    }
    return p->pool[p->pool_used++];
}

// launch wrapper recording events when timing is on
template <typename F>
cudaError_t timed(dasp_plan_s* p, int kernel, cudaStream_t s, bool on, F&& launch) {
    if (!on) return launch();
    cudaEvent_t a = take_event(p), b = take_event(p);
    if (a) cudaEventRecord(a, s);
    cudaError_t e = launch();
    if (b) cudaEventRecord(b, s);
    if (a && b) p->recs.push_back({kernel, a, b});
    return e;
}

int64_t alg_bytes(const dasp_plan_s* p, bool beta) {
    const HostFormat& f = p->host;
    const int64_t s_v = f.geo.sv, s_x = sx(p->dtype), s_y = sy(p->dtype), s_a = sa(p->dtype);
    const int64_t nmp = f.nrb * 8;
    const int64_t nout = 64 * f.t13 + 32 * f.t4 + 64 * f.t22 + 128 * f.ts;
    int64_t b = 0;
    b += f.n_groups_padded * f.geo.G * (s_v + 4) + 2 * f.n_groups_padded * s_a + 8 * (f.row_long + 1) + 4 * f.row_long;
    b += (f.nnz_reg_new + f.nnz_irreg) * (s_v + 4) + 8 * (f.nrb + 1) + 8 * (nmp + 1) + 4 * nmp;
    b += f.nnz_short_new * (s_v + 4) + 4 * nout;
    b += 4 * f.n0;
    b += f.n * s_x + f.m * s_y * (beta ? 2 : 1);
    return b;
}

}  // namespace

extern "C" {

const char* dasp_version(void) { return "dasp-b200 0.1 (sm_100a)"; }

void dasp_options_default(dasp_options_t* o) {
    if (!o) return;
    o->device = 0;
    o->variant = DASP_VARIANT_CUDACORE;   // measured >= the MMA variant on B200
    o->validate = 1;
    o->keep_host = 0;
    o->medium_rb_per_warp = 0;
    o->num_threads = 0;
    o->panel_rows = 0;
    o->max_len = 256;
    o->threshold = 0.75;
    o->x_stage = 0;
}

const char* dasp_status_string(dasp_status_t s) {
    switch (s) {
    case DASP_OK: return "DASP_OK";
    case DASP_ERR_INVALID_ARG: return "DASP_ERR_INVALID_ARG";
    case DASP_ERR_INVALID_CSR: return "DASP_ERR_INVALID_CSR";
    case DASP_ERR_OUT_OF_MEMORY: return "DASP_ERR_OUT_OF_MEMORY";
    case DASP_ERR_CUDA: return "DASP_ERR_CUDA";
    case DASP_ERR_UNSUPPORTED: return "DASP_ERR_UNSUPPORTED";
    case DASP_ERR_INTERNAL: return "DASP_ERR_INTERNAL";
    }
    return "DASP_ERR_UNKNOWN";
}

}  // extern "C"

namespace {

// Launch metadata shared by host- and device-built plans: LOOP_NUM, the per-panel descriptors of
// the medium/short kernel, the long-unit schedule, and their device copies.  `panel_table` (host) is the DASP_ARR_PANELS content; `unit_first_col[u]` the
// column of the first element of long unit u (for the column-bucket schedule).
// narrow_slots[rb] = max(K nreg, longest row) = K nreg(rb) + irregular length of the row-block's
// first (longest) row: the slots each of its rows spans (rows are sorted by length, so within a
// panel this is non-increasing and the narrow row-blocks are a suffix).  rb_ptr [nrb+1] and
// irr_first [2 nrb] = irr_ptr[8 rb], irr_ptr[8 rb + 1], host copies.
std::vector<int32_t> narrow_slots(const HostFormat& f, const int64_t* rb_ptr, const int64_t* irr_first) {
    std::vector<int32_t> ns(static_cast<size_t>(f.nrb));
    const int64_t be = static_cast<int64_t>(f.geo.K) * 8;
    for (int64_t rb = 0; rb < f.nrb; ++rb)
        ns[rb] = static_cast<int32_t>((rb_ptr[rb + 1] - rb_ptr[rb]) / be * f.geo.K + (irr_first[2 * rb + 1] - irr_first[2 * rb]));
    return ns;
}

// x-window staging table (kernels.cuh StageEnt; north_star (3) "shared-memory or TMA staging where
// reuse exists"), from the host arrays of a host-built plan.  A main block is staged when all its
// warps are wide medium warps, the columns they gather span at most STAGE_MAX_SPAN tiles of STAGE_T
// columns, the referenced tiles (after merging the smallest gaps down to STAGE_RUNS runs) fill at
// most STAGE_MAX_SLOTS slots, and each staged column is gathered at least kStageReuse times on
// average (a 27-point stencil block: ~5.5; a power-law block: far below 1).  Tiles not wholly
// inside x are never staged.  Returns the staged block count; st[b].ntile = 0 for the others.
constexpr double kStageReuse = 2.0;
// automatic mode (x_stage = 0) stages a plan when a quarter of its main blocks qualify; 0: the
// automatic mode never stages (measured slower than the L1-served gathers)
#ifndef DASP_X_STAGE_AUTO
#define DASP_X_STAGE_AUTO 0
#endif
int64_t build_stage_table(const HostFormat& f, const std::vector<uint64_t>& warp_word,
                          const std::vector<dasp::PanelDesc>& desc, int rbw, int wide_il,
                          std::vector<dasp::StageEnt>& st, int* max_span, int* max_slots) {
    using dasp::STAGE_T;
    const int64_t nb = static_cast<int64_t>(warp_word.size() + dasp::WARPS_PER_BLOCK - 1) / dasp::WARPS_PER_BLOCK;
    st.assign(static_cast<size_t>(nb), dasp::StageEnt{});
    const int64_t* rbp = static_cast<const int64_t*>(f.arr[DASP_ARR_RB_PTR].ptr);
    const int64_t* ip = static_cast<const int64_t*>(f.arr[DASP_ARR_IRR_PTR].ptr);
    const int32_t* rc = static_cast<const int32_t*>(f.arr[DASP_ARR_REG_COL].ptr);
    const int32_t* ic = static_cast<const int32_t*>(f.arr[DASP_ARR_IRR_COL].ptr);
    if (!rbp || !ip || (!rc && f.nnz_reg_new) || (!ic && f.nnz_irreg)) return 0;
    const int64_t full_tiles = f.n / STAGE_T;   // tiles wholly inside x
    int64_t staged = 0;
    int mspan = 0, mslots = 0;
#pragma omp parallel for schedule(dynamic, 16) reduction(+ : staged) reduction(max : mspan, mslots)
    for (int64_t b = 0; b < nb; ++b) {
        std::vector<int64_t> rbs;
        bool ok = true;
        for (int k = 0; k < dasp::WARPS_PER_BLOCK && ok; ++k) {
            const size_t gi = static_cast<size_t>(b * dasp::WARPS_PER_BLOCK + k);
            if (gi >= warp_word.size() || warp_word[gi] == ~0ull) { ok = false; break; }
            const dasp::PanelDesc& d = desc[warp_word[gi] >> 32];
            const int64_t w = static_cast<int64_t>(warp_word[gi] & 0xffffffffu);
            if (w >= d.nmwd) { ok = false; break; }
            // the row-blocks of wide warp w (kernels.cu medium_warp)
            const int64_t rbe = d.rb0 + d.rbm, gw = w & ~int64_t(dasp::WARPS_PER_BLOCK - 1);
            const int64_t stg = wide_il ? std::min<int64_t>(dasp::WARPS_PER_BLOCK, d.nmwd - gw) : 1;
            const int64_t r0 = wide_il ? d.rb0 + gw * rbw + (w - gw) : d.rb0 + w * rbw;
            const int64_t r1 = std::min(r0 - (w - gw) * (wide_il != 0) + stg * rbw, rbe);
            for (int64_t rb = r0; rb < r1; rb += stg) rbs.push_back(rb);
        }
        if (!ok || rbs.empty()) continue;
        int64_t tmin = INT64_MAX, tmax = -1, gathers = 0;
        auto each_col = [&](auto&& fn) {
            for (int64_t rb : rbs) {
                for (int64_t e = rbp[rb]; e < rbp[rb + 1]; ++e) fn(rc[e]);
                for (int64_t e = ip[8 * rb]; e < ip[8 * rb + 8]; ++e) fn(ic[e]);
            }
        };
        each_col([&](int32_t c) {
            if (c < 0 || c / STAGE_T >= full_tiles) return;
            const int64_t t = c / STAGE_T;
            tmin = std::min(tmin, t); tmax = std::max(tmax, t); ++gathers;
        });
        if (tmax < 0 || tmax - tmin + 1 > dasp::STAGE_MAX_SPAN) continue;
        const int span = static_cast<int>(tmax - tmin + 1);
        std::vector<uint8_t> used(static_cast<size_t>(span), 0);
        each_col([&](int32_t c) {
            if (c < 0 || c / STAGE_T >= full_tiles) return;
            used[static_cast<size_t>(c / STAGE_T - tmin)] = 1;
        });
        std::vector<std::pair<int, int>> runs;   // [t0, t1)
        for (int i = 0; i < span; ++i) {
            if (!used[i]) continue;
            if (!runs.empty() && runs.back().second == i) runs.back().second = i + 1;
            else runs.push_back({i, i + 1});
        }
        int64_t distinct = 0;
        for (auto& r : runs) distinct += r.second - r.first;
        while (static_cast<int>(runs.size()) > dasp::STAGE_RUNS) {   // merge the smallest gap
            size_t g = 0;
            for (size_t k = 1; k + 1 < runs.size(); ++k)
                if (runs[k + 1].first - runs[k].second < runs[g + 1].first - runs[g].second) g = k;
            runs[g].second = runs[g + 1].second;
            runs.erase(runs.begin() + static_cast<std::ptrdiff_t>(g) + 1);
        }
        int slots = 0;
        for (auto& r : runs) slots += r.second - r.first;
        if (slots > dasp::STAGE_MAX_SLOTS || static_cast<double>(gathers) < kStageReuse * distinct * STAGE_T) continue;
        dasp::StageEnt& e = st[static_cast<size_t>(b)];
        e.xbase = static_cast<int32_t>(tmin * STAGE_T);
        e.ntile = span;
        e.meta = static_cast<int32_t>(runs.size()) | (slots << 8);
        for (size_t r = 0; r < runs.size(); ++r) {
            e.run_t0[r] = static_cast<uint16_t>(runs[r].first);
            e.run_nt[r] = static_cast<uint16_t>(runs[r].second - runs[r].first);
        }
        ++staged;
        mspan = std::max(mspan, span);
        mslots = std::max(mslots, slots);
    }
    *max_span = mspan;
    *max_slots = mslots;
    return staged;
}

// mid (two-lanes-per-row) row-blocks: rows spanning at most mid_max_slots(K) slots; experiment knob
// DASP_MID_MUL_F16 (FP16, K = 8): the multiple of K up to which row-blocks go to the mid path
#ifndef DASP_MID_MUL_F16
#define DASP_MID_MUL_F16 4
#endif
inline int mid_slots(int K) { return K == 8 ? DASP_MID_MUL_F16 * K : dasp::mid_max_slots(K); }

dasp_status_t setup_launch(dasp_plan_s* p, const dasp_options_t& o, const int64_t* panel_table,
                           const std::vector<int32_t>& unit_first_col, const std::vector<int32_t>& nslots) {
    HostFormat& f = p->host;
    p->rbw = o.medium_rb_per_warp > 0 ? o.medium_rb_per_warp : auto_rbw(f.row_medium, f.nnz_medium, f.sumsq_medium);
    // a block's wide medium warps interleave their row-blocks when the medium rows are ragged
    // (LOOP_NUM 4 or less): C5 +1 % (FP64) .. +7 % (FP16), C3 neutral; uniform stencil rows
    // (LOOP_NUM 8) keep contiguous ranges (C2+ -2 % .. -5 % interleaved; profiles/r01d/wide_interleave.jsonl)
    p->wide_il = p->rbw <= 4 ? 1 : 0;
    p->narrow_il = DASP_NARROW_IL;
    int64_t nrw = static_cast<int64_t>(nslots.size()) == f.nrb ? dasp::narrow_rb_per_warp(p->dtype) : 0;
    // small matrices (LOOP_NUM 1) keep more warps in flight: one pass of 4 row-blocks
    if (nrw > 4 && p->rbw <= 1) nrw = 4;
    p->nrw = static_cast<int>(nrw);
    p->rb_mid = p->rb_narrow = 0;
    std::vector<dasp::PanelDesc> desc(static_cast<size_t>(f.n_panels));
    std::vector<int64_t> panel_warps(static_cast<size_t>(f.n_panels));
    int64_t blk = 0;
    // FP16 with the CUDA-core default: the main kernel runs its 5-block / 48-register instantiation
    // unless wide medium row-blocks (the register-hungry path, which spills there) are the majority
    // of the plan's row-blocks: C2 FP16 -13 %, C2+ -15 %, C6 -5 %, C3 +-0; C5 (wide rows) +4 % and
    // keeps 4 blocks (profiles/r02/f16_occupancy5.jsonl)
    int64_t wide_rbs = 0;
    for (int64_t q = 0; q < f.n_panels; ++q) {
        const int64_t* e = panel_table + q * dasp::PANEL_FIELDS;
        int64_t rbm = e[5];
        if (nrw > 0)
            while (rbm > 0 && nslots[e[4] + rbm - 1] <= mid_slots(f.geo.K)) --rbm;
        wide_rbs += rbm;
    }
    p->occ5 = p->dtype == DASP_R_16F && p->variant == DASP_VARIANT_CUDACORE && 4 * wide_rbs <= f.nrb;
    p->tpw = dasp::short_tiles_per_warp(p->dtype, p->occ5);
    for (int64_t q = 0; q < f.n_panels; ++q) {
        const int64_t* e = panel_table + q * dasp::PANEL_FIELDS;
        dasp::PanelDesc& d = desc[q];
        d.blk0 = blk;
        d.unit0 = e[2]; d.nunits = e[3]; d.rb0 = e[4]; d.nrb = e[5];
        d.rbn = d.nrb;
        if (nrw > 0)
            while (d.rbn > 0 && nslots[d.rb0 + d.rbn - 1] <= dasp::narrow_max_slots(f.geo.K)) --d.rbn;
        d.rbm = d.rbn;
        if (nrw > 0)
            while (d.rbm > 0 && nslots[d.rb0 + d.rbm - 1] <= mid_slots(f.geo.K)) --d.rbm;
        d.nmwd = (d.rbm + p->rbw - 1) / p->rbw;
        d.nmwm = d.nmwd + (nrw > 0 ? (d.rbn - d.rbm + nrw - 1) / nrw : 0);
        d.nmw = d.nmwm + (nrw > 0 ? (d.nrb - d.rbn + nrw - 1) / nrw : 0);
        p->rb_mid += d.rbn - d.rbm;
        p->rb_narrow += d.nrb - d.rbn;
        d.tile0 = e[6]; d.t13 = e[7]; d.t4 = e[8]; d.t22 = e[9]; d.ts = e[10]; d.out0 = e[11];
        const int64_t tpw = p->tpw;
        const int64_t warps = d.nmw + (d.t13 + d.t4 + d.t22 + d.ts + tpw - 1) / tpw;   // long units: own kernel
        panel_warps[q] = warps;
        blk += (warps + dasp::WARPS_PER_BLOCK - 1) / dasp::WARPS_PER_BLOCK;
    }
    // warp table of the main kernel.  Heavy warps first: a panel's first warps hold its longest
    // medium row-blocks (rows are length-sorted), which walk many chunks one round trip after the
    // other and finish long after the panel's other warps; dispatching them for every panel at the
    // start of the grid overlaps them with everything else instead of leaving them as the tail of
    // the launch.  Panels are packed back to back (DASP_PACK_WARPS) or each padded to whole blocks.
    std::vector<uint64_t> warp_word;
    {
        const int64_t heavy = (f.n_panels > 1 ? (p->dtype == DASP_R_16F ? DASP_HEAVY_FIRST_F16 : DASP_HEAVY_FIRST) : 0) *
                              dasp::WARPS_PER_BLOCK;
        auto emit = [&](int64_t q, int64_t w0, int64_t w1) {
            for (int64_t w = w0; w < w1; ++w) warp_word.push_back((static_cast<uint64_t>(q) << 32) | static_cast<uint64_t>(w));
            if (!DASP_PACK_WARPS)
                while (warp_word.size() % dasp::WARPS_PER_BLOCK) warp_word.push_back(~0ull);
        };
        for (int64_t q = 0; q < f.n_panels; ++q) emit(q, 0, std::min(heavy, panel_warps[q]));
        for (int64_t q = 0; q < f.n_panels; ++q) emit(q, std::min(heavy, panel_warps[q]), panel_warps[q]);
    }
    p->n_mwarps = static_cast<int64_t>(warp_word.size());
    p->blocks = (p->n_mwarps + dasp::WARPS_PER_BLOCK - 1) / dasp::WARPS_PER_BLOCK;
    p->n_units = f.n_groups_padded / f.geo.UG;

    // long-unit execution order (a launch schedule, not part of the format): inside each panel
    // the units run bucketed by the column of their first element, so that the warps in flight
    // gather from ~1/kColBuckets of x at a time instead of all of it (long rows' columns are
    // sorted, so a unit covers a narrow column range).  Partials are per group and summed in
    // group order by the finish kernel: the result is bitwise independent of this order.
    std::vector<int32_t> unit_order(static_cast<size_t>(p->n_units));
    {
        // memory order when there is no column space to bucket (n = 0)
        const int mode = f.n > 0 ? DASP_LONG_ORDER : 0;
        std::vector<dasp::PanelDesc> all(1);   // global order: one pseudo-panel over every unit
        all[0].unit0 = 0;
        all[0].nunits = p->n_units;
        for (const auto& d : (mode == 2 ? all : desc)) {
            std::vector<int64_t> cnt(kColBuckets + 1, 0);
            auto bucket = [&](int64_t u) {
                const int32_t c = unit_first_col[u];
                return c < 0 ? kColBuckets - 1 : static_cast<int>(static_cast<int64_t>(c) * kColBuckets / f.n);
            };
            if (mode == 0) {
                for (int64_t w = 0; w < d.nunits; ++w) unit_order[d.unit0 + w] = static_cast<int32_t>(d.unit0 + w);
                continue;
            }
            for (int64_t w = 0; w < d.nunits; ++w) ++cnt[bucket(d.unit0 + w) + 1];
            for (int b = 0; b < kColBuckets; ++b) cnt[b + 1] += cnt[b];
            for (int64_t w = 0; w < d.nunits; ++w) unit_order[d.unit0 + cnt[bucket(d.unit0 + w)]++] = static_cast<int32_t>(d.unit0 + w);
        }
    }
    // x-window staging (x_stage: 0 automatic -- on when at least a quarter of the main blocks
    // qualify --, 1 off, 2 wherever a block qualifies); host-built CUDA-core plans only
    p->stage_blocks = 0;
    p->stage_smem = p->stage_map_bytes = 0;
    std::vector<dasp::StageEnt> stab;
    const bool want_stage = o.x_stage == 2 || (o.x_stage == 0 && DASP_X_STAGE_AUTO);
    if (want_stage && p->variant == DASP_VARIANT_CUDACORE && f.arr[DASP_ARR_REG_COL].ptr && p->blocks > 0) {
        int mspan = 0, mslots = 0;
        const int64_t ns = build_stage_table(f, warp_word, desc, p->rbw, p->wide_il, stab, &mspan, &mslots);
        if (ns > 0 && (o.x_stage == 2 || (DASP_X_STAGE_AUTO && 4 * ns >= p->blocks))) {
            p->stage_blocks = ns;
            p->stage_map_bytes = (mspan + 127) / 128 * 128;
            p->stage_smem = p->stage_map_bytes + mslots * dasp::STAGE_T * sx(p->dtype);
        }
    }
    if (p->device < 0) return DASP_OK;

    auto upload = [&](void** dst, const void* src, size_t bytes) -> dasp_status_t {
        if (cudaMalloc(dst, std::max<size_t>(bytes, 16)) != cudaSuccess) return DASP_ERR_OUT_OF_MEMORY;
        p->device_bytes += static_cast<int64_t>(bytes);
        if (bytes && cudaMemcpy(*dst, src, bytes, cudaMemcpyHostToDevice) != cudaSuccess) return DASP_ERR_CUDA;
        return DASP_OK;
    };
    const int64_t pb = std::max<int64_t>(f.n_groups_padded, 1) * sa(p->dtype);
    if (cudaMalloc(&p->d_partial, static_cast<size_t>(pb)) != cudaSuccess) return DASP_ERR_OUT_OF_MEMORY;
    p->device_bytes += pb;
    dasp_status_t st;
    if ((st = upload(&p->d_panels, desc.data(), desc.size() * sizeof(dasp::PanelDesc))) != DASP_OK) return st;
    if ((st = upload(&p->d_warp_word, warp_word.data(), warp_word.size() * 8)) != DASP_OK) return st;
    if ((st = upload(&p->d_unit_order, unit_order.data(), unit_order.size() * 4)) != DASP_OK) return st;
    if (p->stage_blocks > 0) {
        // tile maps: span tile -> slot (runs back to back), 0xff elsewhere; 16-byte aligned per block
        std::vector<unsigned char> maps;
        for (auto& e : stab) {
            if (e.ntile <= 0) continue;
            e.map16 = static_cast<int32_t>(maps.size() / 16);
            const size_t at = maps.size();
            maps.resize(at + ((static_cast<size_t>(e.ntile) + 15) & ~size_t(15)), 0xff);
            int slot = 0;
            for (int r = 0; r < (e.meta & 0xff); ++r)
                for (int k = 0; k < e.run_nt[r]; ++k) maps[at + e.run_t0[r] + k] = static_cast<unsigned char>(slot++);
        }
        if ((st = upload(&p->d_stage, stab.data(), stab.size() * sizeof(dasp::StageEnt))) != DASP_OK) return st;
        if ((st = upload(&p->d_stage_map, maps.data(), maps.size())) != DASP_OK) return st;
    }

    return DASP_OK;
}

dasp_status_t check_create_args(dasp_plan_t* plan_out, int64_t m, int64_t n, int64_t nnz, const void* row_ptr,
                                const void* col_idx, const void* val, dasp_dtype_t dtype, const dasp_options_t* opts,
                                dasp_options_t& o) {
    if (!plan_out) return DASP_ERR_INVALID_ARG;
    *plan_out = nullptr;
    if (m < 0 || n < 0 || nnz < 0 || n > 0x7fffffffLL || m > 0x7fffffffLL) return DASP_ERR_INVALID_ARG;
    if (dtype != DASP_R_64F && dtype != DASP_R_16F && dtype != DASP_R_32F) return DASP_ERR_INVALID_ARG;
    if (!row_ptr || (nnz > 0 && (!col_idx || !val))) return DASP_ERR_INVALID_ARG;
    dasp_options_default(&o);
    if (opts) o = *opts;
    if (o.variant != DASP_VARIANT_MMA && o.variant != DASP_VARIANT_CUDACORE) o.variant = DASP_VARIANT_CUDACORE;
    return DASP_OK;
}

// Automatic panel size (R28).  Default 2^20 rows.  Ragged medium lengths (coefficient of variation >=
// 0.5) take 8192-row panels -- a row-block's 8 length-sorted rows, and a block's row-blocks, then come
// from within 8192 original rows, so their local x windows overlap in L1 and the gathers issue fewer
// L2 requests -- except heavy-tailed lengths (cv >= 1) in FP64 / FP32, whose main kernel is latency-
// bound and pays the small panels' fragmentation instead (profiles/r02/panel_size_small*.jsonl:
// 8192 rows C5 FP64 -4.8 %, FP32 -8.6 %, FP16 -5.9 %, C3 FP16 -5.3 %; C3 FP64 +2 %, stencils +0.5..+2.5 %).
constexpr int64_t kSmallPanelRows = 8192;
int64_t auto_panel_rows(int dtype, int64_t cnt, int64_t sum, int64_t sumsq) {
    if (cnt < 2) return kAutoPanelRows;
    const double mean = static_cast<double>(sum) / static_cast<double>(cnt);
    const double var = static_cast<double>(sumsq) / static_cast<double>(cnt) - mean * mean;
    const double cv = var > 0 ? std::sqrt(var) / mean : 0.0;
    if (cv >= 0.5 && (dtype == DASP_R_16F || cv < 1.0)) return kSmallPanelRows;
    return kAutoPanelRows;
}
int64_t resolve_panel_rows(const dasp_options_t& o, int dtype, int64_t cnt, int64_t sum, int64_t sumsq) {
    // -1 one panel (the paper's global format); 0 automatic; > 0 as given
    return o.panel_rows == 0 ? auto_panel_rows(dtype, cnt, sum, sumsq) : (o.panel_rows < 0 ? 0 : o.panel_rows);
}
// medium-class length statistics of a host row_ptr (automatic panel size)
void host_medium_stats(const int64_t* rp, int64_t m, int64_t max_len, int64_t* cnt, int64_t* sum, int64_t* sumsq) {
    int64_t c = 0, s1 = 0, s2 = 0;
#pragma omp parallel for schedule(static) reduction(+ : c, s1, s2)
    for (int64_t i = 0; i < m; ++i) {
        const int64_t L = rp[i + 1] - rp[i];
        if (L >= dasp::MIN_MEDIUM_LEN && L <= max_len) { ++c; s1 += L; s2 += L * L; }
    }
    *cnt = c; *sum = s1; *sumsq = s2;
}

dasp_status_t fail(dasp_plan_s* p, dasp_status_t st) {
    if (p->device >= 0) {
        DeviceGuard guard(p->device);
        free_device(p);
    }
    p->host.release();
    delete p;
    return st;
}

}  // namespace

extern "C" {

dasp_status_t dasp_plan_create(dasp_plan_t* plan_out, int64_t m, int64_t n, int64_t nnz, const int64_t* row_ptr,
                               const int32_t* col_idx, const void* val, dasp_dtype_t dtype, const dasp_options_t* opts) {
    dasp_options_t o;
    dasp_status_t st = check_create_args(plan_out, m, n, nnz, row_ptr, col_idx, val, dtype, opts, o);
    if (st != DASP_OK) return st;
    if (o.validate && row_ptr[m] != nnz) return DASP_ERR_INVALID_CSR;

    dasp_plan_s* p = new (std::nothrow) dasp_plan_s;
    if (!p) return DASP_ERR_OUT_OF_MEMORY;
    p->dtype = dtype;
    p->device = o.device;
    p->variant = o.variant;
    p->keep_host = o.keep_host != 0 || o.device < 0;

    auto t0 = std::chrono::steady_clock::now();
    int64_t mc = 0, ms = 0, mq = 0;
    if (o.panel_rows == 0) host_medium_stats(row_ptr, m, o.max_len > 0 ? o.max_len : dasp::MAX_LEN, &mc, &ms, &mq);
    int bst = dasp::build_format(p->host, dtype, m, n, row_ptr, col_idx, val, o.num_threads, o.validate != 0,
                                 resolve_panel_rows(o, dtype, mc, ms, mq), o.max_len, o.threshold);
    auto t1 = std::chrono::steady_clock::now();
    p->build_ms = std::chrono::duration<double, std::milli>(t1 - t0).count();
    if (bst != DASP_OK) {
        delete p;
        return static_cast<dasp_status_t>(bst);
    }
    HostFormat& f = p->host;
    for (int a = 0; a < DASP_ARR_COUNT; ++a) p->bytes[a] = f.arr[a].bytes;
    std::vector<int32_t> first_col(static_cast<size_t>(f.n_groups_padded / f.geo.UG));
    {
        const int32_t* lc = static_cast<const int32_t*>(f.arr[DASP_ARR_LONG_COL].ptr);
        const int64_t ue = static_cast<int64_t>(f.geo.UG) * f.geo.G;
        for (size_t u = 0; u < first_col.size(); ++u) first_col[u] = lc[u * ue];
    }
    std::vector<int64_t> irr_first(static_cast<size_t>(2 * f.nrb));
    {
        const int64_t* ip = static_cast<const int64_t*>(f.arr[DASP_ARR_IRR_PTR].ptr);
        for (int64_t rb = 0; rb < f.nrb; ++rb) { irr_first[2 * rb] = ip[8 * rb]; irr_first[2 * rb + 1] = ip[8 * rb + 1]; }
    }
    const std::vector<int32_t> nslots =
        f.nrb ? narrow_slots(f, static_cast<const int64_t*>(f.arr[DASP_ARR_RB_PTR].ptr), irr_first.data()) : std::vector<int32_t>();
    std::unique_ptr<DeviceGuard> guard;
    if (p->device >= 0) guard.reset(new DeviceGuard(p->device));
    st = setup_launch(p, o, static_cast<const int64_t*>(f.arr[DASP_ARR_PANELS].ptr), first_col, nslots);
    if (st != DASP_OK) return fail(p, st);
    if (p->device >= 0) {
        for (int a = 0; a < DASP_ARR_COUNT; ++a) {
            if (p->bytes[a] == 0) continue;
            // 256 B alignment from cudaMalloc keeps every lane's 16/32 B vector load aligned
            if (cudaMalloc(&p->d[a], static_cast<size_t>(p->bytes[a] + kAllocPad)) != cudaSuccess)
                return fail(p, DASP_ERR_OUT_OF_MEMORY);
            p->device_bytes += p->bytes[a];
        }
        auto u0 = std::chrono::steady_clock::now();
        for (int a = 0; a < DASP_ARR_COUNT; ++a) {
            if (p->bytes[a] == 0) continue;
            if (cudaMemcpy(p->d[a], f.arr[a].ptr, static_cast<size_t>(p->bytes[a]), cudaMemcpyHostToDevice) != cudaSuccess)
                return fail(p, DASP_ERR_CUDA);
        }
        auto u1 = std::chrono::steady_clock::now();
        p->upload_ms = std::chrono::duration<double, std::milli>(u1 - u0).count();
        if (!p->keep_host) f.release();
    }
    *plan_out = p;
    return DASP_OK;
}

dasp_status_t dasp_plan_create_device(dasp_plan_t* plan_out, int64_t m, int64_t n, int64_t nnz,
                                      const int64_t* d_row_ptr, const int32_t* d_col_idx, const void* d_val,
                                      dasp_dtype_t dtype, const dasp_options_t* opts, void* stream) {
    dasp_options_t o;
    dasp_status_t st = check_create_args(plan_out, m, n, nnz, d_row_ptr, d_col_idx, d_val, dtype, opts, o);
    if (st != DASP_OK) return st;
    if (o.device < 0) return DASP_ERR_INVALID_ARG;
    dasp_plan_s* p = new (std::nothrow) dasp_plan_s;
    if (!p) return DASP_ERR_OUT_OF_MEMORY;
    p->dtype = dtype;
    p->device = o.device;
    p->variant = o.variant;
    p->keep_host = false;
    DeviceGuard guard(p->device);
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    auto t0 = std::chrono::steady_clock::now();
    int64_t mc = 0, ms = 0, mq = 0;
    if (o.panel_rows == 0 &&
        dasp::medium_length_stats(d_row_ptr, m, o.max_len > 0 ? o.max_len : dasp::MAX_LEN, &mc, &ms, &mq, s) != cudaSuccess) {
        delete p;
        return DASP_ERR_CUDA;
    }
    int bst = dasp::build_format_device(p->host, p->d, dtype, m, n, nnz, d_row_ptr, d_col_idx, d_val, o.validate != 0,
                                        resolve_panel_rows(o, dtype, mc, ms, mq), o.max_len, o.threshold, s);
    auto t1 = std::chrono::steady_clock::now();
    p->build_ms = std::chrono::duration<double, std::milli>(t1 - t0).count();
    if (bst != DASP_OK) {
        delete p;
        return static_cast<dasp_status_t>(bst);
    }
    HostFormat& f = p->host;
    for (int a = 0; a < DASP_ARR_COUNT; ++a) {
        p->bytes[a] = f.arr[a].bytes;
        p->device_bytes += p->bytes[a];
    }
    // first column of every long unit, gathered on the device
    std::vector<int32_t> first_col(static_cast<size_t>(f.n_groups_padded / f.geo.UG));
    if (!first_col.empty() &&
        dasp::gather_unit_first_col(static_cast<const int32_t*>(p->d[DASP_ARR_LONG_COL]), f.geo.UG * f.geo.G,
                                    static_cast<int64_t>(first_col.size()), first_col.data(), s) != cudaSuccess)
        return fail(p, DASP_ERR_CUDA);
    std::vector<int32_t> nslots;
    if (f.nrb > 0) {   // rb_ptr and irr_ptr[8 rb .. 8 rb + 1] back from the device
        std::vector<int64_t> rbp(static_cast<size_t>(f.nrb + 1)), irr_first(static_cast<size_t>(2 * f.nrb));
        if (cudaMemcpyAsync(rbp.data(), p->d[DASP_ARR_RB_PTR], rbp.size() * 8, cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaMemcpy2DAsync(irr_first.data(), 16, p->d[DASP_ARR_IRR_PTR], 64, 16, static_cast<size_t>(f.nrb),
                              cudaMemcpyDeviceToHost, s) != cudaSuccess ||
            cudaStreamSynchronize(s) != cudaSuccess)
            return fail(p, DASP_ERR_CUDA);
        nslots = narrow_slots(f, rbp.data(), irr_first.data());
    }
    st = setup_launch(p, o, f.panel_table.data(), first_col, nslots);
    if (st != DASP_OK) return fail(p, st);
    *plan_out = p;
    return DASP_OK;
}

static dasp_status_t spmv_impl(dasp_plan_t p, const void* x, void* y, const dasp::ExtraDst& extra, double alpha,
                               double beta, void* stream, int32_t variant);

dasp_status_t dasp_spmv_ex(dasp_plan_t p, const void* x, void* y, double alpha, double beta, void* stream, int32_t variant) {
    dasp::ExtraDst none{};
    none.n = 0;
    return spmv_impl(p, x, y, none, alpha, beta, stream, variant);
}

dasp_status_t dasp_spmv_scatter(dasp_plan_t p, const void* x, void* const* y_dst, int32_t ndst, double alpha,
                                double beta, void* stream) {
    if (!p || !y_dst || ndst < 1 || ndst > dasp::MAX_EXTRA_DST + 1) return DASP_ERR_INVALID_ARG;
    dasp::ExtraDst ex{};
    ex.n = ndst - 1;
    for (int d = 1; d < ndst; ++d) {
        if (!y_dst[d] || y_dst[d] == x) return DASP_ERR_INVALID_ARG;
        ex.ptr[d - 1] = y_dst[d];
    }
    return spmv_impl(p, x, y_dst[0], ex, alpha, beta, stream, DASP_VARIANT_DEFAULT);
}

static dasp_status_t spmv_impl(dasp_plan_t p, const void* x, void* y, const dasp::ExtraDst& extra, double alpha,
                               double beta, void* stream, int32_t variant) {
    if (!p) return DASP_ERR_INVALID_ARG;
    if (p->device < 0) return DASP_ERR_UNSUPPORTED;
    const HostFormat& f = p->host;
    if (f.m == 0) return DASP_OK;
    if (!y) return DASP_ERR_INVALID_ARG;
    if (x == y) return DASP_ERR_INVALID_ARG;
    if (variant == DASP_VARIANT_DEFAULT) variant = p->variant;
    if (variant != DASP_VARIANT_MMA && variant != DASP_VARIANT_CUDACORE) return DASP_ERR_INVALID_ARG;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    DeviceGuard guard(p->device);
    const bool on = p->timing_calls < p->timing_cap;
    if (on) ++p->timing_calls;
    cudaError_t e;
    if (alpha == 0.0) {  // quick path: y = beta*y
        if (beta == 1.0 && extra.n == 0) return DASP_OK;
        e = timed(p, DASP_K_SCALE, s, on, [&] { return dasp::launch_scale(y, f.m, beta, p->dtype, s, extra); });
        return e == cudaSuccess ? DASP_OK : DASP_ERR_CUDA;
    }
    if (!x && f.n > 0) return DASP_ERR_INVALID_ARG;
    dasp::MainParams mp{};
    mp.long_val = p->d[DASP_ARR_LONG_VAL];
    mp.long_col = static_cast<const int32_t*>(p->d[DASP_ARR_LONG_COL]);
    mp.partial = p->d_partial;
    mp.rb_ptr = static_cast<const int64_t*>(p->d[DASP_ARR_RB_PTR]);
    mp.reg_val = p->d[DASP_ARR_REG_VAL];
    mp.reg_col = static_cast<const int32_t*>(p->d[DASP_ARR_REG_COL]);
    mp.irr_ptr = static_cast<const int64_t*>(p->d[DASP_ARR_IRR_PTR]);
    mp.irr_val = p->d[DASP_ARR_IRR_VAL];
    mp.irr_col = static_cast<const int32_t*>(p->d[DASP_ARR_IRR_COL]);
    mp.med_out = static_cast<const int32_t*>(p->d[DASP_ARR_MED_OUT]);
    mp.short_val = p->d[DASP_ARR_SHORT_VAL];
    mp.short_col = static_cast<const int32_t*>(p->d[DASP_ARR_SHORT_COL]);
    mp.short_out = static_cast<const int32_t*>(p->d[DASP_ARR_SHORT_OUT]);
    mp.x = x;
    mp.y = y;
    mp.alpha = alpha;
    mp.beta = beta;
    mp.panels = static_cast<const dasp::PanelDesc*>(p->d_panels);
    mp.warp_word = static_cast<const uint64_t*>(p->d_warp_word);
    mp.n_mwarps = p->n_mwarps;
    mp.unit_order = static_cast<const int32_t*>(p->d_unit_order);
    mp.rbw = p->rbw;
    mp.wide_il = p->wide_il;
    mp.narrow_il = p->narrow_il;
    mp.nrw = p->nrw;
    mp.extra = extra;
    mp.class_mask = DASP_CLASS_MASK;
    mp.tpw = p->tpw;
    const int64_t n0 = (beta == 1.0 && extra.n == 0) ? 0 : f.n0;   // scatter mode must still copy them
    mp.group_ptr = static_cast<const int64_t*>(p->d[DASP_ARR_GROUP_PTR]);
    mp.long_out = static_cast<const int32_t*>(p->d[DASP_ARR_LONG_OUT]);
    mp.empty_rows = static_cast<const int32_t*>(p->d[DASP_ARR_EMPTY_ROWS]);
    if (p->n_units > 0) {
        e = timed(p, DASP_K_LONG, s, on, [&] { return dasp::launch_long(mp, p->dtype, variant, p->n_units, s); });
        if (e != cudaSuccess) return DASP_ERR_CUDA;
    }
    // long-row phase 2 and the empty rows run as the first warps of the main kernel (the long
    // kernel before it has written every partial)
    mp.row_long = f.row_long;
    mp.n0 = n0;
    mp.fin_warps = dasp::finish_warps(mp.row_long, n0);
    const int64_t fin_blocks = (mp.fin_warps + dasp::WARPS_PER_BLOCK - 1) / dasp::WARPS_PER_BLOCK;
    // x-window staging: CUDA-core calls without scatter destinations whose x is 16-byte aligned
    // (cp.async.bulk source alignment); any other call runs the unstaged instantiation
    int stage_smem = 0;
    if (p->d_stage && variant == DASP_VARIANT_CUDACORE && extra.n == 0 && (reinterpret_cast<uintptr_t>(x) & 15) == 0) {
        mp.stage = static_cast<const dasp::StageEnt*>(p->d_stage);
        mp.stage_map = static_cast<const unsigned char*>(p->d_stage_map);
        mp.stage_map_bytes = p->stage_map_bytes;
        stage_smem = p->stage_smem;
    }
    e = timed(p, DASP_K_MAIN, s, on, [&] {
        return dasp::launch_main(mp, p->dtype, variant, p->blocks + fin_blocks, s, p->occ5, stage_smem);
    });
    if (e != cudaSuccess) return DASP_ERR_CUDA;
    return DASP_OK;
}

dasp_status_t dasp_spmv(dasp_plan_t p, const void* x, void* y, double alpha, double beta, void* stream) {
    return dasp_spmv_ex(p, x, y, alpha, beta, stream, DASP_VARIANT_DEFAULT);
}

// Host -> device copy of a caller's buffer (copy engine; SM loads over UVA measured slower inside the
// pipelined e2e step)
static cudaError_t copy_h2d(void* dst, const void* src, size_t bytes, cudaStream_t s) {
    return cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, s);
}

dasp_status_t dasp_spmv_host(dasp_plan_t p, const void* x_host, void* y_host, double alpha, double beta, void* stream) {
    if (!p) return DASP_ERR_INVALID_ARG;
    if (p->device < 0) return DASP_ERR_UNSUPPORTED;
    const HostFormat& f = p->host;
    if (f.m == 0) return DASP_OK;
    if (!y_host || (!x_host && f.n > 0 && alpha != 0.0)) return DASP_ERR_INVALID_ARG;
    DeviceGuard guard(p->device);
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const size_t xb = static_cast<size_t>(f.n) * sx(p->dtype), yb = static_cast<size_t>(f.m) * sy(p->dtype);
    if (!p->d_xh && xb && cudaMalloc(&p->d_xh, xb) != cudaSuccess) return DASP_ERR_OUT_OF_MEMORY;
    if (!p->d_yh && cudaMalloc(&p->d_yh, yb) != cudaSuccess) return DASP_ERR_OUT_OF_MEMORY;
    if (xb && alpha != 0.0 && copy_h2d(p->d_xh, x_host, xb, s) != cudaSuccess) return DASP_ERR_CUDA;
    if (beta != 0.0 && copy_h2d(p->d_yh, y_host, yb, s) != cudaSuccess) return DASP_ERR_CUDA;
    dasp_status_t st = dasp_spmv(p, p->d_xh, p->d_yh, alpha, beta, stream);
    if (st != DASP_OK) return st;
    if (cudaMemcpyAsync(y_host, p->d_yh, yb, cudaMemcpyDeviceToHost, s) != cudaSuccess) return DASP_ERR_CUDA;
    return cudaStreamSynchronize(s) == cudaSuccess ? DASP_OK : DASP_ERR_CUDA;
}

dasp_status_t dasp_spmv_host_stream(dasp_plan_t p, const void* x_host, int64_t ldx, void* y_host, int64_t ldy,
                                    int64_t nvec, double alpha, double beta, void* stream) {
    if (!p || nvec < 0) return DASP_ERR_INVALID_ARG;
    if (p->device < 0) return DASP_ERR_UNSUPPORTED;
    const HostFormat& f = p->host;
    if (f.m == 0 || nvec == 0) return DASP_OK;
    const bool need_x = f.n > 0 && alpha != 0.0;
    if (!y_host || (!x_host && need_x)) return DASP_ERR_INVALID_ARG;
    if ((need_x && ldx < f.n) || ldy < f.m) return DASP_ERR_INVALID_ARG;
    DeviceGuard guard(p->device);
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const size_t xb = static_cast<size_t>(f.n) * sx(p->dtype), yb = static_cast<size_t>(f.m) * sy(p->dtype);
    const size_t xs = static_cast<size_t>(ldx) * sx(p->dtype), ys = static_cast<size_t>(ldy) * sy(p->dtype);
    for (int b = 0; b < 2; ++b) {
        if (!p->d_xs[b] && xb && cudaMalloc(&p->d_xs[b], xb) != cudaSuccess) return DASP_ERR_OUT_OF_MEMORY;
        if (!p->d_ys[b] && cudaMalloc(&p->d_ys[b], yb) != cudaSuccess) return DASP_ERR_OUT_OF_MEMORY;
        for (cudaEvent_t* e : {&p->ev_x[b], &p->ev_done[b], &p->ev_yout[b]})
            if (!*e && cudaEventCreateWithFlags(e, cudaEventDisableTiming) != cudaSuccess) return DASP_ERR_CUDA;
    }
    if (!p->s_h2d && cudaStreamCreateWithFlags(&p->s_h2d, cudaStreamNonBlocking) != cudaSuccess) return DASP_ERR_CUDA;
    if (!p->s_d2h && cudaStreamCreateWithFlags(&p->s_d2h, cudaStreamNonBlocking) != cudaSuccess) return DASP_ERR_CUDA;
    // order the copy streams after everything already enqueued on `stream`
    if (cudaEventRecord(p->ev_yout[0], s) != cudaSuccess || cudaEventRecord(p->ev_yout[1], s) != cudaSuccess ||
        cudaEventRecord(p->ev_done[0], s) != cudaSuccess || cudaEventRecord(p->ev_done[1], s) != cudaSuccess)
        return DASP_ERR_CUDA;
    const char* xh = static_cast<const char*>(x_host);
    char* yh = static_cast<char*>(y_host);
    bool ok = true;
    for (int64_t j = 0; j < nvec && ok; ++j) {
        const int b = static_cast<int>(j & 1);
        // h2d: vector j into slot b once SpMV j-2 has read it (and, for beta != 0, y_j once y_{j-2} left)
        ok = ok && cudaStreamWaitEvent(p->s_h2d, p->ev_done[b], 0) == cudaSuccess;
        if (need_x) ok = ok && copy_h2d(p->d_xs[b], xh + j * xs, xb, p->s_h2d) == cudaSuccess;
        if (beta != 0.0) {
            ok = ok && cudaStreamWaitEvent(p->s_h2d, p->ev_yout[b], 0) == cudaSuccess;
            ok = ok && copy_h2d(p->d_ys[b], yh + j * ys, yb, p->s_h2d) == cudaSuccess;
        }
        ok = ok && cudaEventRecord(p->ev_x[b], p->s_h2d) == cudaSuccess;
        // compute: SpMV j on `stream` after its inputs landed and y slot b was drained
        ok = ok && cudaStreamWaitEvent(s, p->ev_x[b], 0) == cudaSuccess;
        ok = ok && cudaStreamWaitEvent(s, p->ev_yout[b], 0) == cudaSuccess;
        if (!ok) break;
        dasp_status_t st = dasp_spmv(p, p->d_xs[b], p->d_ys[b], alpha, beta, stream);
        if (st != DASP_OK) return st;
        ok = ok && cudaEventRecord(p->ev_done[b], s) == cudaSuccess;
        // d2h: y_j back while x_{j+1} comes in and SpMV j+1 runs
        ok = ok && cudaStreamWaitEvent(p->s_d2h, p->ev_done[b], 0) == cudaSuccess;
        ok = ok && cudaMemcpyAsync(yh + j * ys, p->d_ys[b], yb, cudaMemcpyDeviceToHost, p->s_d2h) == cudaSuccess;
        ok = ok && cudaEventRecord(p->ev_yout[b], p->s_d2h) == cudaSuccess;
    }
    if (!ok) return DASP_ERR_CUDA;
    if (cudaStreamWaitEvent(s, p->ev_yout[0], 0) != cudaSuccess || cudaStreamWaitEvent(s, p->ev_yout[1], 0) != cudaSuccess)
        return DASP_ERR_CUDA;
    return cudaStreamSynchronize(s) == cudaSuccess ? DASP_OK : DASP_ERR_CUDA;
}

dasp_status_t dasp_plan_destroy(dasp_plan_t p) {
    if (!p) return DASP_OK;
    if (p->device >= 0) {
        DeviceGuard guard(p->device);
        cudaDeviceSynchronize();
        free_device(p);
    }
    p->host.release();
    delete p;
    return DASP_OK;
}

dasp_status_t dasp_plan_get_info(dasp_plan_t p, dasp_plan_info_t* o) {
    if (!p || !o) return DASP_ERR_INVALID_ARG;
    const HostFormat& f = p->host;
    std::memset(o, 0, sizeof(*o));
    o->m = f.m; o->n = f.n; o->nnz = f.nnz;
    o->dtype = p->dtype; o->device = p->device;
    o->n_empty = f.n0; o->n_len1 = f.n1; o->n_len2 = f.n2; o->n_len3 = f.n3; o->n_len4 = f.n4;
    o->row_medium = f.row_medium; o->row_long = f.row_long; o->rowblocks = f.nrb;
    o->n_groups = f.n_groups; o->n_groups_padded = f.n_groups_padded;
    o->tiles_13 = f.t13; o->tiles_4 = f.t4; o->tiles_22 = f.t22; o->tiles_single = f.ts;
    o->nnz_long_new = f.nnz_long_new; o->nnz_reg_new = f.nnz_reg_new; o->nnz_irreg = f.nnz_irreg;
    o->nnz_short_new = f.nnz_short_new;
    o->nnz_long = f.nnz_long; o->nnz_medium = f.nnz_medium; o->nnz_short = f.nnz_short;
    o->device_bytes = p->device_bytes;
    o->alg_bytes_beta0 = alg_bytes(p, false);
    o->alg_bytes_beta1 = alg_bytes(p, true);
    o->medium_rb_per_warp = p->rbw;
    o->launches_per_spmv = (p->n_units > 0 ? 1 : 0) + (p->blocks + f.row_long + f.n0 > 0 ? 1 : 0);
    o->panel_rows = f.panel_rows;
    o->n_panels = f.n_panels;
    o->rowblocks_mid = p->rb_mid;
    o->rowblocks_narrow = p->rb_narrow;
    o->narrow_rb_per_warp = p->nrw;
    o->main_blocks_per_sm = p->occ5 ? 5 : 4;
    o->short_tiles_per_warp = p->tpw;
    o->x_stage_blocks = p->stage_blocks;
    o->x_stage_smem = p->stage_smem;
    o->max_len = f.max_len;
    o->threshold = f.tau;
    o->build_ms = p->build_ms;
    o->upload_ms = p->upload_ms;
    return DASP_OK;
}

dasp_status_t dasp_plan_copy_array(dasp_plan_t p, int32_t id, void* dst, int64_t* bytes) {
    if (!p || !bytes || id < 0 || id >= DASP_ARR_COUNT) return DASP_ERR_INVALID_ARG;
    const int64_t nb = p->bytes[id];
    if (!dst) { *bytes = nb; return DASP_OK; }
    if (*bytes < nb) { *bytes = nb; return DASP_ERR_INVALID_ARG; }
    *bytes = nb;
    if (nb == 0) return DASP_OK;
    if (p->host.arr[id].ptr) {
        std::memcpy(dst, p->host.arr[id].ptr, static_cast<size_t>(nb));
        return DASP_OK;
    }
    if (p->device < 0 || !p->d[id]) return DASP_ERR_INTERNAL;
    DeviceGuard guard(p->device);
    return cudaMemcpy(dst, p->d[id], static_cast<size_t>(nb), cudaMemcpyDeviceToHost) == cudaSuccess ? DASP_OK : DASP_ERR_CUDA;
}

dasp_status_t dasp_partition_rows(const int64_t* row_ptr, int64_t m, int32_t nparts, int64_t* starts) {
    if (!row_ptr || !starts || nparts < 1 || m < 0) return DASP_ERR_INVALID_ARG;
    const int64_t nnz = row_ptr[m];
    starts[0] = 0;
    for (int32_t q = 1; q < nparts; ++q) {
        // first row r with row_ptr[r] >= q*nnz/nparts (balanced by nonzeros)
        const int64_t target = static_cast<int64_t>((static_cast<__int128>(nnz) * q) / nparts);
        const int64_t* it = std::lower_bound(row_ptr, row_ptr + m + 1, target);
        int64_t r = it - row_ptr;
        starts[q] = std::max(starts[q - 1], std::min(r, m));
    }
    starts[nparts] = m;
    return DASP_OK;
}

dasp_status_t dasp_remap_columns(int32_t* col, int64_t nnz, const int64_t* starts, int32_t nparts, int64_t* stride) {
    if ((!col && nnz > 0) || !starts || nparts < 1 || !stride) return DASP_ERR_INVALID_ARG;
    int64_t S = 0;
    for (int32_t q = 0; q < nparts; ++q) S = std::max(S, starts[q + 1] - starts[q]);
    if (S * nparts > 0x7fffffffLL) return DASP_ERR_INVALID_ARG;
    *stride = S;
    const int64_t n = starts[nparts];
    int bad = 0;
#pragma omp parallel for schedule(static) reduction(| : bad)
    for (int64_t k = 0; k < nnz; ++k) {
        const int64_t c = col[k];
        if (c < 0 || c >= n) { bad |= 1; continue; }
        const int64_t q = std::upper_bound(starts, starts + nparts + 1, c) - starts - 1;
        col[k] = static_cast<int32_t>(q * S + (c - starts[q]));
    }
    return bad ? DASP_ERR_INVALID_ARG : DASP_OK;
}

dasp_status_t dasp_gather_halo(const void* src, const int32_t* idx, int64_t n, void* dst, int32_t elem_bytes,
                               void* stream) {
    if (n < 0 || (n > 0 && (!src || !idx || !dst)) || (elem_bytes != 2 && elem_bytes != 4 && elem_bytes != 8))
        return DASP_ERR_INVALID_ARG;
    return dasp::launch_gather(src, idx, n, dst, elem_bytes, static_cast<cudaStream_t>(stream)) == cudaSuccess
               ? DASP_OK : DASP_ERR_CUDA;
}

dasp_status_t dasp_plan_set_timing(dasp_plan_t p, int32_t capacity) {
    if (!p || capacity < 0) return DASP_ERR_INVALID_ARG;
    p->timing_cap = capacity;
    p->timing_calls = 0;
    return DASP_OK;
}

dasp_status_t dasp_plan_read_timing(dasp_plan_t p, double* ms, int64_t* launches) {
    if (!p || !ms || !launches) return DASP_ERR_INVALID_ARG;
    for (int k = 0; k < DASP_K_COUNT; ++k) { ms[k] = 0; launches[k] = 0; }
    if (p->device < 0) return DASP_OK;
    DeviceGuard guard(p->device);
    for (auto& r : p->recs) {
        if (cudaEventSynchronize(r.b) != cudaSuccess) return DASP_ERR_CUDA;
        float t = 0;
        if (cudaEventElapsedTime(&t, r.a, r.b) != cudaSuccess) return DASP_ERR_CUDA;
        ms[r.kernel] += t;
        launches[r.kernel] += 1;
    }
    p->recs.clear();
    p->pool_used = 0;
    p->timing_calls = 0;
    return DASP_OK;
}

}  // extern "C"
