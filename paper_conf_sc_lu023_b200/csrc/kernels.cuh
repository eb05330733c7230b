// kernels.cuh — launch interface of the sm_100a DASP kernels (kernels.cu).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

namespace dasp {

#ifndef DASP_MAIN_THREADS
#define DASP_MAIN_THREADS 256
#endif
constexpr int MAIN_THREADS = DASP_MAIN_THREADS;   // threads per block of the main / long / short kernels
constexpr int MAX_EXTRA_DST = 7;   // dasp_spmv_scatter: up to 8 destinations (this GPU + 7 peers)

// Extra destinations of y (dasp_spmv_scatter): every value stored into y is also stored at the
// same row offset of each extra[d] -- typically a peer GPU's x buffer mapped over NVLink, so
// iterated SpMV needs no separate all-gather.
struct ExtraDst {
    void* ptr[MAX_EXTRA_DST];
    int32_t n;
};
constexpr int WARPS_PER_BLOCK = MAIN_THREADS / 32;

// One row panel (R28) as the medium/short kernel sees it.  Its main warps are, in
// order: nmw medium warps -- nmwd of them over the row-blocks [0, rbm) with rbw row-blocks each
// (Alg. 3, LOOP_NUM P:L271), nmwm - nmwd mid narrow warps over [rbm, rbn) whose rows all fit in
// 4K slots (two lanes per row), nmw - nmwm narrow warps over [rbn, nrb) whose rows fit in 2K
// slots (one lane per row), narrow_rb_per_warp() row-blocks each -- then one warp per short tile
// (1&3 | len4 | 2&2 | singles).  Its long units (unit0, nunits) run either in their own kernel
// (dasp_long_kernel) or, co-scheduled, as long blocks of the main kernel interleaved with the
// panel's main blocks (MainParams::blk_word).
struct PanelDesc {
    int64_t blk0;
    int64_t unit0, nunits;
    int64_t rb0, nrb, nmw;
    int64_t tile0, t13, t4, t22, ts, out0;
    int64_t rbm, rbn, nmwd, nmwm;
};

// Everything the fused main kernel reads.
struct MainParams {
    const void* long_val;
    const int32_t* long_col;
    void* partial;            // [n_groups_padded] f64 (FP64) / f32 (FP16) workspace
    const int64_t* rb_ptr;
    const void* reg_val;
    const int32_t* reg_col;
    const int64_t* irr_ptr;
    const void* irr_val;
    const int32_t* irr_col;
    const int32_t* med_out;
    const void* short_val;
    const int32_t* short_col;
    const int32_t* short_out;
    const PanelDesc* panels;
    // role of every block after the fin blocks: bit 63 = long block (8 long units of the panel,
    // co-scheduled mode), bits 32..62 = panel, bits 0..31 = block index among the panel's blocks
    // of that kind
    const uint64_t* blk_word;
    const int32_t* unit_order;// long units in execution order (column-bucketed per panel)
    const void* x;
    void* y;
    double alpha, beta;
    int32_t rbw;
    int32_t wide_il;          // 1: a block's wide medium warps interleave their row-blocks (kernels.cu medium_warp)
    int32_t narrow_il;        // 1: a block's narrow / mid warps interleave their passes (medium_narrow)
    int32_t nrw;              // row-blocks per narrow / mid warp (4 or 8: a multiple of 4)
    int32_t class_mask;       // bit 0 long, bit 1 medium, bit 2 short (profiling; 7 = all)
    ExtraDst extra;
    // dynamic schedule of the main kernel (launch_main_dyn): panel q's work items are
    // [item_start[q], item_start[q+1]) = its medium warps' row-block chunks, then its short tiles
    const int64_t* item_start;
    unsigned long long* sched;  // [0] next item, [1] finished warps; both 0 between launches
    // long-row phase 2 + empty rows fused into the main kernel (its first fin_warps warps / items;
    // the long kernel has completed, so every group partial is final)
    const int64_t* group_ptr;
    const int32_t* long_out;
    const int32_t* empty_rows;
    int64_t row_long, n0, fin_warps;
    // co-scheduled long units (blk_word long blocks): group_row[g] = long row of group g (-1 for
    // the pad groups); long_cnt[r] = groups of row r not yet summed in this launch (reset to the
    // row's group count by the warp that completes the row, which then runs phase 2 for it)
    const int32_t* group_row;
    int32_t* long_cnt;
};
// finish work of the fused main kernel: 4 long rows per warp, then 128 empty rows per warp
inline int64_t finish_warps(int64_t row_long, int64_t n0) { return (row_long + 3) / 4 + (n0 + 127) / 128; }

struct FinishParams {
    const void* partial;
    const int64_t* group_ptr;
    const int32_t* long_out;
    const int32_t* empty_rows;
    void* y;
    double alpha, beta;
    int64_t row_long, n0;
    ExtraDst extra;
};

// variant: 1 = MMA (DMMA/HMMA diagonal trick), 2 = CUDA-core.  dtype: 0 = FP64, 1 = FP16.
// apw_bytes > 0: launch with an L2 access-policy window (persisting) over [apw_base, +apw_bytes)
cudaError_t launch_main(const MainParams& p, int dtype, int variant, int64_t blocks, cudaStream_t s,
                        const void* apw_base = nullptr, size_t apw_bytes = 0, float apw_hit = 1.0f);
cudaError_t launch_long(const MainParams& p, int dtype, int variant, int64_t n_units, cudaStream_t s,
                        const void* apw_base = nullptr, size_t apw_bytes = 0, float apw_hit = 1.0f);
// short tiles one main-kernel warp processes (build knob DASP_SHORT_TPW)
int short_tiles_per_warp(int dtype);
// narrow medium row-blocks (rows of at most narrow_max_slots(K) = 2K slots: max(K*nreg, longest
// row)): the most row-blocks one narrow warp processes, 0 = no narrow path for this dtype
int narrow_rb_per_warp(int dtype);
constexpr int narrow_max_slots(int K) { return 2 * K; }
constexpr int mid_max_slots(int K) { return 4 * K; }
// co-scheduled mode metadata from group_ptr: long_cnt[r] = groups of row r, group_row[g] = row
// (group_row must be pre-filled with -1 for the pad groups)
cudaError_t launch_long_meta(const int64_t* group_ptr, int64_t row_long, int32_t* long_cnt, int32_t* group_row,
                             cudaStream_t s);
// persistent main kernel with dynamic (atomic counter) work distribution over the items of
// MainParams::item_start; blocks = resident blocks (main_dyn_occupancy x SMs) or fewer
cudaError_t launch_main_dyn(const MainParams& p, int dtype, int variant, int64_t blocks, int64_t n_items, cudaStream_t s);
cudaError_t main_dyn_occupancy(int dtype, int variant, int* blocks_per_sm);
cudaError_t launch_short(const MainParams& p, int dtype, int variant, const uint64_t* tile_meta, int64_t n_tiles,
                         cudaStream_t s);
cudaError_t launch_finish(const FinishParams& p, int dtype, cudaStream_t s);

// Persistent TMA-staged pipeline kernel (kernels.cu): items are 64-bit words
// (kind<<62 | payload; see kernels.cu item_kind / produce).
size_t pipe_smem_bytes();
int pipe_warps_per_block();
cudaError_t pipe_occupancy(int dtype, int variant, int* blocks_per_sm);   // also sets the smem attribute
cudaError_t launch_pipe(const MainParams& p, int dtype, int variant, const uint64_t* items, int64_t n_items,
                        int64_t blocks, cudaStream_t s);
cudaError_t launch_scale(void* y, int64_t m, double beta, int dtype, cudaStream_t s, const ExtraDst& extra);
// dst[k] = src[idx[k]] for k < n, elements of elem_bytes (2, 4 or 8) bytes
cudaError_t launch_gather(const void* src, const int32_t* idx, int64_t n, void* dst, int elem_bytes, cudaStream_t s);
// host -> device copy by SM loads; host_src must be page-locked (device-accessible under UVA) and 16-B aligned
cudaError_t launch_h2d_sm(void* dst, const void* host_src, size_t bytes, int sms, cudaStream_t s);

}  // namespace dasp
