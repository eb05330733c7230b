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
// slots (one lane per row), narrow_rb_per_warp() row-blocks each -- then one warp per
// short_tiles_per_warp() short tiles (1&3 | len4 | 2&2 | singles).  Its long units (unit0,
// nunits) run in the long-row kernel (dasp_long_kernel).
struct PanelDesc {
    int64_t blk0;
    int64_t unit0, nunits;
    int64_t rb0, nrb, nmw;
    int64_t tile0, t13, t4, t22, ts, out0;
    int64_t rbm, rbn, nmwd, nmwm;
};

// Shared-memory staging of x windows (north_star (3): "shared-memory or TMA staging where reuse
// exists").  One entry per main-kernel block (after the finish blocks).  A staged
// block's wide medium warps gather x from shared memory: the block's referenced columns, in tiles
// of STAGE_T consecutive columns, are copied by cp.async.bulk (TMA) at block start as up to
// STAGE_RUNS runs of consecutive tiles, together with the block's tile map (plan-built, in the
// stage_map array at 16-byte offset map16): span tile i (columns xbase + STAGE_T i ..) lives in
// slot tmap[i] (0xff = not staged: gathered from global memory).
constexpr int STAGE_T = 32;          // columns per tile
constexpr int STAGE_RUNS = 4;        // bulk copies per block
constexpr int STAGE_MAX_SPAN = 4096; // tiles in a block's span (one byte of tile map each)
constexpr int STAGE_MAX_SLOTS = 96;  // staged tiles per block (FP64: 24 KB)
struct StageEnt {
    int32_t xbase;                   // first column of span tile 0 (a multiple of STAGE_T)
    int32_t ntile;                   // span tiles; 0 = block not staged
    uint16_t run_t0[STAGE_RUNS];     // run r: span tiles [run_t0[r], run_t0[r] + run_nt[r]),
    uint16_t run_nt[STAGE_RUNS];     //   stored in slots after the previous runs'
    int32_t meta;                    // nrun | slots << 8
    int32_t map16;                   // tile map offset in stage_map, 16-byte units
};
static_assert(sizeof(StageEnt) == 32, "StageEnt layout");

// Everything the long-row and main kernels read.
struct MainParams {
    const void* long_val;
    const int32_t* long_col;
    void* partial;            // [n_groups_padded] f64 (FP64 / FP32) / f32 (FP16) workspace
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
    // every main-kernel warp after the fin warps: panel << 32 | warp index within the panel
    // (~0 = an idle padding slot); n_mwarps entries
    const uint64_t* warp_word;
    int64_t n_mwarps;
    const int32_t* unit_order;// long units in execution order (column-bucketed per panel)
    const void* x;
    void* y;
    double alpha, beta;
    int32_t rbw;
    int32_t wide_il;          // 1: a block's wide medium warps interleave their row-blocks (kernels.cu medium_warp)
    int32_t narrow_il;        // 1: a block's narrow / mid warps interleave their passes (medium_narrow)
    int32_t nrw;              // row-blocks per narrow / mid warp (4 or 8: a multiple of 4)
    int32_t class_mask;       // bit 1 medium, bit 2 short (7 = all; build knob DASP_CLASS_MASK for class timings)
    int32_t tpw;              // short tiles per short warp in the plan's layout (short_tiles_per_warp)
    ExtraDst extra;           // scatter destinations (extra.n > 0 selects the scatter instantiation)
    // long-row phase 2 + empty rows fused into the main kernel (its first fin_warps warps; the
    // long kernel has completed, so every group partial is final)
    const int64_t* group_ptr;
    const int32_t* long_out;
    const int32_t* empty_rows;
    int64_t row_long, n0, fin_warps;
    // x-window staging (staged instantiation only): per-block table and the tile-map bytes that
    // precede the staged tiles in dynamic shared memory
    const StageEnt* stage;
    const unsigned char* stage_map;   // every staged block's tile map (16-byte aligned each)
    int32_t stage_map_bytes;
};
// finish work of the fused main kernel: 4 long rows per warp, then 128 empty rows per warp
inline int64_t finish_warps(int64_t row_long, int64_t n0) { return (row_long + 3) / 4 + (n0 + 127) / 128; }

// variant: 1 = MMA (DMMA/HMMA diagonal trick), 2 = CUDA-core.  dtype: 0 = FP64, 1 = FP16, 2 = FP32.
// occ5: FP16 CUDA-core plans without a wide-medium majority run the 5-block / 48-register
// instantiation (its short warps take DASP_SHORT_TPW_OCC5 tiles: short_tiles_per_warp(dtype, true))
// stage_smem > 0 (with p.stage set): the x-window staging instantiation, that many bytes of dynamic
// shared memory per block
cudaError_t launch_main(const MainParams& p, int dtype, int variant, int64_t blocks, cudaStream_t s, bool occ5 = false,
                        int stage_smem = 0);
cudaError_t launch_long(const MainParams& p, int dtype, int variant, int64_t n_units, cudaStream_t s);
// short tiles one main-kernel warp processes (build knobs DASP_SHORT_TPW_*)
int short_tiles_per_warp(int dtype, bool occ5 = false);
// narrow medium row-blocks (rows of at most narrow_max_slots(K) = 2K slots: max(K*nreg, longest
// row)): the most row-blocks one narrow warp processes
int narrow_rb_per_warp(int dtype);
constexpr int narrow_max_slots(int K) { return 2 * K; }
constexpr int mid_max_slots(int K) { return 4 * K; }
cudaError_t launch_scale(void* y, int64_t m, double beta, int dtype, cudaStream_t s, const ExtraDst& extra);
// dst[k] = src[idx[k]] for k < n, elements of elem_bytes (2, 4 or 8) bytes
cudaError_t launch_gather(const void* src, const int32_t* idx, int64_t n, void* dst, int elem_bytes, cudaStream_t s);

}  // namespace dasp
