/*
 * dasp.h — C-ABI of the B200-native DASP SpMV hot path (libdasp.so).
 *
 * Operation (the hot path): general sparse matrix-vector multiply
 *
 *        y = alpha * A * x + beta * y
 *
 * with A in CSR (Val, ColIdx, RowPtr; §2.1 of /root/reference/PAPER.md, cited P:Lnnn)
 * and x, y dense.  Alg. 1 defines the result; DASP (§3) computes it
 * by binning rows into long / medium / short classes, packing each class into
 * small padded MMA-shaped blocks, computing block inner products on the MMA
 * units and writing y.  alpha/beta are the BLAS generalisation of Alg. 1 l.7
 * asked for by BASELINE.json north_star (reading R16).
 *
 * Precisions (north_star):
 *   DASP_R_64F : val f64, x f64, y f64; products and sums in f64 (DMMA m8n8k4).
 *   DASP_R_16F : val f16 (IEEE binary16 bits), x f16, y f32; products exact in f32 and sums
 *                in f32 (HMMA m16n8k8 f16->f32, R14/R15).  alpha/beta are applied
 *                in f32.
 *   DASP_R_32F : val f32, x f32, y f32 (R29): operands widened
 *                exactly to f64, products and sums in f64 (FP64 block geometry), y rounded once.
 *
 * No torch or CUDA types cross this boundary: device pointers are plain pointers, the CUDA
 * stream is passed as `void*` (a cudaStream_t, NULL = legacy default stream).
 *
 * Error behaviour: every entry point returns a dasp_status_t; nothing aborts or throws
 * across the ABI.  Asynchronous device faults surface at the caller's next synchronisation.
 */
#ifndef DASP_H
#define DASP_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct dasp_plan_s* dasp_plan_t;

typedef enum { DASP_R_64F = 0, DASP_R_16F = 1, DASP_R_32F = 2 } dasp_dtype_t;

typedef enum {
    DASP_OK = 0,
    DASP_ERR_INVALID_ARG = 1,   /* null/negative/aliasing argument (see each call)            */
    DASP_ERR_INVALID_CSR = 2,   /* row_ptr[0]!=0, decreasing row_ptr, row_ptr[m]!=nnz, col out of range */
    DASP_ERR_OUT_OF_MEMORY = 3, /* host or device allocation failed                           */
    DASP_ERR_CUDA = 4,          /* a CUDA runtime call or kernel launch failed                */
    DASP_ERR_UNSUPPORTED = 5,   /* e.g. dasp_spmv on a host-only plan                         */
    DASP_ERR_INTERNAL = 6
} dasp_status_t;

/* Compute variant of the block inner products (north_star (3)): the same packed arrays are
 * read either way; only the arithmetic differs.                                            */
typedef enum {
    DASP_VARIANT_DEFAULT = 0,   /* the plan's default (options.variant)                       */
    DASP_VARIANT_MMA = 1,       /* DMMA m8n8k4 (FP64, FP32) / HMMA m16n8k8 (FP16) + diagonal
                                   extraction by shuffles (Alg. 2-4)              */
    DASP_VARIANT_CUDACORE = 2   /* per-lane FMA + warp-shuffle segmented reduction            */
} dasp_variant_t;

typedef struct {
    int32_t device;             /* CUDA device ordinal; -1 = host-only plan (builder only)   */
    int32_t variant;            /* default variant of dasp_spmv (0: DASP_VARIANT_CUDACORE, the
                                   faster one on B200 in our measurements)      */
    int32_t validate;           /* 1: O(nnz) CSR validation (default); 0: skip               */
    int32_t keep_host;          /* 1: keep the host staging copy of the packed arrays        */
    int32_t medium_rb_per_warp; /* row-blocks per warp in the medium kernel (P:L271-273
                                   LOOP_NUM); 0 = automatic                                   */
    int32_t num_threads;        /* host builder threads; 0 = all available                   */
    int64_t panel_rows;         /* rows per panel (R28): each panel of consecutive
                                   rows is classified, sorted and pieced on its own so x and y
                                   windows stay L2-resident; 0 = automatic, -1 = one panel
                                   (the paper's global format)                        */
    int32_t max_len;            /* MAX_LEN, "an adjustable parameter": long iff len >
                                   max_len; 0 = 256; must be >= 4                             */
    double threshold;           /* tau, "a customized parameter": an 8 x MMA_K block is
                                   regular iff it holds more than 8*MMA_K*tau nonzeros;
                                   0 = 0.75; must be <= 1                                     */
    int32_t x_stage;            /* shared-memory staging of x windows for the wide medium
                                   row-blocks ("shared-memory or TMA staging where reuse exists",
                                   north_star (3)): 0 = automatic (the build's
                                   DASP_X_STAGE_AUTO rule; default build: off, staging measured
                                   slower than the L1-served gathers), 1 = off, 2 = on for every
                                   block whose warps gather from a few dense column windows
                                   (e.g. stencils).  Host-built CUDA-core plans only.            */
} dasp_options_t;

/* Fills `opts` with the defaults: device 0, CUDA-core variant, validate, no keep_host, auto
 * LOOP_NUM, automatic panel size, MAX_LEN 256, tau 0.75, automatic x staging. */
void dasp_options_default(dasp_options_t* opts);

/* Plan statistics (Fig. 12's class shares; build cost). */
typedef struct {
    int64_t m, n, nnz;
    int32_t dtype, device;
    int64_t n_empty, n_len1, n_len2, n_len3, n_len4;   /* short classes + empty rows (R1)   */
    int64_t row_medium, row_long;
    int64_t rowblocks;                                 /* ceil(row_medium/8) (R7)   */
    int64_t n_groups, n_groups_padded;                 /* long groups of 2*MMA_M*MMA_K      */
    int64_t tiles_13, tiles_4, tiles_22, tiles_single; /* short tiles of 32 4-slot rows /128 singles */
    int64_t nnz_long_new, nnz_reg_new, nnz_irreg, nnz_short_new; /* P:L156-164 array sizes  */
    int64_t nnz_long, nnz_medium, nnz_short;           /* real nonzeros per class           */
    int64_t device_bytes;                              /* device memory held by the plan    */
    int64_t alg_bytes_beta0;                           /* bytes one dasp_spmv must move with
                                                          beta == 0 (DESIGN.md §6 B_alg)     */
    int64_t alg_bytes_beta1;                           /* ... with beta != 0                */
    int32_t medium_rb_per_warp;
    int32_t launches_per_spmv;                         /* kernels one dasp_spmv enqueues    */
    int64_t panel_rows, n_panels;                      /* resolved panel size and count     */
    int64_t max_len;                                   /* resolved MAX_LEN                   */
    double threshold;                                  /* resolved tau                       */
    double build_ms, upload_ms;                        /* host build; host->device upload   */
    int64_t rowblocks_mid, rowblocks_narrow;           /* medium row-blocks on the two-lanes-
                                                          per-row / one-lane-per-row warps
                                                          (launch schedule)    */
    int32_t narrow_rb_per_warp;                        /* row-blocks per narrow / mid warp   */
    int32_t main_blocks_per_sm;                        /* 4, or 5 for FP16 plans without a wide-
                                                          medium majority      */
    int32_t short_tiles_per_warp;                      /* short tiles per short warp         */
    int64_t x_stage_blocks;                            /* main blocks that stage x windows   */
    int32_t x_stage_smem;                              /* their dynamic shared memory (bytes) */
} dasp_plan_info_t;

/*
 * dasp_plan_create — preprocessing (§3.2; Fig. 13 cost).
 *
 *   m, n, nnz : rows, columns, nonzeros (m, n, nnz >= 0; n <= INT32_MAX).  Rectangular ok.
 *   row_ptr   : HOST int64[m+1], row_ptr[0] = 0, non-decreasing, row_ptr[m] = nnz.
 *   col_idx   : HOST int32[nnz], 0 <= col < n.  Unsorted columns and duplicates are allowed
 *               (duplicates are summed like any other entry).
 *   val       : HOST double[nnz] (DASP_R_64F), uint16_t[nnz] binary16 bits (DASP_R_16F) or
 *               float[nnz] (DASP_R_32F).
 *   opts      : NULL for defaults.
 *
 * Copies everything it needs (the caller may free the CSR on return), builds the DASP
 * arrays on the host (multithreaded) and uploads them to `opts->device` (skipped for a
 * host-only plan).  Returns INVALID_ARG (plan_out NULL, negative sizes, n > INT32_MAX,
 * null arrays with nnz/m > 0), INVALID_CSR (validation failure), OUT_OF_MEMORY or CUDA.
 * On error *plan_out is set to NULL.
 */
dasp_status_t dasp_plan_create(dasp_plan_t* plan_out, int64_t m, int64_t n, int64_t nnz,
                               const int64_t* row_ptr, const int32_t* col_idx, const void* val,
                               dasp_dtype_t dtype, const dasp_options_t* opts);

/*
 * dasp_plan_create_device — the same plan built ON THE GPU: the CSR is
 * given as DEVICE pointers on opts->device (d_row_ptr int64[m+1], d_col_idx int32[nnz], d_val
 * double or binary16 [nnz]); classification, sorts, scans and scatters run as kernels on `stream`
 * (cudaStream_t as void*), the packed arrays are written in place in device memory and are
 * byte-identical to dasp_plan_create's.  Synchronises `stream`.  opts->device must be >= 0;
 * keep_host is ignored.  nnz must equal d_row_ptr[m] (checked before any kernel reads col/val:
 * INVALID_CSR otherwise).  Errors as dasp_plan_create.
 */
dasp_status_t dasp_plan_create_device(dasp_plan_t* plan_out, int64_t m, int64_t n, int64_t nnz,
                                      const int64_t* d_row_ptr, const int32_t* d_col_idx, const void* d_val,
                                      dasp_dtype_t dtype, const dasp_options_t* opts, void* stream);

/*
 * dasp_spmv — the hot path (§3.3, Alg. 2-5):  y = alpha*A*x + beta*y.
 *
 *   x : DEVICE pointer on the plan's device, n elements (f64 / f16 bits / f32 by dtype).
 *   y : DEVICE pointer, m elements (f64 / f32 / f32 by dtype).  Read only if beta != 0
 *       (BLAS convention: beta == 0 overwrites y, NaNs in y do not propagate).
 *   stream : cudaStream_t as void* (NULL = default stream).  Enqueue only; no host sync.
 *
 * alpha == 0 is a quick path (y = beta*y; A and x are not read).  m == 0 is a no-op.
 * Calls on one plan must be stream-ordered (the long-row partial-sum workspace is shared).
 * Returns INVALID_ARG (null plan; x == y; x NULL with n > 0 and alpha != 0; y NULL with
 * m > 0), UNSUPPORTED (host-only plan) or CUDA (launch error).
 */
dasp_status_t dasp_spmv(dasp_plan_t plan, const void* x, void* y, double alpha, double beta,
                        void* stream);

/* As dasp_spmv with an explicit compute variant (dasp_variant_t). */
dasp_status_t dasp_spmv_ex(dasp_plan_t plan, const void* x, void* y, double alpha, double beta,
                           void* stream, int32_t variant);

/*
 * dasp_spmv_scatter — dasp_spmv whose result is written to several buffers at once, the fused
 * SpMV + all-gather of the row-slab multi-GPU mode:
 *   y_dst[0]          this GPU's y (read if beta != 0), m elements;
 *   y_dst[1..ndst-1]  further device-visible destinations that receive the same m values at the
 *                     same offsets -- normally the peer GPUs' x buffers mapped into this process
 *                     over NVLink (CUDA IPC / symmetric memory), so every rank's slab lands in every
 *                     rank's next x directly from the epilogue, tile by tile, with no collective.
 * 1 <= ndst <= 8.  The caller orders the peers' next reads after this call (e.g. a device-side
 * barrier across ranks).  Returns INVALID_ARG for ndst out of range or a null destination.
 */
dasp_status_t dasp_spmv_scatter(dasp_plan_t plan, const void* x, void* const* y_dst, int32_t ndst,
                                double alpha, double beta, void* stream);

/*
 * dasp_spmv_host — end-to-end call with HOST buffers: copies x (and y if beta != 0) to
 * plan-owned device buffers, runs dasp_spmv on `stream`, copies y back and synchronises
 * `stream`.  x_host: n elements, y_host: m elements, same element types as dasp_spmv.
 * Pinned (page-locked) host buffers give full PCIe/C2C bandwidth; pageable ones work.
 */
dasp_status_t dasp_spmv_host(dasp_plan_t plan, const void* x_host, void* y_host, double alpha,
                             double beta, void* stream);

/*
 * dasp_spmv_host_stream — dasp_spmv_host over a stream of `nvec` independent right-hand sides:
 * y_j = alpha*A*x_j + beta*y_j for j = 0..nvec-1 (Alg. 1; the iterated / many-vector use
 * the paper amortises its preprocessing over).  x_host holds the vectors at a stride of
 * ldx >= n elements, y_host at a stride of ldy >= m elements (element types as dasp_spmv).  The
 * call pipelines them through two plan-owned device slots: the host->device copy of x_{j+1} and
 * the device->host copy of y_{j-1} run on two plan-owned copy streams while SpMV j runs on
 * `stream`, so per vector the cost approaches max(H2D, kernel, D2H) rather than their sum.  Every
 * vector is copied in and its result copied out (no caching).  Results are identical to nvec
 * dasp_spmv_host calls.  Synchronises `stream` before returning; the host buffers must stay valid
 * until then and should be pinned (pageable memory serialises the copies).  Copies use
 * cudaMemcpyAsync on the copy engines.  Returns INVALID_ARG
 * (null plan, nvec < 0, ldx < n with x needed, ldy < m, null buffers), UNSUPPORTED (host-only plan),
 * OUT_OF_MEMORY or CUDA.
 */
dasp_status_t dasp_spmv_host_stream(dasp_plan_t plan, const void* x_host, int64_t ldx, void* y_host,
                                    int64_t ldy, int64_t nvec, double alpha, double beta, void* stream);

/* Frees every host and device buffer of the plan.  No call on the plan may be in flight
 * (the call synchronises the plan's device).  NULL is accepted. */
dasp_status_t dasp_plan_destroy(dasp_plan_t plan);

/* Static string for a status code. */
const char* dasp_status_string(dasp_status_t s);

/* Fills *out with the plan's statistics. */
dasp_status_t dasp_plan_get_info(dasp_plan_t plan, dasp_plan_info_t* out);

/* Packed arrays of the plan (DESIGN.md §4 FORMAT), for the builder's byte-for-byte test. */
typedef enum {
    DASP_ARR_LONG_VAL = 0, DASP_ARR_LONG_COL, DASP_ARR_GROUP_PTR, DASP_ARR_LONG_OUT,
    DASP_ARR_RB_PTR, DASP_ARR_REG_VAL, DASP_ARR_REG_COL, DASP_ARR_IRR_PTR, DASP_ARR_IRR_VAL,
    DASP_ARR_IRR_COL, DASP_ARR_MED_OUT, DASP_ARR_SHORT_VAL, DASP_ARR_SHORT_COL,
    DASP_ARR_SHORT_OUT, DASP_ARR_EMPTY_ROWS,
    DASP_ARR_PANELS,        /* int64 [n_panels][12]: row0, rows, unit0, nunits, rb0, nrb, tile0,
                               t13, t4, t22, ts, out0                           */
    DASP_ARR_COUNT
} dasp_array_t;

/*
 * dasp_plan_copy_array — copies packed array `id` into HOST memory `dst` (device plans copy
 * from device memory and synchronise; host-only or keep_host plans copy from the staging
 * copy).  *bytes: in = capacity of dst, out = size of the array.  dst == NULL only queries
 * the size.  Returns INVALID_ARG for an unknown id or too small a capacity.
 */
dasp_status_t dasp_plan_copy_array(dasp_plan_t plan, int32_t id, void* dst, int64_t* bytes);

/*
 * dasp_partition_rows — nnz-balanced contiguous row slabs for the multi-GPU mode (§8(e)):
 * starts[0] = 0, starts[nparts] = m, starts[p] = the first row r with row_ptr[r] >=
 * p*nnz/nparts (binary search on HOST row_ptr[m+1]).  nparts >= 1.
 */
dasp_status_t dasp_partition_rows(const int64_t* row_ptr, int64_t m, int32_t nparts, int64_t* starts);

/*
 * dasp_remap_columns — column remap of a slab into the padded, all-gathered x layout:
 * global column c owned by part p (starts[p] <= c < starts[p+1]) becomes
 * p*S + (c - starts[p]) with S = max_p (starts[p+1]-starts[p]).  In place on HOST col[nnz]
 * (valid for square matrices partitioned like their rows).  Returns S through *stride.
 */
dasp_status_t dasp_remap_columns(int32_t* col, int64_t nnz, const int64_t* starts, int32_t nparts,
                                 int64_t* stride);

/*
 * dasp_gather_halo — the pack step of the sparse x exchange:
 * dst[k] = src[idx[k]] for 0 <= k < n, on DEVICE arrays, enqueued on `stream`.  elem_bytes is the
 * x element size (8 = f64, 4 = f32, 2 = f16 bits); values are copied bit for bit.  idx[k] must be
 * in [0, len(src)) (not checked on the device).  n == 0 is a no-op.  Errors: DASP_ERR_INVALID_ARG
 * (null pointer with n > 0, n < 0, elem_bytes not 2/4/8), DASP_ERR_CUDA (launch failure).
 */
dasp_status_t dasp_gather_halo(const void* src, const int32_t* idx, int64_t n, void* dst, int32_t elem_bytes,
                               void* stream);

/* Kernel ids of the per-kernel timing below. */
typedef enum {
    DASP_K_MAIN = 0,      /* dasp_main_kernel: long phase 2 (Alg. 2 l.17-25) + empty rows as its
                             first warps, then medium + short/single warps panel by panel (Alg. 3-5) */
    DASP_K_LONG = 1,      /* dasp_long_kernel: long phase 1 (Alg. 2 l.1-16) */
    DASP_K_SCALE = 2,     /* alpha == 0 quick path */
    DASP_K_COUNT = 3
} dasp_kernel_t;

/*
 * Per-kernel device timing with CUDA events recorded on the launch stream (for bench.py's
 * roofline line).  dasp_plan_set_timing(plan, capacity): record events for up to `capacity`
 * subsequent dasp_spmv calls (0 disables).  dasp_plan_read_timing synchronises, returns for
 * each kernel id the summed milliseconds and the number of timed launches, and resets.
 */
dasp_status_t dasp_plan_set_timing(dasp_plan_t plan, int32_t capacity);
dasp_status_t dasp_plan_read_timing(dasp_plan_t plan, double* ms_per_kernel /* [DASP_K_COUNT] */,
                                    int64_t* launches_per_kernel /* [DASP_K_COUNT] */);

/* Library version string. */
const char* dasp_version(void);

#ifdef __cplusplus
}
#endif
#endif /* DASP_H */
