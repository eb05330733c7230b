// format.hpp — host-side DASP format (DESIGN.md §4 FORMAT) shared by the production builder,
// the plan/ABI code and (as launch metadata) the CUDA kernels.  Not shared with oracle/.
#pragma once
#include <cstddef>
#include <cstdint>
#include <vector>

#include "../../include/dasp.h"

namespace dasp {

// Per-dtype block geometry.  FP64: mma.sync m8n8k4 (MMA_M=8, MMA_N=8, MMA_K=4).
// FP16: the minimum f16 shape mma.sync m16n8k8 with A rows 0-7 live (R14): 8 x 8 blocks.
struct Geometry {
    int sv;   // bytes per value
    int K;    // MMA_K (slots per row per block)
    int BE;   // elements per 8 x K block
    int EPL;  // elements per lane per block (BE / 32)
    int G;    // long-row group = 2 * MMA_M * MMA_K
    int UG;   // groups per long warp unit (R18): one unit = 32 lanes x (UG*G/32) elements
    int CW;   // medium chunk width in blocks (R18)
};

inline Geometry geometry(int dtype) {
    if (dtype == DASP_R_64F) return Geometry{8, 4, 32, 1, 64, 4, 4};
    if (dtype == DASP_R_32F) return Geometry{4, 4, 32, 1, 64, 4, 4};   // FP64 blocks, 4-byte values (R29)
    return Geometry{2, 8, 64, 2, 128, 4, 4};
}

constexpr int MAX_LEN = 256;     // P:L152 (default; plan option max_len)
constexpr int MIN_MEDIUM_LEN = 5; // short iff len <= 4
constexpr int MMA_M = 8;
constexpr int32_t PAD_COL = -1;  // R12: sentinel column of pads (x read as 0)
constexpr int SHORT_TILE = 128;  // elements per short tile (32 four-slot rows)
constexpr int PANEL_FIELDS = 12; // row0, rows, unit0, nunits, rb0, nrb, tile0, t13, t4, t22, ts, out0

struct HostBuf {
    void* ptr = nullptr;
    int64_t bytes = 0;
};

struct HostFormat {
    Geometry geo{};
    int dtype = 0;
    int64_t m = 0, n = 0, nnz = 0;
    int64_t n0 = 0, n1 = 0, n2 = 0, n3 = 0, n4 = 0, row_medium = 0, row_long = 0;
    int64_t nrb = 0, n_groups = 0, n_groups_padded = 0, t13 = 0, t4 = 0, t22 = 0, ts = 0;
    int64_t nnz_long_new = 0, nnz_reg_new = 0, nnz_irreg = 0, nnz_short_new = 0;
    int64_t nnz_long = 0, nnz_medium = 0, nnz_short = 0;
    int64_t sumsq_medium = 0;  // sum of squared medium row lengths (launch tuning)
    int64_t max_len = MAX_LEN; // long iff len > max_len
    double tau = 0.75;         // regular iff count > BE * tau
    std::vector<int64_t> panel_table;   // device-built plans: host copy of the panel table
    int64_t panel_rows = 0;   // rows per panel (R28); >= m: one panel = the paper's global format
    int64_t n_panels = 0;
    HostBuf arr[DASP_ARR_COUNT];
    void release();
};

// Builds the format on the host.  Returns a dasp_status_t.
int build_format(HostFormat& f, int dtype, int64_t m, int64_t n, const int64_t* row_ptr,
                 const int32_t* col, const void* val, int nthreads, bool validate, int64_t panel_rows,
                 int64_t max_len, double tau);

}  // namespace dasp
