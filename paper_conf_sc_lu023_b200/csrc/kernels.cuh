// kernels.cuh — launch interface of the sm_100a DASP kernels (kernels.cu).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>

namespace dasp {

// Everything the fused main kernel reads.  Warp ranges (global warp index w):
//   [0, w_long)                 long phase 1: one unit of UG groups per warp (Alg. 2 l.1-16)
//   [w_long, w_long + w_med)    medium: `rbw` row-blocks per warp (Alg. 3, LOOP_NUM P:L271)
//   [w_long + w_med, w_total)   short: one tile per warp (1&3 | len4 | 2&2 | singles; Alg. 4-5)
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
    const void* x;
    void* y;
    double alpha, beta;
    int64_t nrb;
    int64_t t13, t4, t22, ts;
    int64_t w_long, w_med, w_total;
    int32_t rbw;
};

struct FinishParams {
    const void* partial;
    const int64_t* group_ptr;
    const int32_t* long_out;
    const int32_t* empty_rows;
    void* y;
    double alpha, beta;
    int64_t row_long, n0;
};

// variant: 1 = MMA (DMMA/HMMA diagonal trick), 2 = CUDA-core.  dtype: 0 = FP64, 1 = FP16.
// w_begin/w_end select a sub-range of the main kernel's warps (whole range for a normal call).
cudaError_t launch_main(const MainParams& p, int dtype, int variant, int64_t w_begin, int64_t w_end,
                        cudaStream_t s);
cudaError_t launch_finish(const FinishParams& p, int dtype, cudaStream_t s);
cudaError_t launch_scale(void* y, int64_t m, double beta, int dtype, cudaStream_t s);

constexpr int MAIN_THREADS = 256;

}  // namespace dasp
