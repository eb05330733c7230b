// gpu_builder.cuh — device-side DASP format builder (gpu_builder.cu).
#pragma once
#include <cuda_runtime.h>

#include "format.hpp"

namespace dasp {

constexpr int64_t kDeviceArrayPad = 64;   // every device array gets this tail (vector loads past the end)

// Builds the format from a device CSR (d_row_ptr[m+1], d_col[nnz], d_val[nnz] on the current
// device) straight into device arrays d_arrays[DASP_ARR_COUNT] (cudaMalloc'ed here, byte sizes in
// f.arr[a].bytes, host pointers null) and fills f's counts and f.panel_table.  nnz is the length of
// d_col / d_val: DASP_ERR_INVALID_CSR unless d_row_ptr[m] == nnz (checked before any kernel reads
// them).  Returns a dasp_status_t; on error nothing stays allocated.
int build_format_device(HostFormat& f, void** d_arrays, int dtype, int64_t m, int64_t n, int64_t nnz,
                        const int64_t* d_row_ptr, const int32_t* d_col, const void* d_val, bool validate,
                        int64_t panel_rows, int64_t max_len, double tau, cudaStream_t s);

// count / sum / sum of squares of the row lengths in [MIN_MEDIUM_LEN, max_len] (the medium class) of a
// device row_ptr (the automatic panel size, api.cu)
cudaError_t medium_length_stats(const int64_t* d_row_ptr, int64_t m, int64_t max_len, int64_t* count, int64_t* sum,
                                int64_t* sumsq, cudaStream_t s);

// host_out[u] = long_col[u * unit_elems] for u < n_units (device gather + one copy)
cudaError_t gather_unit_first_col(const int32_t* d_long_col, int64_t unit_elems, int64_t n_units, int32_t* host_out,
                                  cudaStream_t s);

}  // namespace dasp
