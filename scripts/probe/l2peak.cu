// Probe: random 8-byte gather throughput from an L2-resident (or larger) buffer on B200 -- the
// sector-request ceiling that bounds x gathers (one 32-B L2 sector per scattered 8-B load).
// Addresses come from a hash (no index loads), 8 independent loads in flight per thread.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC -o libl2peak.so l2peak.cu
#include <cuda_runtime.h>
#include <cstdint>

__device__ __forceinline__ uint64_t mix(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

template <int MLP>
__global__ void __launch_bounds__(256) gather_kernel(const double* __restrict__ x, uint64_t n, int iters, double* out) {
    const uint64_t tid = blockIdx.x * 256ull + threadIdx.x;
    double acc = 0.0;
    for (int it = 0; it < iters; ++it) {
        double v[MLP];
#pragma unroll
        for (int j = 0; j < MLP; ++j) v[j] = __ldg(x + mix(tid * 131 + it * MLP + j) % n);
#pragma unroll
        for (int j = 0; j < MLP; ++j) acc += v[j];
    }
    if (acc == 12345.678) out[0] = acc;   // keep the loads
}

extern "C" int l2peak_run(const double* x, uint64_t n, int blocks, int iters, int mlp, double* out, void* stream) {
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    if (mlp == 4) gather_kernel<4><<<blocks, 256, 0, s>>>(x, n, iters, out);
    else if (mlp == 8) gather_kernel<8><<<blocks, 256, 0, s>>>(x, n, iters, out);
    else gather_kernel<16><<<blocks, 256, 0, s>>>(x, n, iters, out);
    return cudaGetLastError() == cudaSuccess ? 0 : 1;
}
