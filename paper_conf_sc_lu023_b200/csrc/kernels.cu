// kernels.cu — sm_100a kernels of the DASP SpMV hot path (§3.3, Alg. 2-5).
//
// Two launches per SpMV: the long-row phase-1 kernel (Alg. 2 l.1-16), then the
// main kernel, whose warps are (warp-uniform dispatch on the global warp index) long-row
// phase 2 + empty rows first (Alg. 2 l.17-25), then per row panel the medium row-blocks
// (Alg. 3) and short tiles, two per warp (Alg. 4-5).  Opt-in (options.co_schedule): one launch,
// the long units as blocks of the main kernel and phase 2 run by the warp that completes a
// row's group counter (long_unit_complete).  Every block inner product is computed by one of two
// variants that read the SAME packed arrays (north_star (3)):
//   VAR_MMA      legacy warp MMA: DMMA m8n8k4 f64 (Listing 1) / HMMA m16n8k8
//                f16->f32; the block dot products sit on the diagonal of C (Fig. 4)
//                and are extracted with shuffles (Alg. 2 l.10-13, Alg. 3 l.13-17).
//   VAR_CUDACORE per-lane FMA and a warp-shuffle segmented reduction.
// The packed val/col streams are read with 128/256-bit L1::no_allocate loads carrying an
// L2 evict_first policy (the paper's "cache bypass", R17) so that x stays in L2;
// x is gathered through the read-only path.  Pads carry column -1 and read x = 0 (R12).
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.cuh"

// build knobs of the medium path (experiments: make exp EXPVARS=...)
// (per value type: the register allocation of the fused kernel, and with it the measured best
// setting, differs between the FP64, FP16 and FP32 instantiations; profiles/r01b/knobs*.jsonl)
//   SMALL_PAIR: two row-blocks without a full chunk loaded together
//   CHUNK_PIPE: chunk c+1's stream loads issued while chunk c's gathers are in flight
//   SHORT_TPW : short tiles per warp (1 or 2)
#ifndef DASP_SMALL_PAIR_F64
#define DASP_SMALL_PAIR_F64 0
#endif
#ifndef DASP_SMALL_PAIR_F16
#define DASP_SMALL_PAIR_F16 1
#endif
#ifndef DASP_SMALL_PAIR_F32
#define DASP_SMALL_PAIR_F32 0
#endif
#ifndef DASP_CHUNK_PIPE_F64
#define DASP_CHUNK_PIPE_F64 0
#endif
#ifndef DASP_CHUNK_PIPE_F16
#define DASP_CHUNK_PIPE_F16 0   // 1 spills the FP16 MMA instantiation; off: C3 FP16 MMA main -8 %, CUDA-core -5 % (profiles/r02/f16_spill_free.jsonl)
#endif
#ifndef DASP_CHUNK_PIPE_F32
#define DASP_CHUNK_PIPE_F32 0
#endif
//   RAGGED_FIRST: CUDA-core wide medium path: ragged chunk + first irregular element accumulated first
#ifndef DASP_RAGGED_FIRST_F64
#define DASP_RAGGED_FIRST_F64 0
#endif
#ifndef DASP_RAGGED_FIRST_F32
#define DASP_RAGGED_FIRST_F32 0
#endif
#ifndef DASP_RAGGED_FIRST_F16
#define DASP_RAGGED_FIRST_F16 1   // C3 FP16 main -4.4 %, C2+ -1.4 %, C2 +-0, C5 +0.9 %; spill-free 5-block kernel (same file)
#endif
//   PEEL      : CUDA-core wide medium path: chunk 0, ragged chunk and first irregular element gathered in one round
#ifndef DASP_PEEL_F64
#define DASP_PEEL_F64 1   // C2 FP64 main -3.5 %, C2+ -3.6 %, C3 -0.8 %, C5 -0.6 % (profiles/r02/peel_ragged_first_ab.jsonl)
#endif
#ifndef DASP_PEEL_F32
#define DASP_PEEL_F32 0
#endif
#ifndef DASP_PEEL_F16
#define DASP_PEEL_F16 0
#endif
// 1: wide medium warps (CUDA-core) load the next row-block's metadata with this one's streams
#ifndef DASP_WIDE_META_PF_F64
#define DASP_WIDE_META_PF_F64 1   // C2 main -1.8 %, C2+ -3.8 %, C5 -0.7 %, C3 +-0; FP32 C3 +2.6 %, FP16 +-0 (off there; profiles/r02b/meta_prefetch_ab.jsonl)
#endif
#ifndef DASP_WIDE_META_PF_F16
#define DASP_WIDE_META_PF_F16 0
#endif
#ifndef DASP_WIDE_META_PF_F32
#define DASP_WIDE_META_PF_F32 0
#endif
#ifndef DASP_SHORT_TPW_F64
#define DASP_SHORT_TPW_F64 2
#endif
#ifndef DASP_SHORT_TPW_F16
#define DASP_SHORT_TPW_F16 4
#endif
#ifndef DASP_SHORT_TPW_F32
#define DASP_SHORT_TPW_F32 3
#endif
#ifndef DASP_SHORT_TPW_OCC5
#define DASP_SHORT_TPW_OCC5 2   // the FP16 5-block instantiation (VAR_OCC5): 2 tiles fit its 48 registers
#endif
#define DASP_BY_DT(DT, K) ((DT) == 0 ? K##_F64 : ((DT) == 1 ? K##_F16 : K##_F32))

namespace dasp {
namespace {

constexpr unsigned FULL = 0xffffffffu;
// variant template argument: bits 0-1 the block-dot path, bit 2 the scatter epilogue
// (dasp_spmv_scatter), bit 3 the FP16 CUDA-core instantiation at 5 blocks / 48 registers per
// thread (VAR_OCC5, plans without a wide-medium majority: main_occ5), each instantiated separately
// bit 4 the x-window staging instantiation (VAR_STAGE, CUDA-core only: x_stage plans)
enum { VAR_MMA = 1, VAR_CUDACORE = 2, VAR_SCATTER = 4, VAR_OCC5 = 8, VAR_STAGE = 16 };
__host__ __device__ constexpr int vk(int v) { return v & 3; }
__host__ __device__ constexpr bool vs(int v) { return (v & VAR_SCATTER) != 0; }
__host__ __device__ constexpr bool vo(int v) { return (v & VAR_OCC5) != 0; }
__host__ __device__ constexpr bool vst(int v) { return (v & VAR_STAGE) != 0; }

// ------------------------------------------------------------------------------------------
// memory helpers
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ uint64_t stream_policy() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// experiment only (DASP_EXP_TRACE=1): per-warp phase timestamps of the main kernel's first work
// item -- kind, clock64 at start / streams landed / gathers landed / end, globaltimer start / end,
// SM id -- read back with dasp_exp_trace_read
#ifndef DASP_EXP_TRACE
#define DASP_EXP_TRACE 0
#endif
#if DASP_EXP_TRACE
constexpr int64_t kTraceWarps = 1 << 20;
__device__ uint64_t g_trace[kTraceWarps * 8];
__device__ __forceinline__ uint64_t clk64() {
    uint64_t c;
    asm volatile("mov.u64 %0, %%clock64;" : "=l"(c)::"memory");
    return c;
}
__device__ __forceinline__ uint64_t gtime() {
    uint64_t c;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(c)::"memory");
    return c;
}
__device__ __forceinline__ void wait_on(uint32_t v) {   // an instruction that reads v: the warp waits for it
    uint32_t d;
    asm volatile("mov.b32 %0, %1;" : "=r"(d) : "r"(v) : "memory");
}
__device__ __forceinline__ void wait_on_d(double v) {
    double d;
    asm volatile("mov.f64 %0, %1;" : "=d"(d) : "d"(v) : "memory");
}
struct Trace {
    uint64_t c0, c1, c2, t0;
    int kind;
    __device__ __forceinline__ void start(int k) { kind = k; t0 = gtime(); c0 = clk64(); c1 = c2 = c0; }
    __device__ __forceinline__ void finish(int lane) {
        const uint64_t c3 = clk64(), t1 = gtime();
        if (lane == 0) {
            const int64_t w = static_cast<int64_t>(blockIdx.x) * (blockDim.x >> 5) + (threadIdx.x >> 5);
            if (w < kTraceWarps) {
                uint32_t sm;
                asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
                uint64_t* q = g_trace + w * 8;
                q[0] = static_cast<uint64_t>(kind); q[1] = c0; q[2] = c1; q[3] = c2; q[4] = c3; q[5] = t0; q[6] = t1; q[7] = sm;
            }
        }
    }
};
#endif
__device__ __forceinline__ void ld4_f64(const double* a, uint64_t pol, double (&v)[4]) {
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f64 {%0,%1,%2,%3}, [%4], %5;"
        : "=d"(v[0]), "=d"(v[1]), "=d"(v[2]), "=d"(v[3]) : "l"(a), "l"(pol));
}
__device__ __forceinline__ void ld2_f64(const double* a, uint64_t pol, double& v0, double& v1) {
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0,%1}, [%2], %3;"
        : "=d"(v0), "=d"(v1) : "l"(a), "l"(pol));
}
__device__ __forceinline__ double ld1_f64(const double* a, uint64_t pol) {
    double v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(a), "l"(pol));
    return v;
}
__device__ __forceinline__ void ld8_b32(const void* a, uint64_t pol, uint32_t (&v)[8]) {
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
        : "l"(a), "l"(pol));
}
__device__ __forceinline__ void ld4_b32(const void* a, uint64_t pol, uint32_t (&v)[4]) {
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.b32 {%0,%1,%2,%3}, [%4], %5;"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "l"(a), "l"(pol));
}
__device__ __forceinline__ void ld2_b32(const void* a, uint64_t pol, uint32_t& v0, uint32_t& v1) {
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.b32 {%0,%1}, [%2], %3;"
        : "=r"(v0), "=r"(v1) : "l"(a), "l"(pol));
}
__device__ __forceinline__ uint32_t ld1_b32(const void* a, uint64_t pol) {
    uint32_t v;
    asm("ld.global.nc.L1::no_allocate.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(pol));
    return v;
}
// ------------------------------------------------------------------------------------------
// x-window staging (StageEnt, kernels.cuh): one thread of a staged block arms an mbarrier with
// the byte count and issues up to STAGE_RUNS cp.async.bulk copies (TMA, UBLKCP) of runs of
// STAGE_T-column tiles of x into dynamic shared memory; the block fills the span's tile map;
// the wide medium warps wait on the mbarrier (parity 0) before their first gather and read a
// staged column from shared memory, any other column from global memory.
// ------------------------------------------------------------------------------------------
struct StageSm {
    unsigned long long bar;
    int32_t xbase, ntile;
};
__shared__ StageSm s_stage;
extern __shared__ __align__(128) unsigned char s_dyn[];
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }

// every thread of a staged-instantiation main block (not a finish block) calls this once.  Thread 0
// initialises the mbarrier (no memory dependency) and the block synchronises once; then thread 0
// reads the block's entry, publishes xbase / ntile and arms the barrier with the bytes of the tile
// map and the runs (or arrives without bytes for an unstaged block), while the other warps go on
// to their metadata and stream loads.  Gathering warps wait on phase 0 (stage_wait).
__device__ __forceinline__ void stage_prologue(const MainParams& P, int64_t sb, int sx) {
    const uint32_t bar = smem_u32(&s_stage.bar);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar) : "memory");
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        const StageEnt* e = P.stage + sb;
        const int ntile = __ldg(&e->ntile);
        s_stage.ntile = ntile;
        s_stage.xbase = __ldg(&e->xbase);
        if (ntile > 0) {
            const int meta = __ldg(&e->meta), nrun = meta & 0xff;
            const uint32_t mapb = (static_cast<uint32_t>(ntile) + 15u) & ~15u;
            const uint32_t tx = mapb + static_cast<uint32_t>(meta >> 8) * STAGE_T * sx;
            asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(tx) : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"(smem_u32(s_dyn)), "l"(P.stage_map + static_cast<int64_t>(__ldg(&e->map16)) * 16), "r"(mapb),
                           "r"(bar)
                         : "memory");
            const char* xg = static_cast<const char*>(P.x) + static_cast<int64_t>(__ldg(&e->xbase)) * sx;
            uint32_t dst = smem_u32(s_dyn + P.stage_map_bytes);
            for (int r = 0; r < nrun; ++r) {
                const uint32_t t0 = __ldg(&e->run_t0[r]), nt = __ldg(&e->run_nt[r]);
                const uint32_t bytes = nt * STAGE_T * sx;
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(dst), "l"(xg + static_cast<int64_t>(t0) * STAGE_T * sx), "r"(bytes), "r"(bar)
                             : "memory");
                dst += bytes;
            }
        } else {
            asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
        }
    }
}
// gathering warps: wait for phase 0 (the copies, or thread 0's plain arrive); returns xbase / ntile
__device__ __forceinline__ void stage_wait(int32_t& xbase, int32_t& ntile) {
    const uint32_t bar = smem_u32(&s_stage.bar);
    asm volatile("{\n\t.reg .pred P1;\nWAIT_%=:\n\t"
                 "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 P1, [%0], 0;\n\t"
                 "@!P1 bra WAIT_%=;\n\t}" ::"r"(bar) : "memory");
    xbase = s_stage.xbase;
    ntile = s_stage.ntile;
}
// staged gather: shared memory when the column's tile is staged, else the read-only path
template <typename X>
__device__ __forceinline__ X stage_x(const X* x, const MainParams& P, uint32_t c, int32_t xbase, int32_t ntile) {
    if (static_cast<int32_t>(c) < 0) return X(0);
    const uint32_t d = c - static_cast<uint32_t>(xbase);
    const uint32_t ti = d / STAGE_T;
    if (ti < static_cast<uint32_t>(ntile)) {
        const uint32_t slot = s_dyn[ti];
        if (slot != 0xffu)
            return reinterpret_cast<const X*>(s_dyn + P.stage_map_bytes)[slot * STAGE_T + (d % STAGE_T)];
    }
    return __ldg(x + c);
}

// x gather through the read-only path; column -1 (pad, R12) reads 0 without touching memory
#ifndef DASP_EXP_NOX
#define DASP_EXP_NOX 0   // experiment only: every x gather reads x[c & 255] (cache-resident) -- wrong results
#endif
__device__ __forceinline__ int32_t xi(uint32_t c) {
    return DASP_EXP_NOX ? static_cast<int32_t>(c & 255u) : static_cast<int32_t>(c);
}
__device__ __forceinline__ double gx(const double* x, uint32_t c) {
    return static_cast<int32_t>(c) >= 0 ? __ldg(x + xi(c)) : 0.0;
}
__device__ __forceinline__ double gx_f64(const double* x, uint32_t c) { return gx(x, c); }
__device__ __forceinline__ uint16_t gxh(const uint16_t* x, uint32_t c) {
    return static_cast<int32_t>(c) >= 0 ? __ldg(reinterpret_cast<const unsigned short*>(x) + xi(c))
                                        : static_cast<uint16_t>(0);
}
// Value streams of the m8n8k4-geometry paths: FP64 (DT 0) and FP32 storage (DT 2, computed in
// FP64: every float converts exactly, so the DMMA / FMA arithmetic is the FP64 path's).
template <int DT> struct ValIO;
template <> struct ValIO<0> {
    using T = double;
    using R = double;   // register image of one value while its load is in flight
    static __device__ __forceinline__ double cv(R r) { return r; }
    static __device__ __forceinline__ void ld4r(const T* p, uint64_t pol, R (&v)[4]) { ld4_f64(p, pol, v); }
    static __device__ __forceinline__ R ld1r(const T* p, uint64_t pol) { return ld1_f64(p, pol); }
    static __device__ __forceinline__ void ld2(const T* p, uint64_t pol, double& a, double& b) { ld2_f64(p, pol, a, b); }
    static __device__ __forceinline__ void ld4(const T* p, uint64_t pol, double (&v)[4]) { ld4_f64(p, pol, v); }
    static __device__ __forceinline__ double ld1(const T* p, uint64_t pol) { return ld1_f64(p, pol); }
    static __device__ __forceinline__ double gx(const T* x, uint32_t c) { return gx_f64(x, c); }
};
template <> struct ValIO<2> {
    using T = float;
    using R = uint32_t; // the float's bits: converted at use, one register per value in flight
    static __device__ __forceinline__ double cv(R r) { return static_cast<double>(__uint_as_float(r)); }
    static __device__ __forceinline__ void ld4r(const T* p, uint64_t pol, R (&v)[4]) { ld4_b32(p, pol, v); }
    static __device__ __forceinline__ R ld1r(const T* p, uint64_t pol) { return ld1_b32(p, pol); }
    static __device__ __forceinline__ void ld2(const T* p, uint64_t pol, double& a, double& b) {
        uint32_t u0, u1;
        ld2_b32(p, pol, u0, u1);
        a = static_cast<double>(__uint_as_float(u0));
        b = static_cast<double>(__uint_as_float(u1));
    }
    static __device__ __forceinline__ void ld4(const T* p, uint64_t pol, double (&v)[4]) {
        uint32_t u[4];
        ld4_b32(p, pol, u);
#pragma unroll
        for (int j = 0; j < 4; ++j) v[j] = static_cast<double>(__uint_as_float(u[j]));
    }
    static __device__ __forceinline__ double ld1(const T* p, uint64_t pol) {
        return static_cast<double>(__uint_as_float(ld1_b32(p, pol)));
    }
    static __device__ __forceinline__ double gx(const T* x, uint32_t c) {
        return static_cast<int32_t>(c) >= 0 ? static_cast<double>(__ldg(x + xi(c))) : 0.0;
    }
};
__device__ __forceinline__ float h2f(uint16_t h) { return __half2float(__ushort_as_half(h)); }
__device__ __forceinline__ float2 u2f2(uint32_t u) {  // two packed binary16 -> two f32 (exact)
    return make_float2(h2f(static_cast<uint16_t>(u & 0xffffu)), h2f(static_cast<uint16_t>(u >> 16)));
}
__device__ __forceinline__ uint32_t pack2(uint16_t lo, uint16_t hi) { return static_cast<uint32_t>(lo) | (static_cast<uint32_t>(hi) << 16); }

// ------------------------------------------------------------------------------------------
// MMA wrappers (Listing 1) and diagonal extraction (Fig. 4)
// ------------------------------------------------------------------------------------------
// C(8x8) += A(8x4) * B(4x8); lane (g = lane>>2, t = lane&3) holds A[g][t], B[t][g],
// C[g][2t], C[g][2t+1].
__device__ __forceinline__ void dmma(double& c0, double& c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                 : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
}
// C(16x8) += A(16x8) * B(8x8), f16 inputs, f32 accumulate (m16n8k8, the minimum f16 shape).
// Rows 8-15 of A are zero (R14): a0 = A[g][2t..2t+1]; b0 = B[2t..2t+1][g]; c0,c1 = C[g][2t..2t+1].
__device__ __forceinline__ void hmma(float& c0, float& c1, uint32_t a0, uint32_t b0) {
    float c2 = 0.f, c3 = 0.f;
    asm volatile("mma.sync.aligned.m16n8k8.row.col.f32.f16.f16.f32 {%0,%1,%2,%3}, {%4,%5}, {%6}, {%0,%1,%2,%3};"
                 : "+f"(c0), "+f"(c1), "+f"(c2), "+f"(c3)
                 : "r"(a0), "r"(0u), "r"(b0));
}
// C[g][g] lives in lane 4g + (g>>1), register g&1.  Returns it to every lane of quad g.
template <typename A>
__device__ __forceinline__ A diag_to_quad(A c0, A c1, int lane) {
    const int g = lane >> 2;
    A d = (g & 1) ? c1 : c0;
    return __shfl_sync(FULL, d, 4 * g + (g >> 1));
}
__device__ __forceinline__ bool is_diag_holder(int lane) {
    const int g = lane >> 2;
    return (lane & 3) == (g >> 1);
}

template <int DT> struct Tr;
template <> struct Tr<0> {  // FP64
    using V = double; using Y = double; using A = double; using X = double;
    static constexpr int K = 4, BE = 32, EPL = 1, G = 64, UG = 4, CW = 4;
};
template <> struct Tr<1> {  // FP16 storage, FP32 accumulate
    using V = uint16_t; using Y = float; using A = float; using X = uint16_t;
    static constexpr int K = 8, BE = 64, EPL = 2, G = 128, UG = 4, CW = 4;
};
template <> struct Tr<2> {  // FP32 storage, FP64 accumulate (R29), FP64 geometry
    using V = float; using Y = float; using A = double; using X = float;
    static constexpr int K = 4, BE = 32, EPL = 1, G = 64, UG = 4, CW = 4;
};

// y[row] = alpha*acc + beta*y[row] (beta == 0: y not read, R16); scatter instantiations also
// store the value at the same row of every extra destination (peer x buffers over NVLink)
template <int DT, int VAR>
__device__ __forceinline__ void store_y(const MainParams& P, int32_t row, typename Tr<DT>::A acc) {
    using Y = typename Tr<DT>::Y;
    using A = typename Tr<DT>::A;
    if (row < 0) return;
    Y* y = static_cast<Y*>(P.y);
    A ra = static_cast<A>(P.alpha) * acc;                // in the accumulator type, one final rounding
    if (P.beta != 0.0) ra += static_cast<A>(P.beta) * static_cast<A>(y[row]);   // (FP32 variant, R29)
    const Y r = static_cast<Y>(ra);
    y[row] = r;
    if constexpr (vs(VAR))
        for (int d = 0; d < P.extra.n; ++d) static_cast<Y*>(P.extra.ptr[d])[row] = r;
}

// ------------------------------------------------------------------------------------------
// long rows, phase 1 (Alg. 2 l.1-16): one warp = one unit of UG consecutive groups
// ------------------------------------------------------------------------------------------
// Lane l reads the unit's 16-B value chunks l + 32j (j = 0..3): elements 2(l+32j), 2(l+32j)+1,
// both in group j.  Every load instruction is one contiguous 512-B (values) / 256-B (columns)
// span, and the 32 gathers of one instruction hit 64 consecutive, column-sorted elements of a
// long row, so they share sectors in L1.  Group j is accumulated separately (4 accumulators)
// and reduced over the warp.
template <int DT, int VAR>
__device__ __forceinline__ void long_unit_f64(const MainParams& P, int64_t u, int lane, uint64_t pol) {
    using IO = ValIO<DT>;
    const typename IO::T* lv = static_cast<const typename IO::T*>(P.long_val) + u * 256;
    const int32_t* lc = P.long_col + u * 256;
    const typename IO::T* x = static_cast<const typename IO::T*>(P.x);
    double v[8];
    uint32_t c[8];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        IO::ld2(lv + 2 * (lane + 32 * j), pol, v[2 * j], v[2 * j + 1]);
        ld2_b32(lc + 2 * (lane + 32 * j), pol, c[2 * j], c[2 * j + 1]);
    }
    double xv[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) xv[e] = IO::gx(x, c[e]);
    double gsum[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        if constexpr (vk(VAR) == VAR_MMA) {                  // trace of C_j = sum of group j (Fig. 4 diagonal)
            double c0 = 0.0, c1 = 0.0;
            dmma(c0, c1, v[2 * j], xv[2 * j]);
            dmma(c0, c1, v[2 * j + 1], xv[2 * j + 1]);
            gsum[j] = is_diag_holder(lane) ? (((lane >> 2) & 1) ? c1 : c0) : 0.0;
        } else {
            gsum[j] = fma(v[2 * j], xv[2 * j], v[2 * j + 1] * xv[2 * j + 1]);
        }
    }
    // 4-way transpose-reduce: after it lane l holds the full sum of group (l >> 3) & 3
    {
        const bool hi16 = lane & 16, hi8 = lane & 8;
        double a0 = hi16 ? gsum[0] : gsum[2], a1 = hi16 ? gsum[1] : gsum[3];
        double k0 = hi16 ? gsum[2] : gsum[0], k1 = hi16 ? gsum[3] : gsum[1];
        k0 += __shfl_xor_sync(FULL, a0, 16);          // groups {0,1} on lanes 0-15, {2,3} on 16-31
        k1 += __shfl_xor_sync(FULL, a1, 16);
        double b = hi8 ? k0 : k1, kk = hi8 ? k1 : k0;
        kk += __shfl_xor_sync(FULL, b, 8);             // lane l: group 2*(l>>4) + ((l>>3)&1)
        kk += __shfl_xor_sync(FULL, kk, 4);
        kk += __shfl_xor_sync(FULL, kk, 2);
        kk += __shfl_xor_sync(FULL, kk, 1);
        if ((lane & 7) == 0) static_cast<double*>(P.partial)[u * 4 + 2 * (lane >> 4) + ((lane >> 3) & 1)] = kk;
    }
}

// FP16: lane l reads 8-B value chunks l + 32j (j = 0..3): halves 4(l+32j)..+3, all in group j
// one FP16 long unit in three steps (loads | gathers | block dots + transpose-reduce + partials),
struct LongLdH {
    uint32_t vv[8], c[16];
};
__device__ __forceinline__ void long_load_f16(const MainParams& P, int64_t u, int lane, uint64_t pol, LongLdH& L) {
    const uint16_t* lv = static_cast<const uint16_t*>(P.long_val) + u * 512;
    const int32_t* lc = P.long_col + u * 512;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        ld2_b32(lv + 4 * (lane + 32 * j), pol, L.vv[2 * j], L.vv[2 * j + 1]);
        ld4_b32(lc + 4 * (lane + 32 * j), pol, *reinterpret_cast<uint32_t(*)[4]>(&L.c[4 * j]));
    }
}
__device__ __forceinline__ void long_gather_f16(const MainParams& P, const LongLdH& L, uint16_t (&xh)[16]) {
    const uint16_t* x = static_cast<const uint16_t*>(P.x);
#pragma unroll
    for (int e = 0; e < 16; ++e) xh[e] = gxh(x, L.c[e]);
}
template <int VAR>
__device__ __forceinline__ void long_finish_f16(const MainParams& P, int64_t u, const LongLdH& L, const uint16_t (&xh)[16],
                                                int lane) {
    float gsum[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        if constexpr (vk(VAR) == VAR_MMA) {
            float c0 = 0.f, c1 = 0.f;
            hmma(c0, c1, L.vv[2 * j], pack2(xh[4 * j], xh[4 * j + 1]));
            hmma(c0, c1, L.vv[2 * j + 1], pack2(xh[4 * j + 2], xh[4 * j + 3]));
            gsum[j] = is_diag_holder(lane) ? (((lane >> 2) & 1) ? c1 : c0) : 0.f;
        } else {
            const float2 a = u2f2(L.vv[2 * j]), b = u2f2(L.vv[2 * j + 1]);
            float sacc = a.x * h2f(xh[4 * j]);
            sacc = fmaf(a.y, h2f(xh[4 * j + 1]), sacc);
            sacc = fmaf(b.x, h2f(xh[4 * j + 2]), sacc);
            gsum[j] = fmaf(b.y, h2f(xh[4 * j + 3]), sacc);
        }
    }
    {
        const bool hi16 = lane & 16, hi8 = lane & 8;
        float a0 = hi16 ? gsum[0] : gsum[2], a1 = hi16 ? gsum[1] : gsum[3];
        float k0 = hi16 ? gsum[2] : gsum[0], k1 = hi16 ? gsum[3] : gsum[1];
        k0 += __shfl_xor_sync(FULL, a0, 16);
        k1 += __shfl_xor_sync(FULL, a1, 16);
        float b = hi8 ? k0 : k1, kk = hi8 ? k1 : k0;
        kk += __shfl_xor_sync(FULL, b, 8);
        kk += __shfl_xor_sync(FULL, kk, 4);
        kk += __shfl_xor_sync(FULL, kk, 2);
        kk += __shfl_xor_sync(FULL, kk, 1);
        if ((lane & 7) == 0) static_cast<float*>(P.partial)[u * 4 + 2 * (lane >> 4) + ((lane >> 3) & 1)] = kk;
    }
}
template <int VAR>
__device__ __forceinline__ void long_unit_f16(const MainParams& P, int64_t u, int lane, uint64_t pol) {
    LongLdH L;
    uint16_t xh[16];
    long_load_f16(P, u, lane, pol, L);
    long_gather_f16(P, L, xh);
    long_finish_f16<VAR>(P, u, L, xh, lane);
}

// ------------------------------------------------------------------------------------------
// medium rows (Alg. 3): row-block = 8 rows; regular 8 x K blocks in lane-interleaved chunks
// of CW blocks (R18), then the irregular tails with 4 lanes per row, then y.
// ------------------------------------------------------------------------------------------
// A row-block's metadata: its regular range, this lane's row's irregular range and output row
// (all five loads issued together, ahead of the stream loads that depend on them).
struct RbMeta {
    int64_t base, ib;         // regular region start; this lane's row's irregular start
    int32_t nelem, ilen;      // regular elements (<= 64 blocks); irregular length (<= 256)
    int32_t orow;
};
__device__ __forceinline__ RbMeta rb_meta(const MainParams& P, int64_t rb, int lane) {
    const int64_t i = rb * 8 + (lane >> 2);
    const int64_t base = __ldg(P.rb_ptr + rb), ib = __ldg(P.irr_ptr + i);
    return RbMeta{base, ib, static_cast<int32_t>(__ldg(P.rb_ptr + rb + 1) - base),
                  static_cast<int32_t>(__ldg(P.irr_ptr + i + 1) - ib), __ldg(P.med_out + i)};
}

// A row-block is processed in two halves so that a warp can keep the round-1 loads of two
// row-blocks in flight before it gathers x for the first (DASP_PAIR_*; the loads of a
// row-block depend on nothing but its metadata, R18):
//   medium_load_*   round 1: the first 4-block chunk (256/128-bit loads), the ragged last chunk
//                   and this lane's first irregular element;
//   medium_finish_* the gathers, the remaining chunks, the irregular tail and the y store.
// A row-block with nelem = ilen = 0 and orow = -1 issues no load and stores nothing.
template <int DT> struct MedLd {
    typename ValIO<DT>::R va[4], vr[3], vi;
    uint32_t ca[4], cr[3], ci;
};
// FULL = false: the row-block is known to have no full chunk (nreg < CW), so the chunk state is
// dead code and two such row-blocks fit in the registers of one (the small-pair path).
template <int DT, bool FULL = true>
__device__ __forceinline__ void medium_load_f64(const MainParams& P, const RbMeta& M, int lane, uint64_t pol, MedLd<DT>& L) {
    using IO = ValIO<DT>;
    const int nreg = M.nelem >> 5;
    const int nfull = FULL ? nreg >> 2 : 0, rem = nreg & 3;
    const typename IO::T* rv = static_cast<const typename IO::T*>(P.reg_val) + M.base;
    const int32_t* rc = P.reg_col + M.base;
    if constexpr (FULL) {
#pragma unroll
        for (int j = 0; j < 4; ++j) { L.va[j] = 0; L.ca[j] = 0xffffffffu; }
        if (nfull > 0) { IO::ld4r(rv + lane * 4, pol, L.va); ld4_b32(rc + lane * 4, pol, L.ca); }
    }
    const int64_t rbase = static_cast<int64_t>(nfull) * 128 + lane;   // ragged chunk: block j at 32j (R18)
#pragma unroll
    for (int j = 0; j < 3; ++j) {
        L.vr[j] = 0; L.cr[j] = 0xffffffffu;
        if (j < rem) { L.vr[j] = IO::ld1r(rv + rbase + 32 * j, pol); L.cr[j] = ld1_b32(rc + rbase + 32 * j, pol); }
    }
    const int64_t k = M.ib + (lane & 3);
    L.vi = 0; L.ci = 0xffffffffu;
    if (k < M.ib + M.ilen) { L.vi = IO::ld1r(static_cast<const typename IO::T*>(P.irr_val) + k, pol); L.ci = ld1_b32(P.irr_col + k, pol); }
}
template <int DT, int VAR, bool FULL = true>
__device__ __forceinline__ void medium_finish_f64(const MainParams& P, const RbMeta& M, const MedLd<DT>& L, int lane,
                                                  uint64_t pol) {
    using IO = ValIO<DT>;
    const int t = lane & 3;
    const int nreg = M.nelem >> 5;
    const int nfull = FULL ? nreg >> 2 : 0, rem = nreg & 3;
    const typename IO::T* rv = static_cast<const typename IO::T*>(P.reg_val) + M.base;
    const int32_t* rc = P.reg_col + M.base;
    const typename IO::T* x = static_cast<const typename IO::T*>(P.x);
    // x gather: through shared memory in a staged block (VAR_STAGE), else the read-only path
    int32_t sxb = 0, snt = 0;
    if constexpr (vst(VAR)) stage_wait(sxb, snt);
    auto G = [&](uint32_t c) -> double {
        if constexpr (vst(VAR)) return static_cast<double>(stage_x<typename IO::T>(x, P, c, sxb, snt));
        else return IO::gx(x, c);
    };
    double c0 = 0.0, c1 = 0.0, part = 0.0;
    // CUDA-core RAGGED_FIRST: the ragged last chunk and the first irregular element (loaded in the
    // first round with chunk 0) are gathered and accumulated before the full chunks, so their gathers
    // travel with chunk 0's instead of after the chunk loop, and their registers are free during it
    constexpr bool RF = vk(VAR) == VAR_CUDACORE && DASP_BY_DT(DT, DASP_RAGGED_FIRST) != 0;
    auto ragged_irr = [&]() {
        double xr[3];
#pragma unroll
        for (int j = 0; j < 3; ++j) xr[j] = G(L.cr[j]);   // pads / unused slots read 0
        const double xi = G(L.ci);
#pragma unroll
        for (int j = 0; j < 3; ++j) {
            if (j < rem) {                                     // rem is warp-uniform
                if constexpr (vk(VAR) == VAR_MMA) dmma(c0, c1, IO::cv(L.vr[j]), xr[j]);
                else part = fma(IO::cv(L.vr[j]), xr[j], part);
            }
        }
        if constexpr (vk(VAR) == VAR_MMA) {                        // Alg. 3 l.13-17: diagonal -> quad g
            const double d = diag_to_quad(c0, c1, lane);
            part = t == 0 ? d : 0.0;
        }
        part = fma(IO::cv(L.vi), xi, part);                    // Alg. 3 l.20-24: irregular part
    };
    if constexpr (RF) ragged_irr();
    if constexpr (FULL && vk(VAR) == VAR_CUDACORE && DASP_BY_DT(DT, DASP_PEEL) != 0) {
        // CUDA-core PEEL: chunk 0's gathers, the ragged chunk's and the first irregular element's
        // go out in one round (all were loaded together in the first round); accumulation order
        // chunk 0, ragged, irregular element, chunks 1..nfull-1
        if (nfull > 0) {
            double xa[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) xa[j] = G(L.ca[j]);
            double xr[3];
#pragma unroll
            for (int j = 0; j < 3; ++j) xr[j] = G(L.cr[j]);
            const double xi = G(L.ci);
#pragma unroll
            for (int j = 0; j < 4; ++j) part = fma(IO::cv(L.va[j]), xa[j], part);
#pragma unroll
            for (int j = 0; j < 3; ++j)
                if (j < rem) part = fma(IO::cv(L.vr[j]), xr[j], part);
            part = fma(IO::cv(L.vi), xi, part);
            for (int ch = 1; ch < nfull; ++ch) {
                typename IO::R va[4];
                uint32_t ca[4];
                IO::ld4r(rv + ch * 128 + lane * 4, pol, va);
                ld4_b32(rc + ch * 128 + lane * 4, pol, ca);
                double xv[4];
#pragma unroll
                for (int j = 0; j < 4; ++j) xv[j] = G(ca[j]);
#pragma unroll
                for (int j = 0; j < 4; ++j) part = fma(IO::cv(va[j]), xv[j], part);
            }
        } else {
            ragged_irr();
        }
    } else if constexpr (FULL) {
        typename IO::R va[4];
        uint32_t ca[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) { va[j] = L.va[j]; ca[j] = L.ca[j]; }
        // software pipeline: chunk ch+1's stream loads are issued while chunk ch's gathers are
        // in flight (one memory round trip per chunk instead of two)
        for (int ch = 0; ch < nfull; ++ch) {
            if (!DASP_BY_DT(DT, DASP_CHUNK_PIPE) && ch > 0) { IO::ld4r(rv + ch * 128 + lane * 4, pol, va); ld4_b32(rc + ch * 128 + lane * 4, pol, ca); }
            double xv[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) xv[j] = G(ca[j]);
            typename IO::R vn[4];
            uint32_t cn[4];
            if (DASP_BY_DT(DT, DASP_CHUNK_PIPE) && ch + 1 < nfull) {
                IO::ld4r(rv + (ch + 1) * 128 + lane * 4, pol, vn);
                ld4_b32(rc + (ch + 1) * 128 + lane * 4, pol, cn);
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                if constexpr (vk(VAR) == VAR_MMA) dmma(c0, c1, IO::cv(va[j]), xv[j]);
                else part = fma(IO::cv(va[j]), xv[j], part);
            }
            if (DASP_BY_DT(DT, DASP_CHUNK_PIPE) && ch + 1 < nfull) {
#pragma unroll
                for (int j = 0; j < 4; ++j) { va[j] = vn[j]; ca[j] = cn[j]; }
            }
        }
    }
    if constexpr (!RF && !(FULL && vk(VAR) == VAR_CUDACORE && DASP_BY_DT(DT, DASP_PEEL) != 0)) ragged_irr();
    const typename IO::T* iv = static_cast<const typename IO::T*>(P.irr_val);
    for (int64_t k = M.ib + t + 4; k < M.ib + M.ilen; k += 4)
        part = fma(IO::ld1(iv + k, pol), G(ld1_b32(P.irr_col + k, pol)), part);
    part += __shfl_xor_sync(FULL, part, 1);
    part += __shfl_xor_sync(FULL, part, 2);
    if (t == 0) store_y<DT, VAR>(P, M.orow, part);              // Alg. 3 l.25 through the output map (R9)
}

struct MedLdH {
    uint32_t va[4], ca[8], vr[3], cr[6], ci;
    uint16_t vi;
};
template <bool FULL = true>
__device__ __forceinline__ void medium_load_f16(const MainParams& P, const RbMeta& M, int lane, uint64_t pol, MedLdH& L) {
    const int nreg = M.nelem >> 6;
    const int nfull = FULL ? nreg >> 2 : 0, rem = nreg & 3;
    const uint16_t* rv = static_cast<const uint16_t*>(P.reg_val) + M.base;
    const int32_t* rc = P.reg_col + M.base;
    if constexpr (FULL) {
#pragma unroll
        for (int j = 0; j < 4; ++j) L.va[j] = 0u;
#pragma unroll
        for (int e = 0; e < 8; ++e) L.ca[e] = 0xffffffffu;
        if (nfull > 0) { ld4_b32(rv + lane * 8, pol, L.va); ld8_b32(rc + lane * 8, pol, L.ca); }
    }
    const int64_t rbase = static_cast<int64_t>(nfull) * 256 + lane * 2;   // ragged chunk: block j at 64j (R18)
#pragma unroll
    for (int j = 0; j < 3; ++j) {
        L.vr[j] = 0u; L.cr[2 * j] = L.cr[2 * j + 1] = 0xffffffffu;
        if (j < rem) { L.vr[j] = ld1_b32(rv + rbase + 64 * j, pol); ld2_b32(rc + rbase + 64 * j, pol, L.cr[2 * j], L.cr[2 * j + 1]); }
    }
    const int64_t k = M.ib + (lane & 3);
    L.vi = 0; L.ci = 0xffffffffu;
    if (k < M.ib + M.ilen) { L.vi = __ldg(static_cast<const unsigned short*>(P.irr_val) + k); L.ci = ld1_b32(P.irr_col + k, pol); }
}
template <int VAR, bool FULL = true>
__device__ __forceinline__ void medium_finish_f16(const MainParams& P, const RbMeta& M, const MedLdH& L, int lane, uint64_t pol) {
    const int t = lane & 3;
    const int nreg = M.nelem >> 6;
    const int nfull = FULL ? nreg >> 2 : 0, rem = nreg & 3;
    const uint16_t* rv = static_cast<const uint16_t*>(P.reg_val) + M.base;
    const int32_t* rc = P.reg_col + M.base;
    const unsigned short* iv = static_cast<const unsigned short*>(P.irr_val);
    const uint16_t* x = static_cast<const uint16_t*>(P.x);
    int32_t sxb = 0, snt = 0;
    if constexpr (vst(VAR)) stage_wait(sxb, snt);
    auto GH = [&](uint32_t c) -> uint16_t {
        if constexpr (vst(VAR)) return stage_x<unsigned short>(reinterpret_cast<const unsigned short*>(x), P, c, sxb, snt);
        else return gxh(x, c);
    };
    float c0 = 0.f, c1 = 0.f, part = 0.f;
    // one 8x8 block: this lane's two slots 2t, 2t+1 of row g
    auto blockx = [&](uint32_t a, uint16_t xa, uint16_t xb) {
        if constexpr (vk(VAR) == VAR_MMA) {
            hmma(c0, c1, a, pack2(xa, xb));
        } else {
            const float2 av = u2f2(a);
            part = fmaf(av.x, h2f(xa), part);
            part = fmaf(av.y, h2f(xb), part);
        }
    };
    auto block = [&](uint32_t a, uint32_t ca, uint32_t cb) { blockx(a, GH(ca), GH(cb)); };
    // CUDA-core RAGGED_FIRST: as in medium_finish_f64
    constexpr bool RF = vk(VAR) == VAR_CUDACORE && DASP_RAGGED_FIRST_F16 != 0;
    auto ragged_irr = [&]() {
#pragma unroll
        for (int j = 0; j < 3; ++j)
            if (j < rem) block(L.vr[j], L.cr[2 * j], L.cr[2 * j + 1]);   // rem is warp-uniform
        if constexpr (vk(VAR) == VAR_MMA) {
            const float d = diag_to_quad(c0, c1, lane);
            part = t == 0 ? d : 0.f;
        }
        part = fmaf(h2f(L.vi), h2f(GH(L.ci)), part);
    };
    if constexpr (RF) ragged_irr();
    constexpr bool PEEL = FULL && vk(VAR) == VAR_CUDACORE && DASP_PEEL_F16 != 0;
    if constexpr (PEEL) {
        if (nfull > 0) {
            uint16_t xa[8], xr[6];
#pragma unroll
            for (int e = 0; e < 8; ++e) xa[e] = GH(L.ca[e]);
#pragma unroll
            for (int e = 0; e < 6; ++e) xr[e] = GH(L.cr[e]);
            const uint16_t xi = GH(L.ci);
#pragma unroll
            for (int j = 0; j < 4; ++j) blockx(L.va[j], xa[2 * j], xa[2 * j + 1]);
#pragma unroll
            for (int j = 0; j < 3; ++j)
                if (j < rem) blockx(L.vr[j], xr[2 * j], xr[2 * j + 1]);
            part = fmaf(h2f(L.vi), h2f(xi), part);
            for (int ch = 1; ch < nfull; ++ch) {
                uint32_t va[4], ca[8];
                ld4_b32(rv + ch * 256 + lane * 8, pol, va);
                ld8_b32(rc + ch * 256 + lane * 8, pol, ca);
                uint16_t xh[8];
#pragma unroll
                for (int e = 0; e < 8; ++e) xh[e] = GH(ca[e]);
#pragma unroll
                for (int j = 0; j < 4; ++j) blockx(va[j], xh[2 * j], xh[2 * j + 1]);
            }
        } else {
            ragged_irr();
        }
    } else if constexpr (FULL) {
        uint32_t va[4], ca[8];
#pragma unroll
        for (int j = 0; j < 4; ++j) va[j] = L.va[j];
#pragma unroll
        for (int e = 0; e < 8; ++e) ca[e] = L.ca[e];
        for (int ch = 0; ch < nfull; ++ch) {   // chunk ch+1's loads overlap chunk ch's gathers
            if (!DASP_CHUNK_PIPE_F16 && ch > 0) { ld4_b32(rv + ch * 256 + lane * 8, pol, va); ld8_b32(rc + ch * 256 + lane * 8, pol, ca); }
            uint16_t xh[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) xh[e] = GH(ca[e]);
            uint32_t vn[4], cn[8];
            if (DASP_CHUNK_PIPE_F16 && ch + 1 < nfull) { ld4_b32(rv + (ch + 1) * 256 + lane * 8, pol, vn); ld8_b32(rc + (ch + 1) * 256 + lane * 8, pol, cn); }
#pragma unroll
            for (int j = 0; j < 4; ++j) blockx(va[j], xh[2 * j], xh[2 * j + 1]);
            if (DASP_CHUNK_PIPE_F16 && ch + 1 < nfull) {
#pragma unroll
                for (int j = 0; j < 4; ++j) va[j] = vn[j];
#pragma unroll
                for (int e = 0; e < 8; ++e) ca[e] = cn[e];
            }
        }
    }
    if constexpr (!RF && !PEEL) ragged_irr();
    for (int64_t k = M.ib + t + 4; k < M.ib + M.ilen; k += 4)
        part = fmaf(h2f(__ldg(iv + k)), h2f(GH(ld1_b32(P.irr_col + k, pol))), part);
    part += __shfl_xor_sync(FULL, part, 1);
    part += __shfl_xor_sync(FULL, part, 2);
    if (t == 0) store_y<1, VAR>(P, M.orow, part);
}

template <int DT, int VAR>
__device__ __forceinline__ void medium_rb_f64(const MainParams& P, const RbMeta& M, int lane, uint64_t pol) {
    MedLd<DT> L;
    medium_load_f64<DT>(P, M, lane, pol, L);
    medium_finish_f64<DT, VAR>(P, M, L, lane, pol);
}
template <int VAR>
__device__ __forceinline__ void medium_rb_f16(const MainParams& P, const RbMeta& M, int lane, uint64_t pol) {
    MedLdH L;
    medium_load_f16(P, M, lane, pol, L);
    medium_finish_f16<VAR>(P, M, L, lane, pol);
}

template <int DT, int VAR>
__device__ __forceinline__ void medium_rbs(const MainParams& P, int64_t rb0, int64_t rb1, int lane, uint64_t pol,
                                           int64_t st = 1) {   // row-blocks rb0, rb0 + st, ... < rb1
    if constexpr (DASP_BY_DT(DT, DASP_SMALL_PAIR) != 0) {
        // small-pair path: two consecutive row-blocks without a full chunk (nreg < CW: rows of
        // up to ~15 nonzeros, most medium rows of a power-law matrix) load together, so a warp
        // keeps two row-blocks' streams and gathers in flight; others take the single path.
        constexpr int FULL_ELEMS = DT == 1 ? 256 : 128;   // elements of one CW-block chunk
        int64_t rb = rb0;
        while (rb < rb1) {
            const RbMeta MA = rb_meta(P, rb, lane);     // both metadata rounds issued together
            const RbMeta MB = rb + st < rb1 ? rb_meta(P, rb + st, lane) : RbMeta{0, 0, FULL_ELEMS, 0, -1};
            {
                if (MA.nelem < FULL_ELEMS && MB.nelem < FULL_ELEMS) {
                    if constexpr (DT == 1) {
                        MedLdH LA, LB;
                        medium_load_f16<false>(P, MA, lane, pol, LA);
                        medium_load_f16<false>(P, MB, lane, pol, LB);
                        medium_finish_f16<VAR, false>(P, MA, LA, lane, pol);
                        medium_finish_f16<VAR, false>(P, MB, LB, lane, pol);
                    } else {
                        MedLd<DT> LA, LB;
                        medium_load_f64<DT, false>(P, MA, lane, pol, LA);
                        medium_load_f64<DT, false>(P, MB, lane, pol, LB);
                        medium_finish_f64<DT, VAR, false>(P, MA, LA, lane, pol);
                        medium_finish_f64<DT, VAR, false>(P, MB, LB, lane, pol);
                    }
                    rb += 2 * st;
                    continue;
                }
            }
            if constexpr (DT == 1) medium_rb_f16<VAR>(P, MA, lane, pol);
            else medium_rb_f64<DT, VAR>(P, MA, lane, pol);
            rb += st;
        }
    } else if constexpr (vk(VAR) == VAR_CUDACORE && !vst(VAR) && DASP_BY_DT(DT, DASP_WIDE_META_PF) != 0) {
        // the next row-block's metadata loads are issued with this row-block's stream loads
        RbMeta Mn = rb_meta(P, rb0, lane);
        for (int64_t rb = rb0; rb < rb1; rb += st) {
            const RbMeta M = Mn;
            if constexpr (DT == 1) {
                MedLdH L;
                medium_load_f16(P, M, lane, pol, L);
                if (rb + st < rb1) Mn = rb_meta(P, rb + st, lane);
                medium_finish_f16<VAR>(P, M, L, lane, pol);
            } else {
                MedLd<DT> L;
                medium_load_f64<DT>(P, M, lane, pol, L);
                if (rb + st < rb1) Mn = rb_meta(P, rb + st, lane);
                medium_finish_f64<DT, VAR>(P, M, L, lane, pol);
            }
        }
    } else {
#if DASP_EXP_TRACE
        Trace tr;
        tr.start(2);
        bool first = true;
#endif
        for (int64_t rb = rb0; rb < rb1; rb += st) {
            // (prefetching the next row-block's metadata here was measured: it costs registers
            // and spills in the FP64 MMA instantiation, net slower; profiles/r01/meta_prefetch_rbw.jsonl)
            const RbMeta M = rb_meta(P, rb, lane);
#if DASP_EXP_TRACE
            if (first) { wait_on(static_cast<uint32_t>(M.base) ^ static_cast<uint32_t>(M.orow)); tr.c1 = clk64(); }
#endif
            if constexpr (DT == 1) medium_rb_f16<VAR>(P, M, lane, pol);
            else medium_rb_f64<DT, VAR>(P, M, lane, pol);
#if DASP_EXP_TRACE
            if (first) { __syncwarp(); tr.c2 = clk64(); first = false; }
#endif
        }
#if DASP_EXP_TRACE
        tr.finish(lane);
#endif
    }
}

// ------------------------------------------------------------------------------------------
// short rows (Alg. 4) and singles (Alg. 5): tiles of 32 four-slot rows.
// One tile is processed in three steps so that a warp can hold TPW tiles' loads and gathers in
// flight together (DASP_SHORT_TPW): short_load_* (values, columns and the output map, issued
// together), short_gather_* (x), short_math_* (block dots, segment masks, y).  Results are
// transposed with shuffles so that lane L writes outputs L and L+32 of a tile: the output map is
// read with coalesced loads.
// ------------------------------------------------------------------------------------------
// cat 0 = 1&3 (seg0 = slot 0, seg1 = slots 1-3), 1 = len-4, 2 = 2&2 (slots 0-1 | 2-3), 3 = singles
__device__ __forceinline__ int seg_of(int cat, int slot) { return cat == 0 ? (slot > 0) : (cat == 2 ? (slot >> 1) : 0); }

struct ShortRef {
    int cat;
    int64_t tile, obase;
};
// tile t of panel D: category and output base (tiles [1&3][len4][2&2][singles])
__device__ __forceinline__ ShortRef short_ref(const PanelDesc* D, int64_t t) {
    const int64_t t13 = __ldg(&D->t13), t4 = __ldg(&D->t4), t22 = __ldg(&D->t22);
    const int64_t out0 = __ldg(&D->out0);
    ShortRef r;
    r.tile = __ldg(&D->tile0) + t;
    if (t < t13) { r.cat = 0; r.obase = out0 + t * 64; }
    else if (t < t13 + t4) { r.cat = 1; r.obase = out0 + 64 * t13 + (t - t13) * 32; }
    else if (t < t13 + t4 + t22) { r.cat = 2; r.obase = out0 + 64 * t13 + 32 * t4 + (t - t13 - t4) * 64; }
    else { r.cat = 3; r.obase = out0 + 64 * t13 + 32 * t4 + 64 * t22 + (t - t13 - t4 - t22) * 128; }
    return r;
}
// the output map: singles 4 consecutive outputs per lane; two-output tiles L and L+32; len-4 L
#ifndef DASP_EXP_SHORT_YSEQ
#define DASP_EXP_SHORT_YSEQ 0   // experiment only: short outputs go to consecutive y slots (no output map; wrong y)
#endif
__device__ __forceinline__ void short_load_out(const MainParams& P, const ShortRef& T, int lane, uint64_t pol,
                                               int32_t (&o)[4]) {
    if (DASP_EXP_SHORT_YSEQ) {
        const int32_t b = static_cast<int32_t>(T.obase % (1 << 23));
        if (T.cat == 3) { for (int j = 0; j < 4; ++j) o[j] = b + lane * 4 + j; }
        else { o[0] = b + lane; o[1] = T.cat != 1 ? b + 32 + lane : -1; o[2] = o[3] = -1; }
        return;
    }
    if (T.cat == 3) {
        ld4_b32(P.short_out + T.obase + lane * 4, pol, *reinterpret_cast<uint32_t(*)[4]>(&o));
    } else {
        o[0] = __ldg(P.short_out + T.obase + lane);
        o[1] = T.cat != 1 ? __ldg(P.short_out + T.obase + 32 + lane) : -1;
        o[2] = o[3] = -1;
    }
}

template <int DT> struct ShortLd {          // FP64 / FP32 (m8n8k4 geometry)
    typename ValIO<DT>::R v[4];
    uint32_t c[4];
    int32_t o[4];
};
#ifndef DASP_SINGLES_T
#define DASP_SINGLES_T 1   // singles: lane L takes singles L, L+32, L+64, L+96 (each store instruction
#endif                     // covers 32 consecutive singles) instead of 4L..4L+3
template <int DT>
__device__ __forceinline__ void short_load_f64(const MainParams& P, const ShortRef& T, int lane, uint64_t pol, ShortLd<DT>& L) {
    using IO = ValIO<DT>;
    const typename IO::T* sv = static_cast<const typename IO::T*>(P.short_val) + T.tile * 128;
    if (DASP_SINGLES_T && T.cat == 3) {
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            L.v[j] = IO::ld1r(sv + 32 * j + lane, pol);
            L.c[j] = ld1_b32(P.short_col + T.tile * 128 + 32 * j + lane, pol);
            L.o[j] = DASP_EXP_SHORT_YSEQ ? static_cast<int32_t>(T.obase % (1 << 23)) + 32 * j + lane
                                         : static_cast<int32_t>(ld1_b32(P.short_out + T.obase + 32 * j + lane, pol));
        }
        return;
    }
    IO::ld4r(sv + lane * 4, pol, L.v);
    ld4_b32(P.short_col + T.tile * 128 + lane * 4, pol, L.c);
    short_load_out(P, T, lane, pol, L.o);
}
template <int DT>
__device__ __forceinline__ void short_gather_f64(const MainParams& P, const ShortLd<DT>& L, double (&xv)[4]) {
    using IO = ValIO<DT>;
#pragma unroll
    for (int j = 0; j < 4; ++j) xv[j] = IO::gx(static_cast<const typename IO::T*>(P.x), L.c[j]);
}
template <int DT, int VAR>
__device__ __forceinline__ void short_math_f64(const MainParams& P, int cat, const ShortLd<DT>& L, const double (&xv)[4],
                                               int lane) {
    using IO = ValIO<DT>;
    if (cat == 3) {                                      // singles (Alg. 5): 4 consecutive len-1 rows
#pragma unroll
        for (int j = 0; j < 4; ++j) store_y<DT, VAR>(P, L.o[j], IO::cv(L.v[j]) * xv[j]);
        return;
    }
    const int g = lane >> 2, t = lane & 3;
    const int nseg = cat == 1 ? 1 : 2;
    const int myseg = seg_of(cat, t);
    // output o = 16j + 8s + g (two outputs per four-slot row) or 8j + g (len-4)
    const int src = 4 * (lane & 7);                      // quad of row g' = lane & 7
    double r0 = 0.0, r1 = 0.0;
#pragma unroll
    for (int j = 0; j < 4; ++j) {                        // four-slot row r = 8j + g, slot t
        for (int s = 0; s < nseg; ++s) {
            double val;
            if constexpr (vk(VAR) == VAR_MMA) {              // x masked to the segment (Alg. 4 l.7-11)
                double cc0 = 0.0, cc1 = 0.0;
                dmma(cc0, cc1, IO::cv(L.v[j]), myseg == s ? xv[j] : 0.0);
                val = __shfl_sync(FULL, (g & 1) ? cc1 : cc0, src + ((lane & 7) >> 1));
            } else {
                double p = myseg == s ? IO::cv(L.v[j]) * xv[j] : 0.0;
                p += __shfl_xor_sync(FULL, p, 1);
                p += __shfl_xor_sync(FULL, p, 2);
                val = __shfl_sync(FULL, p, src);
            }
            const int blk = nseg == 2 ? 2 * j + s : j;   // this result fills outputs 8*blk .. 8*blk+7
            if ((lane >> 3) == blk) r0 = val;
            if ((lane >> 3) == blk - 4) r1 = val;
        }
    }
    store_y<DT, VAR>(P, L.o[0], r0);
    if (nseg == 2) store_y<DT, VAR>(P, L.o[1], r1);
}

struct ShortLdH {                                    // FP16 (two m16n8k8 blocks per tile)
    uint32_t a0, a2, c[4];
    int32_t o[4];
};
__device__ __forceinline__ void short_load_f16(const MainParams& P, const ShortRef& T, int lane, uint64_t pol, ShortLdH& L) {
    const unsigned short* sv = static_cast<const unsigned short*>(P.short_val) + T.tile * 128;
    if (DASP_SINGLES_T && T.cat == 3) {   // singles L + 32 j: (a0 lo, a0 hi, a2 lo, a2 hi) = j 0..3
        uint32_t h[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            h[j] = __ldg(sv + 32 * j + lane);
            L.c[j] = ld1_b32(P.short_col + T.tile * 128 + 32 * j + lane, pol);
            L.o[j] = static_cast<int32_t>(ld1_b32(P.short_out + T.obase + 32 * j + lane, pol));
        }
        L.a0 = h[0] | (h[1] << 16);
        L.a2 = h[2] | (h[3] << 16);
        return;
    }
    ld2_b32(static_cast<const uint16_t*>(P.short_val) + T.tile * 128 + lane * 4, pol, L.a0, L.a2);
    ld4_b32(P.short_col + T.tile * 128 + lane * 4, pol, L.c);
    short_load_out(P, T, lane, pol, L.o);
}
__device__ __forceinline__ void short_gather_f16(const MainParams& P, const ShortLdH& L, uint16_t (&xh)[4]) {
    const uint16_t* x = static_cast<const uint16_t*>(P.x);
#pragma unroll
    for (int e = 0; e < 4; ++e) xh[e] = gxh(x, L.c[e]);
}
template <int VAR>
__device__ __forceinline__ void short_math_f16(const MainParams& P, int cat, const ShortLdH& L, const uint16_t (&xh)[4],
                                               int lane) {
    if (cat == 3) {                                      // singles (Alg. 5)
        const float2 lo = u2f2(L.a0), hi = u2f2(L.a2);
        const float v[4] = {lo.x, lo.y, hi.x, hi.y};
#pragma unroll
        for (int j = 0; j < 4; ++j) store_y<1, VAR>(P, L.o[j], v[j] * h2f(xh[j]));
        return;
    }
    const int g = lane >> 2, t = lane & 3;
    const int nseg = cat == 1 ? 1 : 2;
    // element e: four-slot row group q = (e<2 ? 0 : 2) + (t>>1), slot 2(t&1) + (e&1); elements
    // 0,1 are this lane's slots of m16n8k8 block 0 (rows 0-15), elements 2,3 of block 1 (16-31)
    const int seg0 = seg_of(cat, 2 * (t & 1)), seg1 = seg_of(cat, 2 * (t & 1) + 1);
    const int gs = lane & 7;                              // row g' whose result this lane collects
    float r0 = 0.f, r1 = 0.f;
    float slo[2], shi[2];
    if constexpr (vk(VAR) == VAR_CUDACORE) {
        const float2 vl = u2f2(L.a0), vh = u2f2(L.a2);
        const float p0 = vl.x * h2f(xh[0]), p1 = vl.y * h2f(xh[1]), p2 = vh.x * h2f(xh[2]), p3 = vh.y * h2f(xh[3]);
#pragma unroll
        for (int s = 0; s < 2; ++s) {
            slo[s] = (seg0 == s ? p0 : 0.f) + (seg1 == s ? p1 : 0.f);   // group t>>1
            shi[s] = (seg0 == s ? p2 : 0.f) + (seg1 == s ? p3 : 0.f);   // group 2 + (t>>1)
            slo[s] += __shfl_xor_sync(FULL, slo[s], 1);
            shi[s] += __shfl_xor_sync(FULL, shi[s], 1);
        }
    }
    for (int q = 0; q < 4; ++q) {
        for (int s = 0; s < nseg; ++s) {
            float val;
            if constexpr (vk(VAR) == VAR_MMA) {      // block q>>1, x masked to group q and segment s
                const bool mine = (q & 1) == (t >> 1);
                const bool m0 = seg0 == s, m1 = seg1 == s;
                const int eb = (q >> 1) * 2;
                const uint32_t b0 = mine ? pack2(m0 ? xh[eb] : 0, m1 ? xh[eb + 1] : 0) : 0u;
                float cc0 = 0.f, cc1 = 0.f;
                hmma(cc0, cc1, (q >> 1) ? L.a2 : L.a0, b0);
                val = __shfl_sync(FULL, (g & 1) ? cc1 : cc0, 4 * gs + (gs >> 1));
            } else {
                val = __shfl_sync(FULL, q < 2 ? slo[s] : shi[s], 4 * gs + 2 * (q & 1));
            }
            const int blk = nseg == 2 ? 2 * q + s : q;
            if ((lane >> 3) == blk) r0 = val;
            if ((lane >> 3) == blk - 4) r1 = val;
        }
    }
    store_y<1, VAR>(P, L.o[0], r0);
    if (nseg == 2) store_y<1, VAR>(P, L.o[1], r1);
}

// one tile, all three steps (split short kernel)
template <int DT, int VAR>
__device__ __forceinline__ void short_tile(const MainParams& P, const ShortRef& T, int lane, uint64_t pol) {
    if constexpr (DT == 1) {
        ShortLdH L;
        uint16_t xh[4];
        short_load_f16(P, T, lane, pol, L);
        short_gather_f16(P, L, xh);
        short_math_f16<VAR>(P, T.cat, L, xh, lane);
    } else {
        ShortLd<DT> L;
        double xv[4];
        short_load_f64<DT>(P, T, lane, pol, L);
        short_gather_f64<DT>(P, L, xv);
        short_math_f64<DT, VAR>(P, T.cat, L, xv, lane);
    }
}

// long-row phase 2 (Alg. 2 l.17-25): 8 lanes per long row (4 rows per warp), each lane sums
// the partials g0 + sl + 8j with four independent accumulators (loads in flight), then a
// 3-step shuffle tree.  The order is fixed, so results are deterministic; both the fused main
// kernel and the separate finish kernel use this routine.
template <int DT>
__device__ __forceinline__ typename Tr<DT>::A long_row_sum(const void* partial, const int64_t* group_ptr, int64_t r,
                                                           int64_t row_long, int lane) {
    using A = typename Tr<DT>::A;
    const A* part = static_cast<const A*>(partial);
    const int sl = lane & 7;
    A s0 = 0, s1 = 0, s2 = 0, s3 = 0;
    if (r < row_long) {
        const int64_t g0 = __ldg(group_ptr + r), g1 = __ldg(group_ptr + r + 1);
        int64_t k = g0 + sl;
        for (; k + 24 < g1; k += 32) { s0 += part[k]; s1 += part[k + 8]; s2 += part[k + 16]; s3 += part[k + 24]; }
        for (; k < g1; k += 8) s0 += part[k];
    }
    A s = (s0 + s1) + (s2 + s3);
    s += __shfl_xor_sync(FULL, s, 1);
    s += __shfl_xor_sync(FULL, s, 2);
    s += __shfl_xor_sync(FULL, s, 4);
    return s;
}
// empty rows (R1): y = beta*y (0 when beta == 0, y not read)
template <int DT, int VAR>
__device__ __forceinline__ void empty_row(void* yv, int32_t row, double beta, const ExtraDst& extra) {
    using Y = typename Tr<DT>::Y;
    using A = typename Tr<DT>::A;
    Y* y = static_cast<Y*>(yv);
    const Y r = beta != 0.0 ? static_cast<Y>(static_cast<A>(beta) * static_cast<A>(y[row])) : Y(0);
    y[row] = r;
    if constexpr (vs(VAR))
        for (int d = 0; d < extra.n; ++d) static_cast<Y*>(extra.ptr[d])[row] = r;
}
// finish warp fw of the fused main kernel: long rows 4fw..4fw+3, or empty rows (4 per lane)
// a row of more than kHugeGroups (1024) groups is summed by the whole warp (32 lanes, 4 accumulators each:
// 128 partials per round) instead of 8 lanes with 4 (32 per round): a row of 10^5 nonzeros (1563
// groups) takes 13 dependent rounds instead of 49, a row of 10^7 1221 instead of 4883.  Lane l sums
// partials g0 + l + 32 j into accumulator j mod 4 while 4 more remain, the rest into accumulator 0,
// then (a0+a1)+(a2+a3) and a 5-step shuffle tree: a fixed order, deterministic.
constexpr int64_t kHugeGroups = 1024;   // 128 slowed C7's phase 2 (rows of 129-313 groups): 0.0198 -> 0.0285 ms
template <int DT>
__device__ __forceinline__ typename Tr<DT>::A long_row_sum_warp(const void* partial, int64_t g0, int64_t g1, int lane) {
    using A = typename Tr<DT>::A;
    const A* part = static_cast<const A*>(partial);
    A a0 = 0, a1 = 0, a2 = 0, a3 = 0;
    int64_t k = g0 + lane;
    for (; k + 3 * 32 < g1; k += 4 * 32) { a0 += part[k]; a1 += part[k + 32]; a2 += part[k + 64]; a3 += part[k + 96]; }
    for (; k < g1; k += 32) a0 += part[k];                 // the < 4 remaining partials of this lane
    A s = (a0 + a1) + (a2 + a3);
#pragma unroll
    for (int o = 16; o >= 1; o >>= 1) s += __shfl_xor_sync(FULL, s, o);
    return s;
}
// the 4 rows of a finish warp that holds a huge row, one after the other on all 32 lanes
template <int DT, int VAR>
__device__ __forceinline__ void finish_huge(const MainParams& P, int64_t fw, int lane) {
    for (int q = 0; q < 4; ++q) {
        const int64_t rq = fw * 4 + q;
        if (rq >= P.row_long) break;
        const auto s = long_row_sum_warp<DT>(P.partial, __ldg(P.group_ptr + rq), __ldg(P.group_ptr + rq + 1), lane);
        if (lane == 0) store_y<DT, VAR>(P, __ldg(P.long_out + rq), s);
    }
}
template <int DT, int VAR>
__device__ __forceinline__ void finish_warp(const MainParams& P, int64_t fw, int lane) {
    const int64_t lw = (P.row_long + 3) / 4;
    if (fw < lw) {
        const int64_t r = fw * 4 + (lane >> 3);
        // the warp's 4 rows: any huge one?  (lane 8q reads row q's range; warp-uniform vote)
        bool huge = false;
        if ((lane & 7) == 0 && r < P.row_long) huge = __ldg(P.group_ptr + r + 1) - __ldg(P.group_ptr + r) > kHugeGroups;
        if (__any_sync(FULL, huge)) {
            finish_huge<DT, VAR>(P, fw, lane);
            return;
        }
        const auto s = long_row_sum<DT>(P.partial, P.group_ptr, r, P.row_long, lane);
        if ((lane & 7) == 0 && r < P.row_long) store_y<DT, VAR>(P, __ldg(P.long_out + r), s);
        return;
    }
    const int64_t e0 = (fw - lw) * 128 + lane * 4;
#pragma unroll
    for (int j = 0; j < 4; ++j)
        if (e0 + j < P.n0) empty_row<DT, VAR>(P.y, __ldg(P.empty_rows + e0 + j), P.beta, P.extra);
}

// short warp ws of panel D: tiles ws*TPW .. ws*TPW+TPW-1 (Alg. 4-5).  With TPW = 2 both tiles'
// loads, then both tiles' gathers are in flight before either tile's arithmetic.
template <int DT, int VAR>
__device__ __forceinline__ void short_item(const MainParams& P, const PanelDesc* D, int64_t ws, int lane, uint64_t pol) {
    const int64_t nt = __ldg(&D->t13) + __ldg(&D->t4) + __ldg(&D->t22) + __ldg(&D->ts);
    // compile-time tiles per warp (register arrays); the plan's layout may use fewer (P.tpw: an
    // FP16 plan laid out for the 5-block instantiation, run with another variant)
    constexpr int TPW = vo(VAR) ? DASP_SHORT_TPW_OCC5 : DASP_BY_DT(DT, DASP_SHORT_TPW);
    const int tpw = (DT == 1 && !vo(VAR)) ? P.tpw : TPW;   // only FP16 layouts vary (main_occ5)
    const int64_t t0 = ws * tpw;
    if (t0 >= nt || !(P.class_mask & 4)) return;
    if constexpr (TPW > 2) {   // generic: every tile's loads, then every tile's gathers, then the math
        ShortRef R[TPW];
        const int64_t te = min(t0 + tpw, nt);           // this warp's tiles [t0, te)
#pragma unroll
        for (int k = 0; k < TPW; ++k) R[k] = short_ref(D, min(t0 + k, nt - 1));
        if constexpr (DT == 1) {
            ShortLdH L[TPW];
            uint16_t xh[TPW][4];
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < te) short_load_f16(P, R[k], lane, pol, L[k]);
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < te) short_gather_f16(P, L[k], xh[k]);
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < te) short_math_f16<VAR>(P, R[k].cat, L[k], xh[k], lane);
        } else {
            ShortLd<DT> L[TPW];
            double xv[TPW][4];
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < te) short_load_f64<DT>(P, R[k], lane, pol, L[k]);
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < te) short_gather_f64<DT>(P, L[k], xv[k]);
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < te) short_math_f64<DT, VAR>(P, R[k].cat, L[k], xv[k], lane);
        }
        return;
    }
    const ShortRef A = short_ref(D, t0);
    if (TPW == 1 || tpw < 2 || t0 + 1 >= nt) { short_tile<DT, VAR>(P, A, lane, pol); return; }
    const ShortRef B = short_ref(D, t0 + 1);
    if constexpr (DT == 1) {
        ShortLdH LA, LB;
        uint16_t xa[4], xb[4];
        short_load_f16(P, A, lane, pol, LA);
        short_load_f16(P, B, lane, pol, LB);
        short_gather_f16(P, LA, xa);
        short_gather_f16(P, LB, xb);
        short_math_f16<VAR>(P, A.cat, LA, xa, lane);
        short_math_f16<VAR>(P, B.cat, LB, xb, lane);
    } else {
        ShortLd<DT> LA, LB;
        double xa[4], xb[4];
#if DASP_EXP_TRACE
        Trace tr;
        tr.start(1);
#endif
        short_load_f64<DT>(P, A, lane, pol, LA);
        short_load_f64<DT>(P, B, lane, pol, LB);
#if DASP_EXP_TRACE
        wait_on(LB.c[3] ^ LA.c[3]);
        tr.c1 = clk64();
#endif
        short_gather_f64<DT>(P, LA, xa);
        short_gather_f64<DT>(P, LB, xb);
#if DASP_EXP_TRACE
        wait_on_d(xa[3] + xb[3]);
        tr.c2 = clk64();
#endif
        short_math_f64<DT, VAR>(P, A.cat, LA, xa, lane);
        short_math_f64<DT, VAR>(P, B.cat, LB, xb, lane);
#if DASP_EXP_TRACE
        tr.finish(lane);
#endif
    }
}

// ------------------------------------------------------------------------------------------
// the fused main kernel
// Narrow row-blocks: the suffix [rbn, nrb) of a panel's sorted row-blocks in which every row
// fits in two K-slot groups (max(K nreg, longest row) <= 2K; FP64/FP32 K = 4: rows of 5-8 nonzeros, ~40 % of a
// power-law matrix's medium rows).  The warp-per-row-block path spends three dependent memory
// round trips (metadata, streams, gathers) on ~0.6 KB there; here one lane owns one row, so a
// warp works on four row-blocks side by side (lane = 8 q + g: row-block q, row g) and each lane
// issues its row's two quads in one round: a regular block's row g is 4 contiguous elements at
// 32 b + 4 g (the block-after-block ragged layout, R18, nreg <= 2 < CW), an irregular quad is the
// row's tail in irr_val.  CUDA-core arithmetic (FP64 FMA; FP32 storage widened exactly).
#ifndef DASP_NARROW_RB
#define DASP_NARROW_RB 8     // row-blocks per narrow warp (at most; MainParams::nrw): 4 side by side x 2 passes
#endif
// 1: the next pass's stream loads are issued before this pass's gathers.  Measured
// (profiles/r01d/narrow_pipe.jsonl): FP16 C3 main kernel -3 %, stencils -1 %; FP64 +6 % (spills at
// 64 registers), FP32 neutral -- so FP16 only.
#ifndef DASP_NARROW_PIPE_F64
#define DASP_NARROW_PIPE_F64 0
#endif
#ifndef DASP_NARROW_PIPE_F16
#define DASP_NARROW_PIPE_F16 0   // 1 spills the FP16 CUDA-core instantiation (off with CHUNK_PIPE_F16 0: spill-free)
#endif
#ifndef DASP_NARROW_PIPE_F32
#define DASP_NARROW_PIPE_F32 0
#endif
template <int DT> struct NarLd {                   // one pass of one lane: two K-slot groups
    typename ValIO<DT>::R v[2][4];
    uint32_t c[2][4];
    int32_t orow;
};
template <> struct NarLd<1> {                      // FP16: two octets
    uint32_t v[2][4];
    uint32_t c[2][8];
    int32_t orow;
};
// stream loads of row g of row-block rq (rq < rbe) for this lane's groups 2 sub, 2 sub + 1
template <int DT>
__device__ __forceinline__ void narrow_load(const MainParams& P, int64_t rq, bool act, int g, int sub, uint64_t pol,
                                            NarLd<DT>& L) {
    L.orow = -1;
    if (!act) {
#pragma unroll
        for (int h = 0; h < 2; ++h) {
#pragma unroll
            for (int e = 0; e < (DT == 1 ? 4 : 4); ++e) L.v[h][e] = 0;
#pragma unroll
            for (int e = 0; e < (DT == 1 ? 8 : 4); ++e) L.c[h][e] = 0xffffffffu;
        }
        return;
    }
    const int64_t i = rq * 8 + g;
    const int64_t base = __ldg(P.rb_ptr + rq), ib = __ldg(P.irr_ptr + i);
    const int ilen = static_cast<int>(__ldg(P.irr_ptr + i + 1) - ib);
    L.orow = __ldg(P.med_out + i);
    if constexpr (DT == 1) {
        const uint16_t* rv = static_cast<const uint16_t*>(P.reg_val);
        const unsigned short* iv = static_cast<const unsigned short*>(P.irr_val);
        const int nreg = static_cast<int>((__ldg(P.rb_ptr + rq + 1) - base) >> 6);
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int q = 2 * sub + h;
            if (q < nreg) {   // nreg = 4 (mid rows only): one full lane-interleaved chunk, row g at 32 g
                const int64_t off = base + (nreg >= 4 ? 32 * g + 16 * sub + 8 * h : 64 * q + 8 * g);
                ld4_b32(rv + off, pol, L.v[h]);
                ld8_b32(P.reg_col + off, pol, L.c[h]);
            } else {
                const int k0 = 8 * (q - nreg);
#pragma unroll
                for (int e = 0; e < 8; e += 2) {
                    uint32_t lo = 0, hi = 0;
                    L.c[h][e] = L.c[h][e + 1] = 0xffffffffu;
                    if (k0 + e < ilen) { lo = __ldg(iv + ib + k0 + e); L.c[h][e] = ld1_b32(P.irr_col + ib + k0 + e, pol); }
                    if (k0 + e + 1 < ilen) { hi = __ldg(iv + ib + k0 + e + 1); L.c[h][e + 1] = ld1_b32(P.irr_col + ib + k0 + e + 1, pol); }
                    L.v[h][e >> 1] = lo | (hi << 16);
                }
            }
        }
    } else {
        using IO = ValIO<DT>;
        const typename IO::T* rv = static_cast<const typename IO::T*>(P.reg_val);
        const typename IO::T* iv = static_cast<const typename IO::T*>(P.irr_val);
        const int nreg = static_cast<int>((__ldg(P.rb_ptr + rq + 1) - base) >> 5);
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int q = 2 * sub + h;
            if (q < nreg) {   // nreg = 4 (mid rows only): one full lane-interleaved chunk, row g at 16 g
                const int64_t off = base + (nreg >= 4 ? 16 * g + 8 * sub + 4 * h : 32 * q + 4 * g);
                IO::ld4r(rv + off, pol, L.v[h]);
                ld4_b32(P.reg_col + off, pol, L.c[h]);
            } else {
                const int k0 = 4 * (q - nreg);
#pragma unroll
                for (int e = 0; e < 4; ++e) {
                    L.v[h][e] = 0; L.c[h][e] = 0xffffffffu;
                    if (k0 + e < ilen) { L.v[h][e] = IO::ld1r(iv + ib + k0 + e, pol); L.c[h][e] = ld1_b32(P.irr_col + ib + k0 + e, pol); }
                }
            }
        }
    }
}
// gathers, the row's dot product (fixed order), the LPR-lane sum and the y store
template <int DT, int VAR, int LPR>
__device__ __forceinline__ void narrow_finish(const MainParams& P, const NarLd<DT>& L, int sub) {
    if constexpr (DT == 1) {
        const uint16_t* x = static_cast<const uint16_t*>(P.x);
        uint16_t xh[2][8];
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
            for (int e = 0; e < 8; ++e) xh[h][e] = gxh(x, L.c[h][e]);
        float acc = 0.f;
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const float2 av = u2f2(L.v[h][j]);
                acc = fmaf(av.x, h2f(xh[h][2 * j]), acc);
                acc = fmaf(av.y, h2f(xh[h][2 * j + 1]), acc);
            }
        if constexpr (LPR == 2) acc += __shfl_xor_sync(FULL, acc, 1);
        if (sub == 0) store_y<1, VAR>(P, L.orow, acc);        // orow -1 (inactive / virtual row): no store
    } else {
        using IO = ValIO<DT>;
        const typename IO::T* x = static_cast<const typename IO::T*>(P.x);
        double xv[2][4];
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
            for (int e = 0; e < 4; ++e) xv[h][e] = IO::gx(x, L.c[h][e]);
        double acc = 0.0;
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc = fma(IO::cv(L.v[h][e]), xv[h][e], acc);
        if constexpr (LPR == 2) acc += __shfl_xor_sync(FULL, acc, 1);
        if (sub == 0) store_y<DT, VAR>(P, L.orow, acc);
    }
}
// LPR lanes per row (1: rows spanning <= 2K slots, 4 row-blocks side by side; 2: <= 4K, 2 side
// by side), passes over [rbs, rbe) with a warp-uniform trip count (the LPR = 2 shuffle)
// A narrow warp is warp jl of a group of nwg warps that share the nrw nwg row-blocks (nrw = P.nrw)
// from gb: pass ps of warp jl covers the SIDE row-blocks gb + SIDE (jl + ps nwg) .. (nwg = 1: the
// warp's own contiguous nrw row-blocks; nwg = 8: a block's warps interleaved, so the
// block streams one contiguous region at a time).  Row-blocks >= rbe are skipped.
template <int DT, int VAR, int LPR>
__device__ __forceinline__ void medium_narrow(const MainParams& P, int64_t gb, int64_t jl, int64_t nwg, int64_t rbe,
                                              int lane, uint64_t pol) {
    constexpr int SIDE = 4 / LPR;
    const int g = (lane / LPR) & 7, sub = lane % LPR;
    const int64_t r0 = gb + SIDE * jl + lane / (8 * LPR);
    const int64_t step = SIDE * nwg;
    const int64_t passes = P.nrw / SIDE;
    if constexpr (DASP_BY_DT(DT, DASP_NARROW_PIPE) != 0) {
        NarLd<DT> A;
        narrow_load<DT>(P, r0, r0 < rbe, g, sub, pol, A);
        for (int64_t ps = 0; ps < passes; ++ps) {
            NarLd<DT> B;
            const int64_t rn = r0 + (ps + 1) * step;
            narrow_load<DT>(P, rn, ps + 1 < passes && rn < rbe, g, sub, pol, B);
            narrow_finish<DT, VAR, LPR>(P, A, sub);
            A = B;
        }
    } else {
#if DASP_EXP_TRACE
        Trace tr;
        tr.start(LPR == 1 ? 3 : 4);
#endif
        for (int64_t ps = 0; ps < passes; ++ps) {
            NarLd<DT> A;
            const int64_t rq = r0 + ps * step;
            narrow_load<DT>(P, rq, rq < rbe, g, sub, pol, A);
#if DASP_EXP_TRACE
            if (ps == 0) { wait_on(A.c[1][3] ^ A.c[0][0]); tr.c1 = clk64(); }
#endif
            narrow_finish<DT, VAR, LPR>(P, A, sub);
#if DASP_EXP_TRACE
            if (ps == 0) { __syncwarp(); tr.c2 = clk64(); }
#endif
        }
#if DASP_EXP_TRACE
        tr.finish(lane);
#endif
    }
}

// medium warp w of panel D: a wide warp (LOOP_NUM row-blocks, warp per row-block), a mid narrow
// warp (two lanes per row: rows spanning <= 4K slots) or a narrow one (a lane per row: <= 2K)
template <int DT, int VAR>
__device__ __forceinline__ void medium_warp(const MainParams& P, const PanelDesc* D, int64_t w, int lane, uint64_t pol) {
    const int64_t rbp0 = __ldg(&D->rb0), nmwd = __ldg(&D->nmwd);
    if (w < nmwd) {
        const int64_t rbe = rbp0 + __ldg(&D->rbm);
        // (MainParams::wide_il) the 8 warps of a block take their group's 8 rbw row-blocks
        // interleaved (warp j: j, j+8, ...; a short last group strides by its warp count), so at
        // any time a block streams one contiguous region instead of 8 regions rbw row-blocks apart
        const int64_t gw = w & ~int64_t(WARPS_PER_BLOCK - 1);
        const int64_t stg = P.wide_il ? min(static_cast<int64_t>(WARPS_PER_BLOCK), nmwd - gw) : 1;
        const int64_t rbs = P.wide_il ? rbp0 + gw * P.rbw + (w - gw) : rbp0 + w * P.rbw;
        const int64_t rbend = min(rbs - (w - gw) * (P.wide_il != 0) + stg * P.rbw, rbe);
        medium_rbs<DT, VAR>(P, rbs, rbend, lane, pol, stg);
        return;
    }
    const int64_t nmwm = __ldg(&D->nmwm);
    const bool mid = w < nmwm;
    const int64_t j = mid ? w - nmwd : w - nmwm;                        // warp within its class
    const int64_t rbc = rbp0 + (mid ? __ldg(&D->rbm) : __ldg(&D->rbn));  // the class's first row-block
    const int64_t rbe = rbp0 + (mid ? __ldg(&D->rbn) : __ldg(&D->nrb));
    if constexpr (vk(VAR) == VAR_CUDACORE) {
        const int64_t nwc = mid ? nmwm - nmwd : __ldg(&D->nmw) - nmwm;
        const int64_t gw = P.narrow_il ? (j & ~int64_t(WARPS_PER_BLOCK - 1)) : j;
        const int64_t nwg = P.narrow_il ? min(static_cast<int64_t>(WARPS_PER_BLOCK), nwc - gw) : 1;
        const int64_t gb = rbc + gw * P.nrw;
        if (mid) medium_narrow<DT, VAR, 2>(P, gb, j - gw, nwg, rbe, lane, pol);
        else medium_narrow<DT, VAR, 1>(P, gb, j - gw, nwg, rbe, lane, pol);
    } else {
        const int64_t rb0 = rbc + j * P.nrw, rb1 = min(rb0 + P.nrw, rbe);
        medium_rbs<DT, VAR>(P, rb0, rb1, lane, pol);   // MMA variant: the paper's warp per row-block
    }
}

// ------------------------------------------------------------------------------------------
#ifndef DASP_MIN_BLOCKS
#define DASP_MIN_BLOCKS 4   // caps registers at 64: >= 32 resident warps per SM, no spills
#endif
#ifndef DASP_MIN_BLOCKS_F16
#define DASP_MIN_BLOCKS_F16 4
#endif

#ifndef DASP_MIN_BLOCKS_F32
#define DASP_MIN_BLOCKS_F32 4
#endif
// long rows, phase 1 (Alg. 2 l.1-16), in their own launch: the unit path needs few registers
// and is gather-latency bound, so it runs at higher occupancy (40 registers, 48 warps
// per SM) than the medium path, which needs 64 (profiles/r01/long_kernel_occupancy.jsonl).  Units run in
// the column-bucketed schedule `unit_order`.
#ifndef DASP_LONG_MIN_BLOCKS
#define DASP_LONG_MIN_BLOCKS 8   // 32 registers, 64 warps/SM (C3 long -2 %, C5 -3 % vs 40 registers; profiles/r01d/long_occupancy*.jsonl)
#endif
#ifndef DASP_LONG_MIN_BLOCKS_F16
#define DASP_LONG_MIN_BLOCKS_F16 8   // 32 registers, 64 warps/SM (FP16 / FP32 long: -1..-7 %, profiles/r01d/long_occupancy.jsonl)
#endif
#ifndef DASP_LONG_MIN_BLOCKS_F32
#define DASP_LONG_MIN_BLOCKS_F32 8
#endif
template <int DT, int VAR>
__global__ void __launch_bounds__(MAIN_THREADS, DT == 0 ? DASP_LONG_MIN_BLOCKS
                                                         : (DT == 1 ? DASP_LONG_MIN_BLOCKS_F16 : DASP_LONG_MIN_BLOCKS_F32))
dasp_long_kernel(const MainParams P, int64_t n_units) {
    const int64_t w = (static_cast<int64_t>(blockIdx.x) * MAIN_THREADS + threadIdx.x) >> 5;
    if (w >= n_units) return;
    const int lane = threadIdx.x & 31;
    const uint64_t pol = stream_policy();
    const int64_t u = __ldg(P.unit_order + w);
    if constexpr (DT == 1) long_unit_f16<VAR>(P, u, lane, pol);
    else long_unit_f64<DT, VAR>(P, u, lane, pol);
}

// one main-kernel warp after the finish blocks: its role inside its panel (MainParams::warp_word);
// the descriptor fields are loaded only on the branch that needs them so they do not stay live
// (register pressure = occupancy)
template <int DT, int VAR>
__device__ __forceinline__ void main_warp(const MainParams& P, int64_t fin_blocks, int lane) {
    const int64_t gw = (static_cast<int64_t>(blockIdx.x) - fin_blocks) * WARPS_PER_BLOCK + (threadIdx.x >> 5);
    if (gw >= P.n_mwarps) return;
    const uint64_t ww = __ldg(P.warp_word + gw);
    if (ww == ~0ull) return;                             // padding slot (per-panel block alignment)
    const PanelDesc* D = P.panels + static_cast<int32_t>(ww >> 32);
    const int64_t w = static_cast<int64_t>(ww & 0xffffffffu);
    const uint64_t pol = stream_policy();
    const int64_t nmw = __ldg(&D->nmw);
    if (w < nmw) {                                       // medium rows
        if (!(P.class_mask & 2)) return;
        medium_warp<DT, VAR>(P, D, w, lane, pol);
        return;
    }
    short_item<DT, VAR>(P, D, w - nmw, lane, pol);
}

// medium row-blocks and short tiles of every panel (panel order; Alg. 3-5)
template <int DT, int VAR>
__global__ void __launch_bounds__(MAIN_THREADS, vo(VAR) ? 5
                                                         : (DT == 0 ? DASP_MIN_BLOCKS : (DT == 1 ? DASP_MIN_BLOCKS_F16 : DASP_MIN_BLOCKS_F32)))
dasp_main_kernel(const MainParams P) {
    const int lane = threadIdx.x & 31;
    const int64_t fin_blocks = (P.fin_warps + WARPS_PER_BLOCK - 1) / WARPS_PER_BLOCK;
    if (blockIdx.x < fin_blocks) {                       // long-row phase 2 + empty rows
        const int64_t fw = static_cast<int64_t>(blockIdx.x) * WARPS_PER_BLOCK + (threadIdx.x >> 5);
        if (fw < P.fin_warps) finish_warp<DT, VAR>(P, fw, lane);
        return;
    }
    if constexpr (vst(VAR)) {                            // x-window staging: before any warp returns
        stage_prologue(P, static_cast<int64_t>(blockIdx.x) - fin_blocks, static_cast<int>(sizeof(typename Tr<DT>::X)));
        main_warp<DT, VAR>(P, fin_blocks, lane);
        // the block's shared memory must outlive its bulk copies (a block whose warps gathered
        // nothing would otherwise exit with copies in flight)
        if (threadIdx.x == 0) { int32_t a, b; stage_wait(a, b); }
    } else {
        main_warp<DT, VAR>(P, fin_blocks, lane);
    }
}


template <int DT>
__global__ void dasp_scale_kernel(void* yv, int64_t m, double beta, const ExtraDst extra) {
    using Y = typename Tr<DT>::Y;
    Y* y = static_cast<Y*>(yv);
    for (int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; i < m;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x) {
        using A = typename Tr<DT>::A;
        const Y r = beta != 0.0 ? static_cast<Y>(static_cast<A>(beta) * static_cast<A>(y[i])) : Y(0);
        y[i] = r;
        for (int d = 0; d < extra.n; ++d) static_cast<Y*>(extra.ptr[d])[i] = r;
    }
}


// halo pack for the sparse x exchange: dst[k] = src[idx[k]], elements of
// E bytes moved as raw words (no arithmetic)
template <typename W>
__global__ void __launch_bounds__(256) dasp_gather_kernel(const W* __restrict__ src, const int32_t* __restrict__ idx,
                                                          int64_t n, W* __restrict__ dst) {
    for (int64_t k = static_cast<int64_t>(blockIdx.x) * 256 + threadIdx.x; k < n; k += static_cast<int64_t>(gridDim.x) * 256)
        dst[k] = src[__ldg(idx + k)];
}

}  // namespace

#if DASP_EXP_TRACE
extern "C" int dasp_exp_trace_read(void* dst, int64_t bytes, int clear) {
    const int64_t nb = bytes < kTraceWarps * 64 ? bytes : kTraceWarps * 64;
    if (cudaMemcpyFromSymbol(dst, g_trace, static_cast<size_t>(nb)) != cudaSuccess) return 4;
    if (clear) {
        void* p = nullptr;
        if (cudaGetSymbolAddress(&p, g_trace) != cudaSuccess || cudaMemset(p, 0, kTraceWarps * 64) != cudaSuccess) return 4;
    }
    return 0;
}
#endif
int short_tiles_per_warp(int dtype, bool occ5) { return occ5 ? DASP_SHORT_TPW_OCC5 : DASP_BY_DT(dtype, DASP_SHORT_TPW); }
int narrow_rb_per_warp(int) { return DASP_NARROW_RB; }

template <int DT>
static cudaError_t launch_main_dt(const MainParams& p, int variant, bool scatter, bool occ5, unsigned nb, cudaStream_t s,
                                  int stage_smem) {
    if (stage_smem > 0 && variant == VAR_CUDACORE && !scatter) {   // x-window staging instantiation
        if constexpr (DT == 1) {
            if (occ5) {
                dasp_main_kernel<DT, VAR_CUDACORE | VAR_OCC5 | VAR_STAGE><<<nb, MAIN_THREADS, stage_smem, s>>>(p);
                return cudaGetLastError();
            }
        }
        dasp_main_kernel<DT, VAR_CUDACORE | VAR_STAGE><<<nb, MAIN_THREADS, stage_smem, s>>>(p);
        return cudaGetLastError();
    }
    if constexpr (DT == 1) {
        if (occ5 && variant != VAR_MMA) {
            if (scatter) dasp_main_kernel<1, VAR_CUDACORE | VAR_SCATTER | VAR_OCC5><<<nb, MAIN_THREADS, 0, s>>>(p);
            else dasp_main_kernel<1, VAR_CUDACORE | VAR_OCC5><<<nb, MAIN_THREADS, 0, s>>>(p);
            return cudaGetLastError();
        }
    }
    if (variant == VAR_MMA) {
        if (scatter) dasp_main_kernel<DT, VAR_MMA | VAR_SCATTER><<<nb, MAIN_THREADS, 0, s>>>(p);
        else dasp_main_kernel<DT, VAR_MMA><<<nb, MAIN_THREADS, 0, s>>>(p);
    } else {
        if (scatter) dasp_main_kernel<DT, VAR_CUDACORE | VAR_SCATTER><<<nb, MAIN_THREADS, 0, s>>>(p);
        else dasp_main_kernel<DT, VAR_CUDACORE><<<nb, MAIN_THREADS, 0, s>>>(p);
    }
    return cudaGetLastError();
}

cudaError_t launch_main(const MainParams& p, int dtype, int variant, int64_t blocks, cudaStream_t s, bool occ5,
                        int stage_smem) {
    if (blocks <= 0) return cudaSuccess;
    if (blocks > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    const unsigned nb = static_cast<unsigned>(blocks);
    const bool scatter = p.extra.n > 0;
    if (!p.stage) stage_smem = 0;
    if (dtype == 0) return launch_main_dt<0>(p, variant, scatter, false, nb, s, stage_smem);
    if (dtype == 1) return launch_main_dt<1>(p, variant, scatter, occ5, nb, s, stage_smem);
    return launch_main_dt<2>(p, variant, scatter, false, nb, s, stage_smem);
}

cudaError_t launch_long(const MainParams& p, int dtype, int variant, int64_t n_units, cudaStream_t s) {
    if (n_units <= 0) return cudaSuccess;
    const int64_t blocks = (n_units * 32 + MAIN_THREADS - 1) / MAIN_THREADS;
    if (blocks > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    dim3 grid(static_cast<unsigned>(blocks)), block(MAIN_THREADS);
    const bool mma = variant == VAR_MMA;
    auto k = dtype == 0 ? (mma ? dasp_long_kernel<0, VAR_MMA> : dasp_long_kernel<0, VAR_CUDACORE>)
           : dtype == 1 ? (mma ? dasp_long_kernel<1, VAR_MMA> : dasp_long_kernel<1, VAR_CUDACORE>)
                        : (mma ? dasp_long_kernel<2, VAR_MMA> : dasp_long_kernel<2, VAR_CUDACORE>);
    k<<<grid, block, 0, s>>>(p, n_units);
    return cudaGetLastError();
}

cudaError_t launch_scale(void* y, int64_t m, double beta, int dtype, cudaStream_t s, const ExtraDst& extra) {
    if (m == 0) return cudaSuccess;
    int64_t blocks = (m + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (dtype == 0) dasp_scale_kernel<0><<<static_cast<unsigned>(blocks), 256, 0, s>>>(y, m, beta, extra);
    else if (dtype == 1) dasp_scale_kernel<1><<<static_cast<unsigned>(blocks), 256, 0, s>>>(y, m, beta, extra);
    else dasp_scale_kernel<2><<<static_cast<unsigned>(blocks), 256, 0, s>>>(y, m, beta, extra);
    return cudaGetLastError();
}

cudaError_t launch_gather(const void* src, const int32_t* idx, int64_t n, void* dst, int elem_bytes, cudaStream_t s) {
    if (n == 0) return cudaSuccess;
    int64_t blocks = (n + 255) / 256;
    if (blocks > 148 * 8) blocks = 148 * 8;
    const unsigned b = static_cast<unsigned>(blocks);
    if (elem_bytes == 8)
        dasp_gather_kernel<uint64_t><<<b, 256, 0, s>>>(static_cast<const uint64_t*>(src), idx, n, static_cast<uint64_t*>(dst));
    else if (elem_bytes == 4)
        dasp_gather_kernel<uint32_t><<<b, 256, 0, s>>>(static_cast<const uint32_t*>(src), idx, n, static_cast<uint32_t*>(dst));
    else
        dasp_gather_kernel<uint16_t><<<b, 256, 0, s>>>(static_cast<const uint16_t*>(src), idx, n, static_cast<uint16_t*>(dst));
    return cudaGetLastError();
}

}  // namespace dasp
