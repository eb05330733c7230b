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
#define DASP_CHUNK_PIPE_F16 1
#endif
#ifndef DASP_CHUNK_PIPE_F32
#define DASP_CHUNK_PIPE_F32 0
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
#define DASP_BY_DT(DT, K) ((DT) == 0 ? K##_F64 : ((DT) == 1 ? K##_F16 : K##_F32))

namespace dasp {
namespace {

constexpr unsigned FULL = 0xffffffffu;
enum { VAR_MMA = 1, VAR_CUDACORE = 2 };

// ------------------------------------------------------------------------------------------
// memory helpers
// ------------------------------------------------------------------------------------------
__device__ __forceinline__ uint64_t stream_policy() {
    uint64_t p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
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
// x gather through the read-only path; column -1 (pad, R12) reads 0 without touching memory
#ifndef DASP_GX_MODE
#define DASP_GX_MODE 0   // x gathers: 0 ld.global.nc (LDG.CONSTANT), 1 + L1::evict_last, 2 ld.global.ca
#ifndef DASP_Y_ST
#define DASP_Y_ST 0      // y stores: 0 plain, 1 st.global.cs (streaming), 2 st.global.cg
#endif
#ifndef DASP_PDL
#define DASP_PDL 0       // programmatic dependent launch between consecutive main / long kernels
#endif
#endif
// (DASP_GX_MODE 1 / 2 measured within noise on C2 / C2+ / C3 / C5, profiles/r01d/x_gather_cache_op.jsonl)
__device__ __forceinline__ double gx(const double* x, uint32_t c) {
    if constexpr (DASP_GX_MODE == 0) {
        return static_cast<int32_t>(c) >= 0 ? __ldg(x + static_cast<int32_t>(c)) : 0.0;
    } else {
        if (static_cast<int32_t>(c) < 0) return 0.0;
        const double* a = x + static_cast<int32_t>(c);
        double v;
        if constexpr (DASP_GX_MODE == 1) asm("ld.global.nc.L1::evict_last.f64 %0, [%1];" : "=d"(v) : "l"(a));
        else asm volatile("ld.global.ca.f64 %0, [%1];" : "=d"(v) : "l"(a));
        return v;
    }
}
__device__ __forceinline__ double gx_f64(const double* x, uint32_t c) { return gx(x, c); }
__device__ __forceinline__ uint16_t gxh(const uint16_t* x, uint32_t c) {
    return static_cast<int32_t>(c) >= 0 ? __ldg(reinterpret_cast<const unsigned short*>(x) + static_cast<int32_t>(c))
                                        : static_cast<uint16_t>(0);
}
// L2 bulk prefetch of a contiguous range (one instruction, no registers, no shared memory):
// addr 16-B aligned, bytes a multiple of 16 (callers pass whole 32-element regular regions)
__device__ __forceinline__ void bulk_prefetch_l2(const void* addr, uint32_t bytes) {
    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(addr), "r"(bytes) : "memory");
}
#ifndef DASP_META_L2PF
#define DASP_META_L2PF 0   // 1: wide warps L2-prefetch their metadata lines at warp start (C2 -2.5 %, C2+ +1..3 %, C5 -1 %: off)
#endif
#ifndef DASP_META_PF
#define DASP_META_PF 0     // CUDA-core wide medium warps: next row-block's metadata one row-block ahead
#endif
#ifndef DASP_BULK_PF
#define DASP_BULK_PF 0     // 1: wide medium warps L2-prefetch the next row-block's regular region (measured slower on C2 / C5, profiles/r01d/bulk_prefetch_negative.jsonl)
#endif
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
        return static_cast<int32_t>(c) >= 0 ? static_cast<double>(__ldg(x + static_cast<int32_t>(c))) : 0.0;
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

// y[row] = alpha*acc + beta*y[row] (beta == 0: y not read, R16)
template <int DT>
__device__ __forceinline__ void store_y(const MainParams& P, int32_t row, typename Tr<DT>::A acc) {
    using Y = typename Tr<DT>::Y;
    using A = typename Tr<DT>::A;
    if (row < 0) return;
    Y* y = static_cast<Y*>(P.y);
    A ra = static_cast<A>(P.alpha) * acc;                // in the accumulator type, one final rounding
    if (P.beta != 0.0) ra += static_cast<A>(P.beta) * static_cast<A>(y[row]);   // (FP32 variant, R29)
    const Y r = static_cast<Y>(ra);
#if DASP_Y_ST == 1
    __stcs(y + row, r);                                  // streaming store (evict-first in L1/L2)
#elif DASP_Y_ST == 2
    __stcg(y + row, r);                                  // cache at L2 only
#else
    y[row] = r;
#endif
    for (int d = 0; d < P.extra.n; ++d) static_cast<Y*>(P.extra.ptr[d])[row] = r;   // peers (scatter)
}

// ------------------------------------------------------------------------------------------
// co-scheduled long rows: long units run as blocks of the main kernel, so phase 2
// (Alg. 2 l.17-25) cannot wait for a kernel boundary.  A unit counts its groups off its rows'
// counters after its partials are visible; the warp that brings a row's counter to zero sums
// that row's partials.  The sum is the fixed lane-strided order of long_row_sum_warp whichever
// warp runs it, so results do not depend on the schedule (R19).
// ------------------------------------------------------------------------------------------
template <int DT>
__device__ __forceinline__ typename Tr<DT>::A long_row_sum_warp(const void* partial, int64_t g0, int64_t g1, int lane) {
    using A = typename Tr<DT>::A;
    const A* part = static_cast<const A*>(partial);
    A s0 = 0, s1 = 0, s2 = 0, s3 = 0;
    int64_t k = g0 + lane;                               // L2 reads: written by other SMs in this launch
    for (; k + 96 < g1; k += 128) { s0 += __ldcg(part + k); s1 += __ldcg(part + k + 32); s2 += __ldcg(part + k + 64); s3 += __ldcg(part + k + 96); }
    for (; k < g1; k += 32) s0 += __ldcg(part + k);
    A s = (s0 + s1) + (s2 + s3);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(FULL, s, o);
    return s;
}
template <int DT>
__device__ __forceinline__ void long_unit_complete(const MainParams& P, int64_t u, int lane) {
    __threadfence();                                     // this lane's partial store, device-wide ...
    __syncwarp();                                        // ... before any lane's counter update
    const int32_t gr = lane < 4 ? __ldg(P.group_row + u * 4 + lane) : -1;
    int32_t rr[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) rr[j] = __shfl_sync(FULL, gr, j);   // rows of groups 0..3 (non-decreasing)
    const int32_t prev = __shfl_up_sync(FULL, gr, 1);
    bool fin = false;
    if (lane < 4 && gr >= 0 && (lane == 0 || prev != gr)) {   // first group of its row in this unit
        int cnt = 0;
#pragma unroll
        for (int j = 0; j < 4; ++j) cnt += rr[j] == gr;
        fin = atomicSub(P.long_cnt + gr, cnt) == cnt;
    }
    unsigned done = __ballot_sync(FULL, fin);
    if (!done) return;
    __threadfence();                                     // acquire: other warps' partials of the row
    while (done) {
        const int j = __ffs(done) - 1;
        done &= done - 1;
        const int32_t r = __shfl_sync(FULL, gr, j);
        const int64_t g0 = __ldg(P.group_ptr + r), g1 = __ldg(P.group_ptr + r + 1);
        const auto sum = long_row_sum_warp<DT>(P.partial, g0, g1, lane);
        if (lane == 0) {
            store_y<DT>(P, __ldg(P.long_out + r), sum);
            P.long_cnt[r] = static_cast<int32_t>(g1 - g0);   // ready for the next launch
        }
    }
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
        if constexpr (VAR == VAR_MMA) {                  // trace of C_j = sum of group j (Fig. 4 diagonal)
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
    }    if (P.long_cnt) long_unit_complete<DT>(P, u, lane);
}

// FP16: lane l reads 8-B value chunks l + 32j (j = 0..3): halves 4(l+32j)..+3, all in group j
// one FP16 long unit in three steps (loads | gathers | block dots + transpose-reduce + partials),
// so a warp can hold two units' memory round trips in flight (DASP_LONG_UPW_F16)
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
        if constexpr (VAR == VAR_MMA) {
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
    if (P.long_cnt) long_unit_complete<1>(P, u, lane);
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
    double c0 = 0.0, c1 = 0.0, part = 0.0;
    if constexpr (FULL) {
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
            for (int j = 0; j < 4; ++j) xv[j] = IO::gx(x, ca[j]);
            typename IO::R vn[4];
            uint32_t cn[4];
            if (DASP_BY_DT(DT, DASP_CHUNK_PIPE) && ch + 1 < nfull) {
                IO::ld4r(rv + (ch + 1) * 128 + lane * 4, pol, vn);
                ld4_b32(rc + (ch + 1) * 128 + lane * 4, pol, cn);
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                if constexpr (VAR == VAR_MMA) dmma(c0, c1, IO::cv(va[j]), xv[j]);
                else part = fma(IO::cv(va[j]), xv[j], part);
            }
            if (DASP_BY_DT(DT, DASP_CHUNK_PIPE) && ch + 1 < nfull) {
#pragma unroll
                for (int j = 0; j < 4; ++j) { va[j] = vn[j]; ca[j] = cn[j]; }
            }
        }
    }
    double xr[3];
#pragma unroll
    for (int j = 0; j < 3; ++j) xr[j] = IO::gx(x, L.cr[j]);   // pads / unused slots read 0
    const double xi = IO::gx(x, L.ci);
#pragma unroll
    for (int j = 0; j < 3; ++j) {
        if (j < rem) {                                     // rem is warp-uniform
            if constexpr (VAR == VAR_MMA) dmma(c0, c1, IO::cv(L.vr[j]), xr[j]);
            else part = fma(IO::cv(L.vr[j]), xr[j], part);
        }
    }
    if constexpr (VAR == VAR_MMA) {                        // Alg. 3 l.13-17: diagonal -> quad g
        const double d = diag_to_quad(c0, c1, lane);
        part = t == 0 ? d : 0.0;
    }
    part = fma(IO::cv(L.vi), xi, part);                    // Alg. 3 l.20-24: irregular part
    const typename IO::T* iv = static_cast<const typename IO::T*>(P.irr_val);
    for (int64_t k = M.ib + t + 4; k < M.ib + M.ilen; k += 4)
        part = fma(IO::ld1(iv + k, pol), IO::gx(x, ld1_b32(P.irr_col + k, pol)), part);
    part += __shfl_xor_sync(FULL, part, 1);
    part += __shfl_xor_sync(FULL, part, 2);
    if (t == 0) store_y<DT>(P, M.orow, part);              // Alg. 3 l.25 through the output map (R9)
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
    float c0 = 0.f, c1 = 0.f, part = 0.f;
    // one 8x8 block: this lane's two slots 2t, 2t+1 of row g
    auto blockx = [&](uint32_t a, uint16_t xa, uint16_t xb) {
        if constexpr (VAR == VAR_MMA) {
            hmma(c0, c1, a, pack2(xa, xb));
        } else {
            const float2 av = u2f2(a);
            part = fmaf(av.x, h2f(xa), part);
            part = fmaf(av.y, h2f(xb), part);
        }
    };
    auto block = [&](uint32_t a, uint32_t ca, uint32_t cb) { blockx(a, gxh(x, ca), gxh(x, cb)); };
    if constexpr (FULL) {
        uint32_t va[4], ca[8];
#pragma unroll
        for (int j = 0; j < 4; ++j) va[j] = L.va[j];
#pragma unroll
        for (int e = 0; e < 8; ++e) ca[e] = L.ca[e];
        for (int ch = 0; ch < nfull; ++ch) {   // chunk ch+1's loads overlap chunk ch's gathers
            if (!DASP_CHUNK_PIPE_F16 && ch > 0) { ld4_b32(rv + ch * 256 + lane * 8, pol, va); ld8_b32(rc + ch * 256 + lane * 8, pol, ca); }
            uint16_t xh[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) xh[e] = gxh(x, ca[e]);
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
#pragma unroll
    for (int j = 0; j < 3; ++j)
        if (j < rem) block(L.vr[j], L.cr[2 * j], L.cr[2 * j + 1]);   // rem is warp-uniform
    if constexpr (VAR == VAR_MMA) {
        const float d = diag_to_quad(c0, c1, lane);
        part = t == 0 ? d : 0.f;
    }
    part = fmaf(h2f(L.vi), h2f(gxh(x, L.ci)), part);
    for (int64_t k = M.ib + t + 4; k < M.ib + M.ilen; k += 4)
        part = fmaf(h2f(__ldg(iv + k)), h2f(gxh(x, ld1_b32(P.irr_col + k, pol))), part);
    part += __shfl_xor_sync(FULL, part, 1);
    part += __shfl_xor_sync(FULL, part, 2);
    if (t == 0) store_y<1>(P, M.orow, part);
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

// ------------------------------------------------------------------------------------------
// medium row-blocks with cp.async staging (DASP_MED_ASYNC): the round-1 stream data of the next
// TWO row-blocks is copied into a per-warp shared-memory double buffer (LDGSTS, each lane its
// own bytes, so no cross-lane synchronisation) while the current one gathers x and reduces; the
// metadata runs two row-blocks ahead.  Bytes in flight no longer cost registers.
// Stage layout (3072 B per warp per stage, structure of arrays):
//   m8n8k4 (FP64/FP32, value size sv): VA[32][4 sv] @0, CA[32][16] @1024, VR[3][32][sv] @1536,
//                                      CR[3][32][4] @2304, VI[32][8] @2688, CI[32][4] @2944
//   FP16:                              VA[32][16] @0, CA[32][32] @512, VR[3][32][4] @1536,
//                                      CR[3][32][8] @1920, VI[32][4] @2688, CI[32][4] @2816
// ------------------------------------------------------------------------------------------
#ifndef DASP_MED_ASYNC
#define DASP_MED_ASYNC 0
#endif
constexpr int MED_STAGE = 3072;
__device__ __forceinline__ void cpa16(uint32_t dst, const void* src, uint64_t pol) {
    asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "l"(pol) : "memory");
}
__device__ __forceinline__ void cpa8(uint32_t dst, const void* src, uint64_t pol) {
    asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 8, %2;" ::"r"(dst), "l"(src), "l"(pol) : "memory");
}
__device__ __forceinline__ void cpa4(uint32_t dst, const void* src, uint64_t pol) {
    asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 4, %2;" ::"r"(dst), "l"(src), "l"(pol) : "memory");
}
__device__ __forceinline__ void cpa_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cpa_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

template <int DT>
__device__ __forceinline__ void med_issue(const MainParams& P, const RbMeta& M, int lane, uint64_t pol, uint32_t st) {
    constexpr int SH = DT == 1 ? 6 : 5;
    const int nreg = M.nelem >> SH;
    const int nfull = nreg >> 2, rem = nreg & 3;
    const int32_t* rc = P.reg_col + M.base;
    if constexpr (DT == 1) {
        const uint16_t* rv = static_cast<const uint16_t*>(P.reg_val) + M.base;
        if (nfull > 0) {
            cpa16(st + lane * 16, rv + lane * 8, pol);
            cpa16(st + 512 + lane * 32, rc + lane * 8, pol);
            cpa16(st + 512 + lane * 32 + 16, rc + lane * 8 + 4, pol);
        }
        const int64_t rb = static_cast<int64_t>(nfull) * 256 + lane * 2;
        for (int j = 0; j < rem; ++j) {
            cpa4(st + 1536 + j * 128 + lane * 4, rv + rb + 64 * j, pol);
            cpa8(st + 1920 + j * 256 + lane * 8, rc + rb + 64 * j, pol);
        }
        const int64_t k = M.ib + (lane & 3);
        if (k < M.ib + M.ilen) {   // the aligned 4-B word holding half k (arrays carry a tail pad)
            const uint16_t* iv = static_cast<const uint16_t*>(P.irr_val);
            cpa4(st + 2688 + lane * 4, iv + (k & ~int64_t(1)), pol);
            cpa4(st + 2816 + lane * 4, P.irr_col + k, pol);
        }
    } else {
        using IO = ValIO<DT>;
        constexpr int SV = sizeof(typename IO::T);
        const typename IO::T* rv = static_cast<const typename IO::T*>(P.reg_val) + M.base;
        if (nfull > 0) {
            cpa16(st + lane * 4 * SV, rv + lane * 4, pol);
            if constexpr (SV == 8) cpa16(st + lane * 32 + 16, rv + lane * 4 + 2, pol);
            cpa16(st + 1024 + lane * 16, rc + lane * 4, pol);
        }
        const int64_t rb = static_cast<int64_t>(nfull) * 128 + lane;
        for (int j = 0; j < rem; ++j) {
            if constexpr (SV == 8) cpa8(st + 1536 + j * 256 + lane * 8, rv + rb + 32 * j, pol);
            else cpa4(st + 1536 + j * 256 + lane * 4, rv + rb + 32 * j, pol);
            cpa4(st + 2304 + j * 128 + lane * 4, rc + rb + 32 * j, pol);
        }
        const int64_t k = M.ib + (lane & 3);
        if (k < M.ib + M.ilen) {
            const typename IO::T* iv = static_cast<const typename IO::T*>(P.irr_val);
            if constexpr (SV == 8) cpa8(st + 2688 + lane * 8, iv + k, pol);
            else cpa4(st + 2688 + lane * 8, iv + k, pol);
            cpa4(st + 2944 + lane * 4, P.irr_col + k, pol);
        }
    }
    cpa_commit();
}

template <int DT, int VAR>
__device__ __forceinline__ void med_compute(const MainParams& P, const RbMeta& M, int lane, uint64_t pol, const uint8_t* st) {
    const int t = lane & 3;
    constexpr int SH = DT == 1 ? 6 : 5;
    const int nreg = M.nelem >> SH;
    const int nfull = nreg >> 2, rem = nreg & 3;
    const int32_t* rc = P.reg_col + M.base;
    const bool has_i = M.ib + t < M.ib + M.ilen;
    if constexpr (DT == 1) {
        const uint16_t* rv = static_cast<const uint16_t*>(P.reg_val) + M.base;
        const unsigned short* iv = static_cast<const unsigned short*>(P.irr_val);
        const uint16_t* x = static_cast<const uint16_t*>(P.x);
        float c0 = 0.f, c1 = 0.f, part = 0.f;
        auto block = [&](uint32_t a, uint32_t ca, uint32_t cb) {
            const uint16_t xa = gxh(x, ca), xb = gxh(x, cb);
            if constexpr (VAR == VAR_MMA) {
                hmma(c0, c1, a, pack2(xa, xb));
            } else {
                const float2 av = u2f2(a);
                part = fmaf(av.x, h2f(xa), part);
                part = fmaf(av.y, h2f(xb), part);
            }
        };
        for (int ch = 0; ch < nfull; ++ch) {
            uint32_t va[4], ca[8];
            if (ch == 0) {
                const uint4 a = *reinterpret_cast<const uint4*>(st + lane * 16);
                const uint4 c0v = *reinterpret_cast<const uint4*>(st + 512 + lane * 32);
                const uint4 c1v = *reinterpret_cast<const uint4*>(st + 512 + lane * 32 + 16);
                va[0] = a.x; va[1] = a.y; va[2] = a.z; va[3] = a.w;
                ca[0] = c0v.x; ca[1] = c0v.y; ca[2] = c0v.z; ca[3] = c0v.w;
                ca[4] = c1v.x; ca[5] = c1v.y; ca[6] = c1v.z; ca[7] = c1v.w;
            } else {
                ld4_b32(rv + ch * 256 + lane * 8, pol, va);
                ld8_b32(rc + ch * 256 + lane * 8, pol, ca);
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) block(va[j], ca[2 * j], ca[2 * j + 1]);
        }
#pragma unroll
        for (int j = 0; j < 3; ++j) {
            if (j < rem) {
                const uint2 cc = *reinterpret_cast<const uint2*>(st + 1920 + j * 256 + lane * 8);
                block(*reinterpret_cast<const uint32_t*>(st + 1536 + j * 128 + lane * 4), cc.x, cc.y);
            }
        }
        if constexpr (VAR == VAR_MMA) {
            const float d = diag_to_quad(c0, c1, lane);
            part = t == 0 ? d : 0.f;
        }
        if (has_i) {
            const int64_t k = M.ib + t;
            const uint32_t wv = *reinterpret_cast<const uint32_t*>(st + 2688 + lane * 4);
            const uint16_t h = static_cast<uint16_t>((k & 1) ? (wv >> 16) : (wv & 0xffffu));
            part = fmaf(h2f(h), h2f(gxh(x, *reinterpret_cast<const uint32_t*>(st + 2816 + lane * 4))), part);
        }
        for (int64_t k = M.ib + t + 4; k < M.ib + M.ilen; k += 4)
            part = fmaf(h2f(__ldg(iv + k)), h2f(gxh(x, ld1_b32(P.irr_col + k, pol))), part);
        part += __shfl_xor_sync(FULL, part, 1);
        part += __shfl_xor_sync(FULL, part, 2);
        if (t == 0) store_y<1>(P, M.orow, part);
    } else {
        using IO = ValIO<DT>;
        constexpr int SV = sizeof(typename IO::T);
        const typename IO::T* rv = static_cast<const typename IO::T*>(P.reg_val) + M.base;
        const typename IO::T* x = static_cast<const typename IO::T*>(P.x);
        double c0 = 0.0, c1 = 0.0, part = 0.0;
        for (int ch = 0; ch < nfull; ++ch) {
            double va[4];
            uint32_t ca[4];
            if (ch == 0) {
                const typename IO::T* sv = reinterpret_cast<const typename IO::T*>(st + lane * 4 * SV);
#pragma unroll
                for (int j = 0; j < 4; ++j) va[j] = static_cast<double>(sv[j]);
                const uint4 cc = *reinterpret_cast<const uint4*>(st + 1024 + lane * 16);
                ca[0] = cc.x; ca[1] = cc.y; ca[2] = cc.z; ca[3] = cc.w;
            } else {
                IO::ld4(rv + ch * 128 + lane * 4, pol, va);
                ld4_b32(rc + ch * 128 + lane * 4, pol, ca);
            }
            double xv[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) xv[j] = IO::gx(x, ca[j]);
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                if constexpr (VAR == VAR_MMA) dmma(c0, c1, va[j], xv[j]);
                else part = fma(va[j], xv[j], part);
            }
        }
#pragma unroll
        for (int j = 0; j < 3; ++j) {
            if (j < rem) {
                const double v = static_cast<double>(*reinterpret_cast<const typename IO::T*>(st + 1536 + j * 256 + lane * SV));
                const double xv = IO::gx(x, *reinterpret_cast<const uint32_t*>(st + 2304 + j * 128 + lane * 4));
                if constexpr (VAR == VAR_MMA) dmma(c0, c1, v, xv);
                else part = fma(v, xv, part);
            }
        }
        if constexpr (VAR == VAR_MMA) {
            const double d = diag_to_quad(c0, c1, lane);
            part = t == 0 ? d : 0.0;
        }
        if (has_i) {
            const double v = static_cast<double>(*reinterpret_cast<const typename IO::T*>(st + 2688 + lane * 8));
            part = fma(v, IO::gx(x, *reinterpret_cast<const uint32_t*>(st + 2944 + lane * 4)), part);
        }
        const typename IO::T* iv = static_cast<const typename IO::T*>(P.irr_val);
        for (int64_t k = M.ib + t + 4; k < M.ib + M.ilen; k += 4)
            part = fma(IO::ld1(iv + k, pol), IO::gx(x, ld1_b32(P.irr_col + k, pol)), part);
        part += __shfl_xor_sync(FULL, part, 1);
        part += __shfl_xor_sync(FULL, part, 2);
        if (t == 0) store_y<DT>(P, M.orow, part);
    }
}

template <int DT, int VAR>
__device__ __forceinline__ void medium_rbs_async(const MainParams& P, int64_t rb0, int64_t rb1, int lane, uint64_t pol,
                                                 uint8_t* wsm) {
    const RbMeta E{0, 0, 0, 0, -1};
    const uint32_t s0 = static_cast<uint32_t>(__cvta_generic_to_shared(wsm));
    RbMeta Ma = rb_meta(P, rb0, lane);
    RbMeta Mb = rb0 + 1 < rb1 ? rb_meta(P, rb0 + 1, lane) : E;
    med_issue<DT>(P, Ma, lane, pol, s0);
    med_issue<DT>(P, Mb, lane, pol, s0 + MED_STAGE);
    int sb = 0;
    for (int64_t rb = rb0; rb < rb1; ++rb) {
        const RbMeta Mc = rb + 2 < rb1 ? rb_meta(P, rb + 2, lane) : E;
        cpa_wait<1>();
        med_compute<DT, VAR>(P, Ma, lane, pol, wsm + sb * MED_STAGE);
        med_issue<DT>(P, Mc, lane, pol, s0 + sb * MED_STAGE);
        sb ^= 1;
        Ma = Mb;
        Mb = Mc;
    }
    cpa_wait<0>();
}

// row-blocks in flight per warp step (1 or 2), per value type
#ifndef DASP_PAIR_F64
#define DASP_PAIR_F64 1
#endif
#ifndef DASP_PAIR_F16
#define DASP_PAIR_F16 1
#endif
#ifndef DASP_PAIR_F32
#define DASP_PAIR_F32 1
#endif
template <int DT> __host__ __device__ constexpr int med_pair() { return DT == 0 ? DASP_PAIR_F64 : (DT == 1 ? DASP_PAIR_F16 : DASP_PAIR_F32); }

template <int DT, int VAR>
__device__ __forceinline__ void medium_rbs(const MainParams& P, int64_t rb0, int64_t rb1, int lane, uint64_t pol,
                                           int64_t st = 1) {   // row-blocks rb0, rb0 + st, ... < rb1
    if constexpr (med_pair<DT>() == 2) {
        for (int64_t rb = rb0; rb < rb1; rb += 2 * st) {
            const RbMeta MA = rb_meta(P, rb, lane);
            const RbMeta MB = rb + st < rb1 ? rb_meta(P, rb + st, lane) : RbMeta{0, 0, 0, 0, -1};
            if constexpr (DT == 1) {
                MedLdH LA, LB;
                medium_load_f16(P, MA, lane, pol, LA);
                medium_load_f16(P, MB, lane, pol, LB);
                medium_finish_f16<VAR>(P, MA, LA, lane, pol);
                medium_finish_f16<VAR>(P, MB, LB, lane, pol);
            } else {
                MedLd<DT> LA, LB;
                medium_load_f64<DT>(P, MA, lane, pol, LA);
                medium_load_f64<DT>(P, MB, lane, pol, LB);
                medium_finish_f64<DT, VAR>(P, MA, LA, lane, pol);
                medium_finish_f64<DT, VAR>(P, MB, LB, lane, pol);
            }
        }
    } else if constexpr (DASP_BY_DT(DT, DASP_SMALL_PAIR) != 0) {
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
    } else {
        if constexpr (DASP_META_PF != 0 && VAR == VAR_CUDACORE) {
            // CUDA-core variant: row-block rb+1's metadata loads are issued before rb is processed
            // (the MMA instantiation spills with it; profiles/r01/meta_prefetch_rbw.jsonl)
            if (rb0 >= rb1) return;
            RbMeta M = rb_meta(P, rb0, lane);
            for (int64_t rb = rb0; rb < rb1; rb += st) {
                const RbMeta N = rb + st < rb1 ? rb_meta(P, rb + st, lane) : RbMeta{0, 0, 0, 0, -1};
                if constexpr (DT == 1) medium_rb_f16<VAR>(P, M, lane, pol);
                else medium_rb_f64<DT, VAR>(P, M, lane, pol);
                M = N;
            }
            return;
        }
        for (int64_t rb = rb0; rb < rb1; rb += st) {
            // (prefetching the next row-block's metadata here was measured: it costs registers
            // and spills in the FP64 MMA instantiation, net slower; profiles/r01/meta_prefetch_rbw.jsonl)
            const RbMeta M = rb_meta(P, rb, lane);
            if (DASP_BULK_PF && lane == 0 && rb + st < rb1 && M.nelem > 0) {
                // row-block rb+1's regular region starts where rb's ends and is no longer (rows
                // sorted by length): prefetch [base + nelem, base + 2 nelem) of values and columns
                const int64_t nb = M.base + M.nelem;
                bulk_prefetch_l2(static_cast<const char*>(P.reg_val) + nb * static_cast<int64_t>(sizeof(typename Tr<DT>::V)),
                                 static_cast<uint32_t>(M.nelem * sizeof(typename Tr<DT>::V)));
                bulk_prefetch_l2(P.reg_col + nb, static_cast<uint32_t>(M.nelem * 4));
            }
            if constexpr (DT == 1) medium_rb_f16<VAR>(P, M, lane, pol);
            else medium_rb_f64<DT, VAR>(P, M, lane, pol);
        }
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
__device__ __forceinline__ void short_load_out(const MainParams& P, const ShortRef& T, int lane, uint64_t pol,
                                               int32_t (&o)[4]) {
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
            L.o[j] = static_cast<int32_t>(ld1_b32(P.short_out + T.obase + 32 * j + lane, pol));
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
        for (int j = 0; j < 4; ++j) store_y<DT>(P, L.o[j], IO::cv(L.v[j]) * xv[j]);
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
            if constexpr (VAR == VAR_MMA) {              // x masked to the segment (Alg. 4 l.7-11)
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
    store_y<DT>(P, L.o[0], r0);
    if (nseg == 2) store_y<DT>(P, L.o[1], r1);
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
        for (int j = 0; j < 4; ++j) store_y<1>(P, L.o[j], v[j] * h2f(xh[j]));
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
    if constexpr (VAR == VAR_CUDACORE) {
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
            if constexpr (VAR == VAR_MMA) {      // block q>>1, x masked to group q and segment s
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
    store_y<1>(P, L.o[0], r0);
    if (nseg == 2) store_y<1>(P, L.o[1], r1);
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
template <int DT>
__device__ __forceinline__ void empty_row(void* yv, int32_t row, double beta, const ExtraDst& extra) {
    using Y = typename Tr<DT>::Y;
    using A = typename Tr<DT>::A;
    Y* y = static_cast<Y*>(yv);
    const Y r = beta != 0.0 ? static_cast<Y>(static_cast<A>(beta) * static_cast<A>(y[row])) : Y(0);
    y[row] = r;
    for (int d = 0; d < extra.n; ++d) static_cast<Y*>(extra.ptr[d])[row] = r;
}
// finish warp fw of the fused main kernel: long rows 4fw..4fw+3, or empty rows (4 per lane)
template <int DT>
__device__ __forceinline__ void finish_warp(const MainParams& P, int64_t fw, int lane) {
    const int64_t lw = (P.row_long + 3) / 4;
    if (fw < lw) {
        const int64_t r = fw * 4 + (lane >> 3);
        const auto s = long_row_sum<DT>(P.partial, P.group_ptr, r, P.row_long, lane);
        if ((lane & 7) == 0 && r < P.row_long) store_y<DT>(P, __ldg(P.long_out + r), s);
        return;
    }
    const int64_t e0 = (fw - lw) * 128 + lane * 4;
#pragma unroll
    for (int j = 0; j < 4; ++j)
        if (e0 + j < P.n0) empty_row<DT>(P.y, __ldg(P.empty_rows + e0 + j), P.beta, P.extra);
}

// short warp ws of panel D: tiles ws*TPW .. ws*TPW+TPW-1 (Alg. 4-5).  With TPW = 2 both tiles'
// loads, then both tiles' gathers are in flight before either tile's arithmetic.
template <int DT, int VAR>
__device__ __forceinline__ void short_item(const MainParams& P, const PanelDesc* D, int64_t ws, int lane, uint64_t pol) {
    const int64_t nt = __ldg(&D->t13) + __ldg(&D->t4) + __ldg(&D->t22) + __ldg(&D->ts);
    constexpr int TPW = DASP_BY_DT(DT, DASP_SHORT_TPW);
    const int64_t t0 = ws * TPW;
    if (t0 >= nt || !(P.class_mask & 4)) return;
    if constexpr (TPW > 2) {   // generic: every tile's loads, then every tile's gathers, then the math
        ShortRef R[TPW];
#pragma unroll
        for (int k = 0; k < TPW; ++k) R[k] = short_ref(D, min(t0 + k, nt - 1));
        if constexpr (DT == 1) {
            ShortLdH L[TPW];
            uint16_t xh[TPW][4];
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < nt) short_load_f16(P, R[k], lane, pol, L[k]);
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < nt) short_gather_f16(P, L[k], xh[k]);
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < nt) short_math_f16<VAR>(P, R[k].cat, L[k], xh[k], lane);
        } else {
            ShortLd<DT> L[TPW];
            double xv[TPW][4];
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < nt) short_load_f64<DT>(P, R[k], lane, pol, L[k]);
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < nt) short_gather_f64<DT>(P, L[k], xv[k]);
#pragma unroll
            for (int k = 0; k < TPW; ++k) if (t0 + k < nt) short_math_f64<DT, VAR>(P, R[k].cat, L[k], xv[k], lane);
        }
        return;
    }
    const ShortRef A = short_ref(D, t0);
    if (TPW == 1 || t0 + 1 >= nt) { short_tile<DT, VAR>(P, A, lane, pol); return; }
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
        short_load_f64<DT>(P, A, lane, pol, LA);
        short_load_f64<DT>(P, B, lane, pol, LB);
        short_gather_f64<DT>(P, LA, xa);
        short_gather_f64<DT>(P, LB, xb);
        short_math_f64<DT, VAR>(P, A.cat, LA, xa, lane);
        short_math_f64<DT, VAR>(P, B.cat, LB, xb, lane);
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
#define DASP_NARROW_PIPE_F16 1
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
template <int DT, int LPR>
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
        if (sub == 0) store_y<1>(P, L.orow, acc);        // orow -1 (inactive / virtual row): no store
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
        if (sub == 0) store_y<DT>(P, L.orow, acc);
    }
}
// LPR lanes per row (1: rows spanning <= 2K slots, 4 row-blocks side by side; 2: <= 4K, 2 side
// by side), passes over [rbs, rbe) with a warp-uniform trip count (the LPR = 2 shuffle)
// A narrow warp is warp jl of a group of nwg warps that share the nrw nwg row-blocks (nrw = P.nrw)
// from gb: pass ps of warp jl covers the SIDE row-blocks gb + SIDE (jl + ps nwg) .. (nwg = 1: the
// warp's own contiguous nrw row-blocks; nwg = 8: a block's warps interleaved, so the
// block streams one contiguous region at a time).  Row-blocks >= rbe are skipped.
template <int DT, int LPR>
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
            narrow_finish<DT, LPR>(P, A, sub);
            A = B;
        }
    } else {
        for (int64_t ps = 0; ps < passes; ++ps) {
            NarLd<DT> A;
            const int64_t rq = r0 + ps * step;
            narrow_load<DT>(P, rq, rq < rbe, g, sub, pol, A);
            narrow_finish<DT, LPR>(P, A, sub);
        }
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
        if constexpr (DASP_META_L2PF != 0) {
            // the warp's row-block metadata (irr_ptr, med_out, rb_ptr lines of its whole range) into
            // L2 with one prefetch per lane, so each row-block's metadata round trip is an L2 hit
            const int64_t r0 = rbs - (w - gw) * (P.wide_il != 0);
            const char* ip = reinterpret_cast<const char*>(P.irr_ptr + 8 * r0);
            const char* mo = reinterpret_cast<const char*>(P.med_out + 8 * r0);
            const int li = static_cast<int>((8 * (rbend - r0) * 8 + 8 + 127) >> 7);
            const int lm = static_cast<int>((8 * (rbend - r0) * 4 + 127) >> 7);
            const char* a = lane < li ? ip + 128 * lane
                          : lane < li + lm ? mo + 128 * (lane - li) : reinterpret_cast<const char*>(P.rb_ptr + r0);
            if (lane <= li + lm) asm volatile("prefetch.global.L2 [%0];" ::"l"(a));
        }
        medium_rbs<DT, VAR>(P, rbs, rbend, lane, pol, stg);
        return;
    }
    const int64_t nmwm = __ldg(&D->nmwm);
    const bool mid = w < nmwm;
    const int64_t j = mid ? w - nmwd : w - nmwm;                        // warp within its class
    const int64_t rbc = rbp0 + (mid ? __ldg(&D->rbm) : __ldg(&D->rbn));  // the class's first row-block
    const int64_t rbe = rbp0 + (mid ? __ldg(&D->rbn) : __ldg(&D->nrb));
    if constexpr (VAR == VAR_CUDACORE) {
        const int64_t nwc = mid ? nmwm - nmwd : __ldg(&D->nmw) - nmwm;
        const int64_t gw = P.narrow_il ? (j & ~int64_t(WARPS_PER_BLOCK - 1)) : j;
        const int64_t nwg = P.narrow_il ? min(static_cast<int64_t>(WARPS_PER_BLOCK), nwc - gw) : 1;
        const int64_t gb = rbc + gw * P.nrw;
        if (mid) medium_narrow<DT, 2>(P, gb, j - gw, nwg, rbe, lane, pol);
        else medium_narrow<DT, 1>(P, gb, j - gw, nwg, rbe, lane, pol);
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
#ifndef DASP_LONG_UPW_F16
#define DASP_LONG_UPW_F16 1   // FP16 long units per warp (2: both units' loads, then both gathers)
#endif
template <int DT, int VAR>
__global__ void __launch_bounds__(MAIN_THREADS, DT == 0 ? DASP_LONG_MIN_BLOCKS
                                                         : (DT == 1 ? DASP_LONG_MIN_BLOCKS_F16 : DASP_LONG_MIN_BLOCKS_F32))
dasp_long_kernel(const MainParams P, int64_t n_units) {
#if DASP_PDL
    asm volatile("griddepcontrol.wait;" ::: "memory");      // the previous grid's writes are visible
    asm volatile("griddepcontrol.launch_dependents;" :::);  // the next SpMV may be dispatched behind us
#endif
    constexpr int UPW = DT == 1 ? DASP_LONG_UPW_F16 : 1;
    const int64_t w = ((static_cast<int64_t>(blockIdx.x) * MAIN_THREADS + threadIdx.x) >> 5) * UPW;
    if (w >= n_units) return;
    const int lane = threadIdx.x & 31;
    const uint64_t pol = stream_policy();
    const int64_t u = __ldg(P.unit_order + w);
    if constexpr (DT == 1 && UPW == 2) {
        if (w + 1 < n_units) {
            const int64_t u2 = __ldg(P.unit_order + w + 1);
            LongLdH A, B;
            uint16_t xa[16], xb[16];
            long_load_f16(P, u, lane, pol, A);
            long_load_f16(P, u2, lane, pol, B);
            long_gather_f16(P, A, xa);
            long_gather_f16(P, B, xb);
            long_finish_f16<VAR>(P, u, A, xa, lane);
            long_finish_f16<VAR>(P, u2, B, xb, lane);
            return;
        }
    }
    if constexpr (DT == 1) long_unit_f16<VAR>(P, u, lane, pol);
    else long_unit_f64<DT, VAR>(P, u, lane, pol);
}

// medium row-blocks and short tiles of every panel (panel order; Alg. 3-5)
template <int DT, int VAR>
__global__ void __launch_bounds__(MAIN_THREADS, DT == 0 ? DASP_MIN_BLOCKS : (DT == 1 ? DASP_MIN_BLOCKS_F16 : DASP_MIN_BLOCKS_F32))
dasp_main_kernel(const MainParams P) {
#if DASP_PDL
    asm volatile("griddepcontrol.wait;" ::: "memory");      // the previous grid's writes are visible
    asm volatile("griddepcontrol.launch_dependents;" :::);  // the next SpMV may be dispatched behind us
#endif
    const int lane = threadIdx.x & 31;
    const int64_t fin_blocks = (P.fin_warps + WARPS_PER_BLOCK - 1) / WARPS_PER_BLOCK;
    if (blockIdx.x < fin_blocks) {                       // long-row phase 2 + empty rows
        const int64_t fw = static_cast<int64_t>(blockIdx.x) * WARPS_PER_BLOCK + (threadIdx.x >> 5);
        if (fw < P.fin_warps) finish_warp<DT>(P, fw, lane);
        return;
    }
    // role of this warp inside its panel; the descriptor fields are loaded only on the branch
    // that needs them so they do not stay live (register pressure = occupancy)
    const uint64_t bw = __ldg(P.blk_word + (static_cast<int64_t>(blockIdx.x) - fin_blocks));
    const PanelDesc* D = P.panels + static_cast<int32_t>((bw >> 32) & 0x7fffffffu);
    int64_t w = static_cast<int64_t>(bw & 0xffffffffu) * WARPS_PER_BLOCK + (threadIdx.x >> 5);
    const uint64_t pol = stream_policy();
    if (bw >> 63) {                                      // co-scheduled long units (Alg. 2)
        if (w < __ldg(&D->nunits)) {
            const int64_t u = __ldg(P.unit_order + __ldg(&D->unit0) + w);
            if constexpr (DT == 1) long_unit_f16<VAR>(P, u, lane, pol);
            else long_unit_f64<DT, VAR>(P, u, lane, pol);
        }
        return;
    }
    const int64_t nmw = __ldg(&D->nmw);
    if (w < nmw) {                                       // medium rows
        if (!(P.class_mask & 2)) return;
#if DASP_MED_ASYNC
        const int64_t rbp0 = __ldg(&D->rb0);
        const int64_t rb0 = rbp0 + w * P.rbw;
        const int64_t rb1 = min(rb0 + P.rbw, rbp0 + __ldg(&D->nrb));
        __shared__ __align__(16) uint8_t med_smem[WARPS_PER_BLOCK * 2 * MED_STAGE];
        medium_rbs_async<DT, VAR>(P, rb0, rb1, lane, pol, med_smem + (threadIdx.x >> 5) * 2 * MED_STAGE);
#else
        medium_warp<DT, VAR>(P, D, w, lane, pol);
#endif
        return;
    }
    short_item<DT, VAR>(P, D, w - nmw, lane, pol);
}

// persistent variant with a dynamic schedule: every warp takes the next work item from a
// global counter (prefetching the following one while it works), walks the panel table
// forward, and runs the same medium chunk / short tile code.  Removes the last-wave tail and
// the per-block straggler slots of the static grid; the last warp to finish resets the
// counters for the next launch.
template <int DT, int VAR>
__global__ void __launch_bounds__(MAIN_THREADS, DT == 0 ? DASP_MIN_BLOCKS : (DT == 1 ? DASP_MIN_BLOCKS_F16 : DASP_MIN_BLOCKS_F32))
dasp_main_dyn_kernel(const MainParams P, int64_t n_items) {
    const int lane = threadIdx.x & 31;
    const uint64_t pol = stream_policy();
    unsigned long long* ctr = P.sched;
    long long c = lane == 0 ? static_cast<long long>(atomicAdd(ctr, 1ull)) : 0;
    c = __shfl_sync(FULL, c, 0);
    int q = 0;
    while (c < n_items) {
        const long long nxt = lane == 0 ? static_cast<long long>(atomicAdd(ctr, 1ull)) : 0;
        if (c < P.fin_warps) {                           // long-row phase 2 + empty rows first
            finish_warp<DT>(P, c, lane);
            c = __shfl_sync(FULL, nxt, 0);
            continue;
        }
        const int64_t ci = c - P.fin_warps;
        while (ci >= __ldg(P.item_start + q + 1)) ++q;
        const PanelDesc* D = P.panels + q;
        const int64_t local = ci - __ldg(P.item_start + q);
        const int64_t nmw = __ldg(&D->nmw);
        if (local < nmw) {
            if (P.class_mask & 2) medium_warp<DT, VAR>(P, D, local, lane, pol);
        } else {
            short_item<DT, VAR>(P, D, local - nmw, lane, pol);
        }
        c = __shfl_sync(FULL, nxt, 0);
    }
    if (lane == 0) {
        __threadfence();
        const unsigned long long total = static_cast<unsigned long long>(gridDim.x) * (MAIN_THREADS / 32);
        if (atomicAdd(ctr + 1, 1ull) == total - 1) {   // every warp has made its last grab
            atomicExch(ctr, 0ull);
            atomicExch(ctr + 1, 0ull);
        }
    }
}

// short tiles in their own launch (split mode): tile_meta[t] = cat << 62 | output base
#ifndef DASP_SHORT_MIN_BLOCKS
#define DASP_SHORT_MIN_BLOCKS 6
#endif
template <int DT, int VAR>
__global__ void __launch_bounds__(MAIN_THREADS, DASP_SHORT_MIN_BLOCKS)
dasp_short_kernel(const MainParams P, const uint64_t* __restrict__ tile_meta, int64_t n_tiles) {
    const int64_t t = (static_cast<int64_t>(blockIdx.x) * MAIN_THREADS + threadIdx.x) >> 5;
    if (t >= n_tiles) return;
    const int lane = threadIdx.x & 31;
    const uint64_t pol = stream_policy();
    const uint64_t meta = __ldg(tile_meta + t);
    const int cat = static_cast<int>(meta >> 62);
    const int64_t obase = static_cast<int64_t>(meta & ((1ull << 62) - 1));
    short_tile<DT, VAR>(P, ShortRef{cat, t, obase}, lane, pol);
}

// long phase 2 (Alg. 2 l.17-25): one warp per long row, lane-strided sum of the group partials
// in a fixed order, butterfly reduction (deterministic, R19); then the empty rows (R1).
template <int DT>
__global__ void __launch_bounds__(256) dasp_finish_kernel(const FinishParams P) {
    const int lane = threadIdx.x & 31;
    const int64_t w = (static_cast<int64_t>(blockIdx.x) * 256 + threadIdx.x) / 32;
    const int64_t lw = (P.row_long + 3) / 4;
    if (w < lw) {
        using Y = typename Tr<DT>::Y;
        const int64_t r = w * 4 + (lane >> 3);
        const auto s = long_row_sum<DT>(P.partial, P.group_ptr, r, P.row_long, lane);
        if ((lane & 7) == 0 && r < P.row_long) {
            Y* y = static_cast<Y*>(P.y);
            const int32_t row = __ldg(P.long_out + r);
            using A = typename Tr<DT>::A;
            A va = static_cast<A>(P.alpha) * s;
            if (P.beta != 0.0) va += static_cast<A>(P.beta) * static_cast<A>(y[row]);
            const Y v = static_cast<Y>(va);
            y[row] = v;
            for (int d = 0; d < P.extra.n; ++d) static_cast<Y*>(P.extra.ptr[d])[row] = v;
        }
        return;
    }
    const int64_t e0 = (w - lw) * 128 + lane * 4;
#pragma unroll
    for (int j = 0; j < 4; ++j)
        if (e0 + j < P.n0) empty_row<DT>(P.y, __ldg(P.empty_rows + e0 + j), P.beta, P.extra);
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

// ==========================================================================================
// Persistent, TMA-staged pipeline.  Each warp walks the item list
// (long unit | medium row-block | short tile, panel by panel) with stride = all warps of the
// grid.  Lane 0 is the producer: NSTAGE items ahead it writes a small header into a
// shared-memory stage and issues cp.async.bulk copies of the item's packed arrays (val, col,
// output map, irregular windows) that complete on the stage's mbarrier; all 32 lanes then
// consume the stage (x gathers from global, MMA / FMA, y stores).  In-flight stream bytes
// live in shared memory instead of registers, so the SM keeps ~NSTAGE items per warp in
// flight while the gathers of the current item are outstanding.
// ==========================================================================================
#ifndef DASP_NSTAGE
#define DASP_NSTAGE 2
#endif
constexpr int NSTAGE = DASP_NSTAGE;
constexpr int STAGE = 3328;                 // bytes per stage (64 B header + up to 3264 B data)
constexpr int HDR = 64;
enum { IT_LONG = 1, IT_MED = 2, IT_SHORT = 3, IT_MED_DIRECT = 4 };

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n}" ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint64_t pol) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
        ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol) : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }

// item word (host-built, api.cu): kind in bits 62-63;
//   long: unit id | medium: row-block id | short: cat (60-61), tile (33-59), output base (0-32)
__device__ __forceinline__ int item_kind(uint64_t w) { return static_cast<int>(w >> 62); }

// medium pointers the producer needs one iteration before it issues the copies
struct MedPtr {
    int64_t base, end, irr0, irr1;
};

template <int DT>
__device__ __forceinline__ void produce(const MainParams& P, uint64_t w, const MedPtr& mp, uint8_t* st, uint64_t* bar,
                                        uint64_t pol) {
    constexpr int sv = DT == 0 ? 8 : 2;
    int64_t* h = reinterpret_cast<int64_t*>(st);
    const int kind = item_kind(w);
    const int64_t pay = static_cast<int64_t>(w & ((1ull << 62) - 1));
    if (kind == IT_LONG) {
        h[0] = IT_LONG;
        h[1] = pay;
        const uint32_t vb = 256 * 8, cb = 256 * 4;   // FP64: 256 elements; FP16: 512 elements
        const uint32_t vbytes = DT == 0 ? vb : 512 * 2, cbytes = DT == 0 ? cb : 512 * 4;
        const int64_t ne = DT == 0 ? 256 : 512;
        mbar_expect_tx(bar, vbytes + cbytes);
        bulk_g2s(st + HDR, static_cast<const uint8_t*>(P.long_val) + pay * ne * sv, vbytes, bar, pol);
        bulk_g2s(st + HDR + vbytes, P.long_col + pay * ne, cbytes, bar, pol);
    } else if (kind == IT_SHORT) {
        const int cat = static_cast<int>((pay >> 60) & 3);
        const int64_t tile = (pay >> 33) & ((1ll << 27) - 1);
        const int64_t obase = pay & ((1ll << 33) - 1);
        h[0] = IT_SHORT;
        h[1] = tile;
        h[2] = obase;
        h[3] = cat;
        const uint32_t vbytes = 128 * sv, cbytes = 128 * 4;
        const uint32_t obytes = cat == 3 ? 128 * 4 : (cat == 1 ? 32 * 4 : 64 * 4);
        mbar_expect_tx(bar, vbytes + cbytes + obytes);
        bulk_g2s(st + HDR, static_cast<const uint8_t*>(P.short_val) + tile * 128 * sv, vbytes, bar, pol);
        bulk_g2s(st + HDR + vbytes, P.short_col + tile * 128, cbytes, bar, pol);
        bulk_g2s(st + HDR + vbytes + cbytes, P.short_out + obase, obytes, bar, pol);
    } else {   // medium row-block
        constexpr int BE = DT == 0 ? 32 : 64;
        constexpr int VA = 16 / sv;                       // value elements per 16 B
        const int64_t rb = pay;
        const int64_t nreg = (mp.end - mp.base) / BE;
        const int64_t ivb = mp.irr0 & ~static_cast<int64_t>(VA - 1), ive = (mp.irr1 + VA - 1) & ~static_cast<int64_t>(VA - 1);
        const int64_t icb = mp.irr0 & ~int64_t(3), ice = (mp.irr1 + 3) & ~int64_t(3);
        const uint32_t rv = static_cast<uint32_t>(nreg * BE * sv), rc = static_cast<uint32_t>(nreg * BE * 4);
        const uint32_t iv = mp.irr1 > mp.irr0 ? static_cast<uint32_t>((ive - ivb) * sv) : 0u;
        const uint32_t ic = mp.irr1 > mp.irr0 ? static_cast<uint32_t>((ice - icb) * 4) : 0u;
        const uint32_t off_rv = HDR + 80 + 32, off_rc = off_rv + rv, off_iv = off_rc + rc, off_ic = off_iv + iv;
        h[1] = rb;
        h[2] = nreg;
        h[3] = ivb;
        h[4] = icb;
        h[5] = off_iv;
        h[6] = off_ic;
        if (off_ic + ic > STAGE) {                       // does not fit: consumer reads global
            h[0] = IT_MED_DIRECT;
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
            return;
        }
        h[0] = IT_MED;
        mbar_expect_tx(bar, 80 + 32 + rv + rc + iv + ic);
        bulk_g2s(st + HDR, P.irr_ptr + rb * 8, 80, bar, pol);            // irr_ptr[8rb .. 8rb+9]
        bulk_g2s(st + HDR + 80, P.med_out + rb * 8, 32, bar, pol);
        if (rv) {
            bulk_g2s(st + off_rv, static_cast<const uint8_t*>(P.reg_val) + mp.base * sv, rv, bar, pol);
            bulk_g2s(st + off_rc, P.reg_col + mp.base, rc, bar, pol);
        }
        if (iv) {
            bulk_g2s(st + off_iv, static_cast<const uint8_t*>(P.irr_val) + ivb * sv, iv, bar, pol);
            bulk_g2s(st + off_ic, P.irr_col + icb, ic, bar, pol);
        }
    }
}

// ---- consumers (all 32 lanes), FP64 ----
template <int VAR>
__device__ __forceinline__ void long_stage_f64(const MainParams& P, const uint8_t* st, int64_t u, int lane) {
    // conflict-free reads: lane l takes 16-B chunks l + 32j, i.e. elements 2(l+32j), 2(l+32j)+1,
    // both in group j of the unit
    const double2* sv = reinterpret_cast<const double2*>(st + HDR);
    const int2* sc = reinterpret_cast<const int2*>(st + HDR + 2048);
    const double* x = static_cast<const double*>(P.x);
    double v[8], xv[8];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        const double2 a = sv[j * 32 + lane];
        const int2 c = sc[j * 32 + lane];
        v[2 * j] = a.x; v[2 * j + 1] = a.y;
        xv[2 * j] = gx(x, static_cast<uint32_t>(c.x));
        xv[2 * j + 1] = gx(x, static_cast<uint32_t>(c.y));
    }
    double gsum[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        if constexpr (VAR == VAR_MMA) {
            double c0 = 0.0, c1 = 0.0;
            dmma(c0, c1, v[2 * j], xv[2 * j]);
            dmma(c0, c1, v[2 * j + 1], xv[2 * j + 1]);
            gsum[j] = is_diag_holder(lane) ? (((lane >> 2) & 1) ? c1 : c0) : 0.0;   // trace terms
        } else {
            gsum[j] = fma(v[2 * j], xv[2 * j], v[2 * j + 1] * xv[2 * j + 1]);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1)
#pragma unroll
        for (int j = 0; j < 4; ++j) gsum[j] += __shfl_xor_sync(FULL, gsum[j], o);
    if (lane < 4) static_cast<double*>(P.partial)[u * 4 + lane] = lane == 0 ? gsum[0] : lane == 1 ? gsum[1] : lane == 2 ? gsum[2] : gsum[3];
}

template <int VAR>
__device__ __forceinline__ void short_compute_f64(const MainParams& P, int cat, const double (&v)[4], const uint32_t (&c)[4],
                                                  int32_t o0, int32_t o1, int lane) {
    const int g = lane >> 2, t = lane & 3;
    const int nseg = cat == 1 ? 1 : 2;
    const double* x = static_cast<const double*>(P.x);
    double xv[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) xv[j] = gx(x, c[j]);
    const int myseg = seg_of(cat, t);
    const int src = 4 * (lane & 7);
    double r0 = 0.0, r1 = 0.0;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        for (int s = 0; s < nseg; ++s) {
            double val;
            if constexpr (VAR == VAR_MMA) {
                double cc0 = 0.0, cc1 = 0.0;
                dmma(cc0, cc1, v[j], myseg == s ? xv[j] : 0.0);
                val = __shfl_sync(FULL, (g & 1) ? cc1 : cc0, src + ((lane & 7) >> 1));
            } else {
                double p = myseg == s ? v[j] * xv[j] : 0.0;
                p += __shfl_xor_sync(FULL, p, 1);
                p += __shfl_xor_sync(FULL, p, 2);
                val = __shfl_sync(FULL, p, src);
            }
            const int blk = nseg == 2 ? 2 * j + s : j;
            if ((lane >> 3) == blk) r0 = val;
            if ((lane >> 3) == blk - 4) r1 = val;
        }
    }
    store_y<0>(P, o0, r0);
    if (nseg == 2) store_y<0>(P, o1, r1);
}

template <int VAR>
__device__ __forceinline__ void short_stage_f64(const MainParams& P, const uint8_t* st, int cat, int lane) {
    const double2* sv = reinterpret_cast<const double2*>(st + HDR);
    const uint4* sc = reinterpret_cast<const uint4*>(st + HDR + 1024);
    const int32_t* so = reinterpret_cast<const int32_t*>(st + HDR + 1024 + 512);
    const double2 a = sv[2 * lane], b = sv[2 * lane + 1];
    const uint4 cc = sc[lane];
    const double v[4] = {a.x, a.y, b.x, b.y};
    const uint32_t c[4] = {cc.x, cc.y, cc.z, cc.w};
    if (cat == 3) {                                       // singles (Alg. 5)
        const int4 o = reinterpret_cast<const int4*>(so)[lane];
        const double* x = static_cast<const double*>(P.x);
        store_y<0>(P, o.x, v[0] * gx(x, c[0]));
        store_y<0>(P, o.y, v[1] * gx(x, c[1]));
        store_y<0>(P, o.z, v[2] * gx(x, c[2]));
        store_y<0>(P, o.w, v[3] * gx(x, c[3]));
        return;
    }
    short_compute_f64<VAR>(P, cat, v, c, so[lane], cat == 1 ? -1 : so[32 + lane], lane);
}

template <int VAR>
__device__ __forceinline__ void medium_stage_f64(const MainParams& P, const uint8_t* st, int lane) {
    const int64_t* h = reinterpret_cast<const int64_t*>(st);
    const int g = lane >> 2, t = lane & 3;
    const int nreg = static_cast<int>(h[2]);
    const int64_t ivb = h[3], icb = h[4];
    const double* siv = reinterpret_cast<const double*>(st + h[5]);
    const int32_t* sic = reinterpret_cast<const int32_t*>(st + h[6]);
    const int64_t* sip = reinterpret_cast<const int64_t*>(st + HDR);
    const int32_t orow = reinterpret_cast<const int32_t*>(st + HDR + 80)[g];
    const double* srv = reinterpret_cast<const double*>(st + HDR + 112);
    const int32_t* src = reinterpret_cast<const int32_t*>(st + HDR + 112 + nreg * 256);
    const double* x = static_cast<const double*>(P.x);
    const int nfull = nreg >> 2, rem = nreg & 3;
    double c0 = 0.0, c1 = 0.0, part = 0.0;
    for (int ch = 0; ch < nfull; ++ch) {
        const double2 a = reinterpret_cast<const double2*>(srv + ch * 128 + lane * 4)[0];
        const double2 b = reinterpret_cast<const double2*>(srv + ch * 128 + lane * 4)[1];
        const uint4 cc = reinterpret_cast<const uint4*>(src + ch * 128 + lane * 4)[0];
        const double va[4] = {a.x, a.y, b.x, b.y};
        const uint32_t ca[4] = {cc.x, cc.y, cc.z, cc.w};
        double xv[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) xv[j] = gx(x, ca[j]);
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            if constexpr (VAR == VAR_MMA) dmma(c0, c1, va[j], xv[j]);
            else part = fma(va[j], xv[j], part);
        }
    }
    const int rbase = nfull * 128 + lane;                // ragged chunk: block j at 32j (R18)
#pragma unroll
    for (int j = 0; j < 3; ++j) {
        if (j < rem) {                                     // rem is warp-uniform
            const double xv = gx(x, static_cast<uint32_t>(src[rbase + 32 * j]));
            if constexpr (VAR == VAR_MMA) dmma(c0, c1, srv[rbase + 32 * j], xv);
            else part = fma(srv[rbase + 32 * j], xv, part);
        }
    }
    if constexpr (VAR == VAR_MMA) {
        const double d = diag_to_quad(c0, c1, lane);
        part = t == 0 ? d : 0.0;
    }
    const int64_t ie = sip[g + 1];
    for (int64_t k = sip[g] + t; k < ie; k += 4) part = fma(siv[k - ivb], gx(x, static_cast<uint32_t>(sic[k - icb])), part);
    part += __shfl_xor_sync(FULL, part, 1);
    part += __shfl_xor_sync(FULL, part, 2);
    if (t == 0) store_y<0>(P, orow, part);
}

// ---- consumers, FP16 ----
template <int VAR>
__device__ __forceinline__ void long_stage_f16(const MainParams& P, const uint8_t* st, int64_t u, int lane) {
    // lane l takes halves 8l..8l+7 (group l/16) and 256+8l.. (group 2 + l/16)
    const uint4* sv = reinterpret_cast<const uint4*>(st + HDR);
    const uint4* sc = reinterpret_cast<const uint4*>(st + HDR + 1024);
    const uint16_t* x = static_cast<const uint16_t*>(P.x);
    float gs[2];
#pragma unroll
    for (int j = 0; j < 2; ++j) {
        const uint4 a = sv[lane + 32 * j];
        const uint4 ca = sc[2 * lane + 64 * j], cb = sc[2 * lane + 64 * j + 1];
        const uint32_t av[4] = {a.x, a.y, a.z, a.w};
        const uint32_t cv[8] = {ca.x, ca.y, ca.z, ca.w, cb.x, cb.y, cb.z, cb.w};
        uint16_t xh[8];
#pragma unroll
        for (int e = 0; e < 8; ++e) xh[e] = gxh(x, cv[e]);
        if constexpr (VAR == VAR_MMA) {
            float c0 = 0.f, c1 = 0.f;
#pragma unroll
            for (int h = 0; h < 4; ++h) hmma(c0, c1, av[h], pack2(xh[2 * h], xh[2 * h + 1]));
            gs[j] = is_diag_holder(lane) ? (((lane >> 2) & 1) ? c1 : c0) : 0.f;
        } else {
            float s = 0.f;
#pragma unroll
            for (int h = 0; h < 4; ++h) {
                const float2 af = u2f2(av[h]);
                s = fmaf(af.x, h2f(xh[2 * h]), s);
                s = fmaf(af.y, h2f(xh[2 * h + 1]), s);
            }
            gs[j] = s;
        }
    }
#pragma unroll
    for (int o = 8; o > 0; o >>= 1) {
        gs[0] += __shfl_xor_sync(FULL, gs[0], o);
        gs[1] += __shfl_xor_sync(FULL, gs[1], o);
    }
    if ((lane & 15) == 0) {
        float* part = static_cast<float*>(P.partial) + u * 4 + (lane >> 4);
        part[0] = gs[0];   // group lane/16
        part[2] = gs[1];   // group 2 + lane/16
    }
}

template <int VAR>
__device__ __forceinline__ void short_stage_f16(const MainParams& P, const uint8_t* st, int cat, int lane) {
    const uint2 a = reinterpret_cast<const uint2*>(st + HDR)[lane];
    const uint4 cc = reinterpret_cast<const uint4*>(st + HDR + 256)[lane];
    const int32_t* so = reinterpret_cast<const int32_t*>(st + HDR + 256 + 512);
    const uint32_t c[4] = {cc.x, cc.y, cc.z, cc.w};
    const uint16_t* x = static_cast<const uint16_t*>(P.x);
    if (cat == 3) {
        const int4 o = reinterpret_cast<const int4*>(so)[lane];
        const float2 lo = u2f2(a.x), hi = u2f2(a.y);
        store_y<1>(P, o.x, lo.x * h2f(gxh(x, c[0])));
        store_y<1>(P, o.y, lo.y * h2f(gxh(x, c[1])));
        store_y<1>(P, o.z, hi.x * h2f(gxh(x, c[2])));
        store_y<1>(P, o.w, hi.y * h2f(gxh(x, c[3])));
        return;
    }
    ShortLdH L;
    L.a0 = a.x;
    L.a2 = a.y;
#pragma unroll
    for (int e = 0; e < 4; ++e) L.c[e] = c[e];
    L.o[0] = so[lane];
    L.o[1] = cat == 1 ? -1 : so[32 + lane];
    L.o[2] = L.o[3] = -1;
    uint16_t xh[4];
    short_gather_f16(P, L, xh);
    short_math_f16<VAR>(P, cat, L, xh, lane);
}

template <int VAR>
__device__ __forceinline__ void medium_stage_f16(const MainParams& P, const uint8_t* st, int lane) {
    const int64_t* h = reinterpret_cast<const int64_t*>(st);
    const int g = lane >> 2, t = lane & 3;
    const int nreg = static_cast<int>(h[2]);
    const int64_t ivb = h[3], icb = h[4];
    const unsigned short* siv = reinterpret_cast<const unsigned short*>(st + h[5]);
    const int32_t* sic = reinterpret_cast<const int32_t*>(st + h[6]);
    const int64_t* sip = reinterpret_cast<const int64_t*>(st + HDR);
    const int32_t orow = reinterpret_cast<const int32_t*>(st + HDR + 80)[g];
    const uint32_t* srv = reinterpret_cast<const uint32_t*>(st + HDR + 112);      // half pairs
    const int32_t* src = reinterpret_cast<const int32_t*>(st + HDR + 112 + nreg * 128);
    const uint16_t* x = static_cast<const uint16_t*>(P.x);
    float c0 = 0.f, c1 = 0.f, part = 0.f;
    auto block = [&](uint32_t a, uint32_t ca, uint32_t cb) {
        const uint16_t xa = gxh(x, ca), xb = gxh(x, cb);
        if constexpr (VAR == VAR_MMA) {
            hmma(c0, c1, a, pack2(xa, xb));
        } else {
            const float2 av = u2f2(a);
            part = fmaf(av.x, h2f(xa), part);
            part = fmaf(av.y, h2f(xb), part);
        }
    };
    const int nfull = nreg >> 2, rem = nreg & 3;
    for (int ch = 0; ch < nfull; ++ch) {             // chunk: lane holds 4 half pairs + 8 columns
        const uint4 a = reinterpret_cast<const uint4*>(srv + ch * 128 + lane * 4)[0];
        const uint4 ca = reinterpret_cast<const uint4*>(src + ch * 256 + lane * 8)[0];
        const uint4 cb = reinterpret_cast<const uint4*>(src + ch * 256 + lane * 8)[1];
        block(a.x, ca.x, ca.y);
        block(a.y, ca.z, ca.w);
        block(a.z, cb.x, cb.y);
        block(a.w, cb.z, cb.w);
    }
#pragma unroll
    for (int j = 0; j < 3; ++j) {
        if (j < rem) {
            const int e = nfull * 128 + 32 * j + lane;     // half-pair index (ragged chunk, R18)
            block(srv[e], static_cast<uint32_t>(src[2 * e]), static_cast<uint32_t>(src[2 * e + 1]));
        }
    }
    if constexpr (VAR == VAR_MMA) {
        const float d = diag_to_quad(c0, c1, lane);
        part = t == 0 ? d : 0.f;
    }
    const int64_t ie = sip[g + 1];
    for (int64_t k = sip[g] + t; k < ie; k += 4)
        part = fmaf(h2f(siv[k - ivb]), h2f(gxh(x, static_cast<uint32_t>(sic[k - icb]))), part);
    part += __shfl_xor_sync(FULL, part, 1);
    part += __shfl_xor_sync(FULL, part, 2);
    if (t == 0) store_y<1>(P, orow, part);
}

#ifndef DASP_PIPE_WARPS
#define DASP_PIPE_WARPS 8
#endif
constexpr int PW = DASP_PIPE_WARPS;

template <int DT, int VAR>
__global__ void __launch_bounds__(PW * 32) dasp_pipe_kernel(const MainParams P, const uint64_t* __restrict__ items,
                                                           int64_t n_items) {
    extern __shared__ __align__(128) uint8_t smem[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint8_t* stages = smem + warp * NSTAGE * STAGE;
    uint64_t* bars = reinterpret_cast<uint64_t*>(smem + PW * NSTAGE * STAGE) + warp * NSTAGE;
    const int64_t NW = static_cast<int64_t>(gridDim.x) * PW;
    const int64_t w0 = static_cast<int64_t>(blockIdx.x) * PW + warp;
    const uint64_t pol = stream_policy();
    if (w0 >= n_items) return;

    // producer state (lane 0): item words and medium pointers, one item of look-ahead
    uint64_t wa = 0, wb = 0;
    MedPtr ma{0, 0, 0, 0}, mb{0, 0, 0, 0};
    auto load_ptrs = [&](uint64_t w, MedPtr& m) {
        if (item_kind(w) == IT_MED) {
            const int64_t rb = static_cast<int64_t>(w & ((1ull << 62) - 1));
            m.base = __ldg(P.rb_ptr + rb); m.end = __ldg(P.rb_ptr + rb + 1);
            m.irr0 = __ldg(P.irr_ptr + rb * 8); m.irr1 = __ldg(P.irr_ptr + rb * 8 + 8);
        }
    };
    if (lane == 0) {
        for (int s = 0; s < NSTAGE; ++s) mbar_init(&bars[s], 1);
        fence_mbar_init();
        fence_proxy_async();
        for (int s = 0; s < NSTAGE; ++s) {
            const int64_t i = w0 + s * NW;
            if (i < n_items) {
                uint64_t w = __ldg(items + i);
                MedPtr m{0, 0, 0, 0};
                load_ptrs(w, m);
                produce<DT>(P, w, m, stages + s * STAGE, &bars[s], pol);
            }
        }
        const int64_t ia = w0 + NSTAGE * NW, ib = ia + NW;
        if (ia < n_items) { wa = __ldg(items + ia); load_ptrs(wa, ma); }
        if (ib < n_items) wb = __ldg(items + ib);
    }
    __syncwarp();
    for (int64_t k = 0;; ++k) {
        const int64_t i = w0 + k * NW;
        if (i >= n_items) break;
        const int s = static_cast<int>(k % NSTAGE);
        uint8_t* st = stages + s * STAGE;
        mbar_wait(&bars[s], static_cast<uint32_t>((k / NSTAGE) & 1));
        const int64_t* h = reinterpret_cast<const int64_t*>(st);
        const int kind = static_cast<int>(h[0]);
        if (kind == IT_LONG) {
            if constexpr (DT == 0) long_stage_f64<VAR>(P, st, h[1], lane);
            else long_stage_f16<VAR>(P, st, h[1], lane);
        } else if (kind == IT_SHORT) {
            if constexpr (DT == 0) short_stage_f64<VAR>(P, st, static_cast<int>(h[3]), lane);
            else short_stage_f16<VAR>(P, st, static_cast<int>(h[3]), lane);
        } else if (kind == IT_MED) {
            if constexpr (DT == 0) medium_stage_f64<VAR>(P, st, lane);
            else medium_stage_f16<VAR>(P, st, lane);
        } else {                                          // row-block larger than a stage
            if constexpr (DT == 0) medium_rb_f64<0, VAR>(P, rb_meta(P, h[1], lane), lane, pol);
            else medium_rb_f16<VAR>(P, rb_meta(P, h[1], lane), lane, pol);
        }
        __syncwarp();
        if (lane == 0) {
            const int64_t inext = i + NSTAGE * NW;
            if (inext < n_items) {
                fence_proxy_async();                      // our generic reads of the stage precede the refill
                produce<DT>(P, wa, ma, st, &bars[s], pol);
                wa = wb;
                ma = MedPtr{0, 0, 0, 0};
                load_ptrs(wa, ma);
                const int64_t ic = inext + 2 * NW;
                wb = ic < n_items ? __ldg(items + ic) : 0;
            }
        }
        __syncwarp();
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

// DASP_CARVEOUT >= 0: preferred shared-memory carveout (percent) set once per kernel before its
// first launch (experiment knob; -1 leaves the driver's choice)
#ifndef DASP_CARVEOUT
#define DASP_CARVEOUT -1
#endif
static void set_carveout(const void* k) {
#if DASP_CARVEOUT >= 0
    static const void* done[32] = {};
    for (int i = 0; i < 32; ++i) {
        if (done[i] == k) return;
        if (!done[i]) {
            cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, DASP_CARVEOUT);
            done[i] = k;
            return;
        }
    }
#else
    (void)k;
#endif
}

template <typename Kern, typename... Args>
static cudaError_t launch_ex(Kern kernel, unsigned blocks, cudaStream_t s, const void* apw_base, size_t apw_bytes,
                             float apw_hit, Args... args) {
    set_carveout(reinterpret_cast<const void*>(kernel));
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(blocks);
    cfg.blockDim = dim3(MAIN_THREADS);
    cfg.stream = s;
    cudaLaunchAttribute attr[2];
    unsigned na = 0;
    if (apw_bytes) {
        attr[na].id = cudaLaunchAttributeAccessPolicyWindow;
        attr[na].val.accessPolicyWindow.base_ptr = const_cast<void*>(apw_base);
        attr[na].val.accessPolicyWindow.num_bytes = apw_bytes;
        attr[na].val.accessPolicyWindow.hitRatio = apw_hit;
        attr[na].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        attr[na].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        ++na;
    }
#if DASP_PDL
    attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
#endif
    if (na) {
        cfg.attrs = attr;
        cfg.numAttrs = na;
    }
    return cudaLaunchKernelEx(&cfg, kernel, args...);
}

namespace {
// one warp per long row: its group count and the row index of each of its groups
__global__ void __launch_bounds__(256) dasp_long_meta_kernel(const int64_t* __restrict__ group_ptr, int64_t row_long,
                                                             int32_t* __restrict__ long_cnt, int32_t* __restrict__ group_row) {
    const int64_t r = (static_cast<int64_t>(blockIdx.x) * 256 + threadIdx.x) >> 5;
    if (r >= row_long) return;
    const int lane = threadIdx.x & 31;
    const int64_t g0 = group_ptr[r], g1 = group_ptr[r + 1];
    if (lane == 0) long_cnt[r] = static_cast<int32_t>(g1 - g0);
    for (int64_t g = g0 + lane; g < g1; g += 32) group_row[g] = static_cast<int32_t>(r);
}
}  // namespace

int short_tiles_per_warp(int dtype) { return DASP_BY_DT(dtype, DASP_SHORT_TPW); }
#ifndef DASP_NARROW_F16
#define DASP_NARROW_F16 1
#endif
int narrow_rb_per_warp(int dtype) { return (DASP_MED_ASYNC || (dtype == 1 && !DASP_NARROW_F16)) ? 0 : DASP_NARROW_RB; }

cudaError_t launch_long_meta(const int64_t* group_ptr, int64_t row_long, int32_t* long_cnt, int32_t* group_row,
                             cudaStream_t s) {
    if (row_long <= 0) return cudaSuccess;
    const int64_t blocks = (row_long * 32 + 255) / 256;
    if (blocks > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    dasp_long_meta_kernel<<<static_cast<unsigned>(blocks), 256, 0, s>>>(group_ptr, row_long, long_cnt, group_row);
    return cudaGetLastError();
}

cudaError_t launch_main(const MainParams& p, int dtype, int variant, int64_t blocks, cudaStream_t s,
                        const void* apw_base, size_t apw_bytes, float apw_hit) {
    if (blocks <= 0) return cudaSuccess;
    if (blocks > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    const unsigned nb = static_cast<unsigned>(blocks);
    cudaError_t e;
    const bool mma = variant == VAR_MMA;
#if DASP_MED_ASYNC
    static bool carve[3][2] = {};                      // 4 blocks x 48 KB staging per SM
    if (!carve[dtype][mma]) {
        const void* k = dtype == 0 ? (mma ? (const void*)dasp_main_kernel<0, VAR_MMA> : (const void*)dasp_main_kernel<0, VAR_CUDACORE>)
                      : dtype == 1 ? (mma ? (const void*)dasp_main_kernel<1, VAR_MMA> : (const void*)dasp_main_kernel<1, VAR_CUDACORE>)
                                   : (mma ? (const void*)dasp_main_kernel<2, VAR_MMA> : (const void*)dasp_main_kernel<2, VAR_CUDACORE>);
        cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, cudaSharedmemCarveoutMaxShared);
        carve[dtype][mma] = true;
    }
#endif
    if (dtype == 0) e = launch_ex(mma ? dasp_main_kernel<0, VAR_MMA> : dasp_main_kernel<0, VAR_CUDACORE>, nb, s, apw_base, apw_bytes, apw_hit, p);
    else if (dtype == 1) e = launch_ex(mma ? dasp_main_kernel<1, VAR_MMA> : dasp_main_kernel<1, VAR_CUDACORE>, nb, s, apw_base, apw_bytes, apw_hit, p);
    else e = launch_ex(mma ? dasp_main_kernel<2, VAR_MMA> : dasp_main_kernel<2, VAR_CUDACORE>, nb, s, apw_base, apw_bytes, apw_hit, p);
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

cudaError_t launch_main_dyn(const MainParams& p, int dtype, int variant, int64_t blocks, int64_t n_items, cudaStream_t s) {
    if (blocks <= 0 || n_items <= 0) return cudaSuccess;
    const unsigned nb = static_cast<unsigned>(blocks);
    const bool mma = variant == VAR_MMA;
    if (dtype == 0) (mma ? dasp_main_dyn_kernel<0, VAR_MMA> : dasp_main_dyn_kernel<0, VAR_CUDACORE>)<<<nb, MAIN_THREADS, 0, s>>>(p, n_items);
    else if (dtype == 1) (mma ? dasp_main_dyn_kernel<1, VAR_MMA> : dasp_main_dyn_kernel<1, VAR_CUDACORE>)<<<nb, MAIN_THREADS, 0, s>>>(p, n_items);
    else (mma ? dasp_main_dyn_kernel<2, VAR_MMA> : dasp_main_dyn_kernel<2, VAR_CUDACORE>)<<<nb, MAIN_THREADS, 0, s>>>(p, n_items);
    return cudaGetLastError();
}

cudaError_t main_dyn_occupancy(int dtype, int variant, int* bps) {
    const bool mma = variant == VAR_MMA;
    if (dtype == 0)
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, mma ? dasp_main_dyn_kernel<0, VAR_MMA> : dasp_main_dyn_kernel<0, VAR_CUDACORE>, MAIN_THREADS, 0);
    if (dtype == 1)
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, mma ? dasp_main_dyn_kernel<1, VAR_MMA> : dasp_main_dyn_kernel<1, VAR_CUDACORE>, MAIN_THREADS, 0);
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(bps, mma ? dasp_main_dyn_kernel<2, VAR_MMA> : dasp_main_dyn_kernel<2, VAR_CUDACORE>, MAIN_THREADS, 0);
}

template <int DT, int VAR>
static cudaError_t pipe_setup(int* blocks_per_sm) {
    const size_t smem = pipe_smem_bytes();
    cudaError_t e = cudaFuncSetAttribute(dasp_pipe_kernel<DT, VAR>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         static_cast<int>(smem));
    if (e != cudaSuccess) return e;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, dasp_pipe_kernel<DT, VAR>, PW * 32, smem);
}

size_t pipe_smem_bytes() { return static_cast<size_t>(PW) * NSTAGE * (STAGE + 8); }
int pipe_warps_per_block() { return PW; }

cudaError_t pipe_occupancy(int dtype, int variant, int* blocks_per_sm) {
    if (dtype == 0) return variant == VAR_MMA ? pipe_setup<0, VAR_MMA>(blocks_per_sm) : pipe_setup<0, VAR_CUDACORE>(blocks_per_sm);
    return variant == VAR_MMA ? pipe_setup<1, VAR_MMA>(blocks_per_sm) : pipe_setup<1, VAR_CUDACORE>(blocks_per_sm);
}

cudaError_t launch_pipe(const MainParams& p, int dtype, int variant, const uint64_t* items, int64_t n_items,
                        int64_t blocks, cudaStream_t s) {
    if (n_items <= 0 || blocks <= 0) return cudaSuccess;
    const size_t smem = pipe_smem_bytes();
    dim3 grid(static_cast<unsigned>(blocks)), block(PW * 32);
    if (dtype == 0) {
        if (variant == VAR_MMA) dasp_pipe_kernel<0, VAR_MMA><<<grid, block, smem, s>>>(p, items, n_items);
        else dasp_pipe_kernel<0, VAR_CUDACORE><<<grid, block, smem, s>>>(p, items, n_items);
    } else {
        if (variant == VAR_MMA) dasp_pipe_kernel<1, VAR_MMA><<<grid, block, smem, s>>>(p, items, n_items);
        else dasp_pipe_kernel<1, VAR_CUDACORE><<<grid, block, smem, s>>>(p, items, n_items);
    }
    return cudaGetLastError();
}

cudaError_t launch_long(const MainParams& p, int dtype, int variant, int64_t n_units, cudaStream_t s,
                        const void* apw_base, size_t apw_bytes, float apw_hit) {
    if (n_units <= 0) return cudaSuccess;
    const int64_t upw = dtype == 1 ? DASP_LONG_UPW_F16 : 1;
    const int64_t blocks = ((n_units + upw - 1) / upw * 32 + MAIN_THREADS - 1) / MAIN_THREADS;
    if (blocks > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    dim3 grid(static_cast<unsigned>(blocks)), block(MAIN_THREADS);
    const bool mma = variant == VAR_MMA;
    auto k = dtype == 0 ? (mma ? dasp_long_kernel<0, VAR_MMA> : dasp_long_kernel<0, VAR_CUDACORE>)
           : dtype == 1 ? (mma ? dasp_long_kernel<1, VAR_MMA> : dasp_long_kernel<1, VAR_CUDACORE>)
                        : (mma ? dasp_long_kernel<2, VAR_MMA> : dasp_long_kernel<2, VAR_CUDACORE>);
    if (apw_bytes || DASP_PDL) return launch_ex(k, grid.x, s, apw_base, apw_bytes, apw_hit, p, n_units);
    set_carveout(reinterpret_cast<const void*>(k));
    k<<<grid, block, 0, s>>>(p, n_units);
    return cudaGetLastError();
}

cudaError_t launch_short(const MainParams& p, int dtype, int variant, const uint64_t* tile_meta, int64_t n_tiles,
                         cudaStream_t s) {
    if (n_tiles <= 0) return cudaSuccess;
    const int64_t blocks = (n_tiles * 32 + MAIN_THREADS - 1) / MAIN_THREADS;
    if (blocks > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    dim3 grid(static_cast<unsigned>(blocks)), block(MAIN_THREADS);
    const bool mma = variant == VAR_MMA;
    auto k = dtype == 0 ? (mma ? dasp_short_kernel<0, VAR_MMA> : dasp_short_kernel<0, VAR_CUDACORE>)
           : dtype == 1 ? (mma ? dasp_short_kernel<1, VAR_MMA> : dasp_short_kernel<1, VAR_CUDACORE>)
                        : (mma ? dasp_short_kernel<2, VAR_MMA> : dasp_short_kernel<2, VAR_CUDACORE>);
    k<<<grid, block, 0, s>>>(p, tile_meta, n_tiles);
    return cudaGetLastError();
}

cudaError_t launch_finish(const FinishParams& p, int dtype, cudaStream_t s) {
    const int64_t warps = finish_warps(p.row_long, p.n0);
    if (warps == 0) return cudaSuccess;
    dim3 grid(static_cast<unsigned>((warps * 32 + 255) / 256)), block(256);
    if (dtype == 0) dasp_finish_kernel<0><<<grid, block, 0, s>>>(p);
    else if (dtype == 1) dasp_finish_kernel<1><<<grid, block, 0, s>>>(p);
    else dasp_finish_kernel<2><<<grid, block, 0, s>>>(p);
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

namespace {
// Host -> device copy by SM loads from page-locked host memory (UVA): 16-B loads, one grid stride.
// Many SMs keep more PCIe read requests outstanding than one copy engine does (C2 x vector: 49.5 vs
// 42 GB/s on the bench box, scripts/probe/h2d_probe.py).
__global__ void __launch_bounds__(256) dasp_h2d_sm_kernel(const int4* __restrict__ src, int4* __restrict__ dst,
                                                          int64_t n16, const uint8_t* __restrict__ src_tail,
                                                          uint8_t* __restrict__ dst_tail, int tail) {
    const int64_t stride = static_cast<int64_t>(gridDim.x) * blockDim.x;
    for (int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; i < n16; i += stride)
        dst[i] = src[i];
    if (blockIdx.x == 0 && static_cast<int>(threadIdx.x) < tail) dst_tail[threadIdx.x] = src_tail[threadIdx.x];
}
}  // namespace

cudaError_t launch_h2d_sm(void* dst, const void* host_src, size_t bytes, int sms, cudaStream_t s) {
    if (bytes == 0) return cudaSuccess;
    const int64_t n16 = static_cast<int64_t>(bytes / 16);
    const int tail = static_cast<int>(bytes % 16);
    const uint8_t* st = static_cast<const uint8_t*>(host_src) + n16 * 16;
    uint8_t* dt = static_cast<uint8_t*>(dst) + n16 * 16;
    dasp_h2d_sm_kernel<<<static_cast<unsigned>(sms > 0 ? sms : 148), 256, 0, s>>>(
        static_cast<const int4*>(host_src), static_cast<int4*>(dst), n16, st, dt, tail);
    return cudaGetLastError();
}

}  // namespace dasp
