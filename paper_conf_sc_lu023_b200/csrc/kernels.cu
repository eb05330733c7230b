// kernels.cu — sm_100a kernels of the DASP SpMV hot path (§3.3, Alg. 2-5).
//
// One fused launch covers the three row classes (warp-uniform dispatch on the global warp
// index), plus a small "finish" launch for long-row phase 2 (Alg. 2 l.17-25)
// and empty rows.  Every block inner product is computed by one of two variants that read
// the SAME packed arrays (north_star (3)):
//   VAR_MMA      legacy warp MMA: DMMA m8n8k4 f64 (Listing 1) / HMMA m16n8k16
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
__device__ __forceinline__ double gx(const double* x, uint32_t c) {
    return static_cast<int32_t>(c) >= 0 ? __ldg(x + static_cast<int32_t>(c)) : 0.0;
}
__device__ __forceinline__ uint16_t gxh(const uint16_t* x, uint32_t c) {
    return static_cast<int32_t>(c) >= 0 ? __ldg(reinterpret_cast<const unsigned short*>(x) + static_cast<int32_t>(c))
                                        : static_cast<uint16_t>(0);
}
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

// y[row] = alpha*acc + beta*y[row] (beta == 0: y not read, R16)
template <int DT>
__device__ __forceinline__ void store_y(const MainParams& P, int32_t row, typename Tr<DT>::A acc) {
    using Y = typename Tr<DT>::Y;
    if (row < 0) return;
    Y* y = static_cast<Y*>(P.y);
    Y r = static_cast<Y>(P.alpha) * acc;
    if (P.beta != 0.0) r += static_cast<Y>(P.beta) * y[row];
    y[row] = r;
}

// ------------------------------------------------------------------------------------------
// long rows, phase 1 (Alg. 2 l.1-16): one warp = one unit of UG consecutive groups
// ------------------------------------------------------------------------------------------
template <int VAR>
__device__ __forceinline__ void long_unit_f64(const MainParams& P, int64_t u, int lane, uint64_t pol) {
    const int64_t base = u * 256 + lane * 8;            // lane holds 8 consecutive elements
    const double* lv = static_cast<const double*>(P.long_val) + base;
    double v[8];
    uint32_t c[8];
    ld4_f64(lv, pol, *reinterpret_cast<double(*)[4]>(&v[0]));
    ld4_f64(lv + 4, pol, *reinterpret_cast<double(*)[4]>(&v[4]));
    ld8_b32(P.long_col + base, pol, c);
    const double* x = static_cast<const double*>(P.x);
    double xv[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) xv[j] = gx(x, c[j]);
    double part;
    if constexpr (VAR == VAR_MMA) {
        double c0 = 0.0, c1 = 0.0;
#pragma unroll
        for (int j = 0; j < 8; ++j) dmma(c0, c1, v[j], xv[j]);   // 8 m8n8k4 = 4 groups of 64
        double d = diag_to_quad(c0, c1, lane);                  // rows 2q, 2q+1 = group q
        part = (lane & 3) == 0 ? d : 0.0;
        part += __shfl_xor_sync(FULL, part, 4);
    } else {
        part = 0.0;
#pragma unroll
        for (int j = 0; j < 8; ++j) part = fma(v[j], xv[j], part);
        part += __shfl_xor_sync(FULL, part, 1);
        part += __shfl_xor_sync(FULL, part, 2);
        part += __shfl_xor_sync(FULL, part, 4);
    }
    if ((lane & 7) == 0) static_cast<double*>(P.partial)[u * 4 + (lane >> 3)] = part;
}

template <int VAR>
__device__ __forceinline__ void long_unit_f16(const MainParams& P, int64_t u, int lane, uint64_t pol) {
    const int64_t base = u * 512 + lane * 16;           // lane holds 16 consecutive elements
    uint32_t vv[8], c[16];
    ld8_b32(static_cast<const uint16_t*>(P.long_val) + base, pol, vv);
    ld8_b32(P.long_col + base, pol, *reinterpret_cast<uint32_t(*)[8]>(&c[0]));
    ld8_b32(P.long_col + base + 8, pol, *reinterpret_cast<uint32_t(*)[8]>(&c[8]));
    const uint16_t* x = static_cast<const uint16_t*>(P.x);
    uint16_t xh[16];
#pragma unroll
    for (int j = 0; j < 16; ++j) xh[j] = gxh(x, c[j]);
    float part;
    if constexpr (VAR == VAR_MMA) {
        float c0 = 0.f, c1 = 0.f;
#pragma unroll
        for (int h = 0; h < 8; ++h)   // elements 2h, 2h+1 -> A[g][2t..2t+1] of one m16n8k8
            hmma(c0, c1, vv[h], pack2(xh[2 * h], xh[2 * h + 1]));
        const float d = diag_to_quad(c0, c1, lane);             // rows 2q, 2q+1 = group q
        part = (lane & 3) == 0 ? d : 0.f;
        part += __shfl_xor_sync(FULL, part, 4);
    } else {
        part = 0.f;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const float2 af = u2f2(vv[j]);
            part = fmaf(af.x, h2f(xh[2 * j]), part);
            part = fmaf(af.y, h2f(xh[2 * j + 1]), part);
        }
        part += __shfl_xor_sync(FULL, part, 1);
        part += __shfl_xor_sync(FULL, part, 2);
        part += __shfl_xor_sync(FULL, part, 4);
    }
    if ((lane & 7) == 0) static_cast<float*>(P.partial)[u * 4 + (lane >> 3)] = part;
}

// ------------------------------------------------------------------------------------------
// medium rows (Alg. 3): row-block = 8 rows; regular 8 x K blocks in lane-interleaved chunks
// of CW blocks (R18), then the irregular tails with 4 lanes per row, then y.
// ------------------------------------------------------------------------------------------
template <int VAR>
__device__ __forceinline__ void medium_rb_f64(const MainParams& P, int64_t rb, int lane, uint64_t pol) {
    const int g = lane >> 2, t = lane & 3;
    const int64_t i = rb * 8 + g;
    // every load that does not depend on data goes out first: the row-block's pointers, the
    // irregular bounds and the output row (one memory round trip instead of three)
    const int64_t base = __ldg(P.rb_ptr + rb), end = __ldg(P.rb_ptr + rb + 1);
    const int64_t ib = __ldg(P.irr_ptr + i), ie = __ldg(P.irr_ptr + i + 1);
    const int32_t orow = __ldg(P.med_out + i);
    const int nreg = static_cast<int>((end - base) >> 5);
    const int nfull = nreg >> 2, rem = nreg & 3;
    const double* rv = static_cast<const double*>(P.reg_val) + base;
    const int32_t* rc = P.reg_col + base;
    const double* iv = static_cast<const double*>(P.irr_val);
    const double* x = static_cast<const double*>(P.x);
    // round 1: first chunk (4 blocks, 256-bit value load), the ragged last chunk and the
    // first irregular element of this lane, all in flight together
    double va[4] = {0.0, 0.0, 0.0, 0.0};
    uint32_t ca[4] = {0xffffffffu, 0xffffffffu, 0xffffffffu, 0xffffffffu};
    if (nfull > 0) { ld4_f64(rv + lane * 4, pol, va); ld4_b32(rc + lane * 4, pol, ca); }
    double vr[3] = {0.0, 0.0, 0.0};
    uint32_t cr[3] = {0xffffffffu, 0xffffffffu, 0xffffffffu};
    const int64_t rbase = static_cast<int64_t>(nfull) * 128 + lane * rem;
#pragma unroll
    for (int j = 0; j < 3; ++j)
        if (j < rem) { vr[j] = ld1_f64(rv + rbase + j, pol); cr[j] = ld1_b32(rc + rbase + j, pol); }
    int64_t k = ib + t;
    double vi = 0.0;
    uint32_t ci = 0xffffffffu;
    if (k < ie) { vi = ld1_f64(iv + k, pol); ci = ld1_b32(P.irr_col + k, pol); }
    double c0 = 0.0, c1 = 0.0, part = 0.0;
    for (int ch = 0; ch < nfull; ++ch) {
        if (ch > 0) { ld4_f64(rv + ch * 128 + lane * 4, pol, va); ld4_b32(rc + ch * 128 + lane * 4, pol, ca); }
        double xv[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) xv[j] = gx(x, ca[j]);
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            if constexpr (VAR == VAR_MMA) dmma(c0, c1, va[j], xv[j]);
            else part = fma(va[j], xv[j], part);
        }
    }
    double xr[3];
#pragma unroll
    for (int j = 0; j < 3; ++j) xr[j] = gx(x, cr[j]);     // pads / unused slots read 0
    const double xi = gx(x, ci);
#pragma unroll
    for (int j = 0; j < 3; ++j) {
        if (j < rem) {                                     // rem is warp-uniform
            if constexpr (VAR == VAR_MMA) dmma(c0, c1, vr[j], xr[j]);
            else part = fma(vr[j], xr[j], part);
        }
    }
    if constexpr (VAR == VAR_MMA) {                        // Alg. 3 l.13-17: diagonal -> quad g
        const double d = diag_to_quad(c0, c1, lane);
        part = t == 0 ? d : 0.0;
    }
    part = fma(vi, xi, part);                              // Alg. 3 l.20-24: irregular part
    for (k += 4; k < ie; k += 4) part = fma(ld1_f64(iv + k, pol), gx(x, ld1_b32(P.irr_col + k, pol)), part);
    part += __shfl_xor_sync(FULL, part, 1);
    part += __shfl_xor_sync(FULL, part, 2);
    if (t == 0) store_y<0>(P, orow, part);                 // Alg. 3 l.25 through the output map (R9)
}

template <int VAR>
__device__ __forceinline__ void medium_rb_f16(const MainParams& P, int64_t rb, int lane, uint64_t pol) {
    const int g = lane >> 2, t = lane & 3;
    const int64_t i = rb * 8 + g;
    const int64_t base = __ldg(P.rb_ptr + rb), end = __ldg(P.rb_ptr + rb + 1);
    const int64_t ib = __ldg(P.irr_ptr + i), ie = __ldg(P.irr_ptr + i + 1);
    const int32_t orow = __ldg(P.med_out + i);
    const int nreg = static_cast<int>((end - base) >> 6);
    const int nfull = nreg >> 2, rem = nreg & 3;
    const uint16_t* rv = static_cast<const uint16_t*>(P.reg_val) + base;
    const int32_t* rc = P.reg_col + base;
    const unsigned short* iv = static_cast<const unsigned short*>(P.irr_val);
    const uint16_t* x = static_cast<const uint16_t*>(P.x);
    float c0 = 0.f, c1 = 0.f, part = 0.f;
    // one 8x8 block: this lane's two slots 2t, 2t+1 of row g
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
    // round 1: first chunk (4 blocks: 16 B values, 32 B columns), the ragged last chunk and
    // the first irregular element
    uint32_t va[4] = {0u, 0u, 0u, 0u}, ca[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) ca[e] = 0xffffffffu;
    if (nfull > 0) { ld4_b32(rv + lane * 8, pol, va); ld8_b32(rc + lane * 8, pol, ca); }
    uint32_t vr[3] = {0u, 0u, 0u}, cr[6];
#pragma unroll
    for (int e = 0; e < 6; ++e) cr[e] = 0xffffffffu;
    const int64_t rbase = static_cast<int64_t>(nfull) * 256 + lane * 2 * rem;
#pragma unroll
    for (int j = 0; j < 3; ++j)
        if (j < rem) { vr[j] = ld1_b32(rv + rbase + 2 * j, pol); ld2_b32(rc + rbase + 2 * j, pol, cr[2 * j], cr[2 * j + 1]); }
    int64_t k = ib + t;
    uint16_t vi = 0;
    uint32_t ci = 0xffffffffu;
    if (k < ie) { vi = __ldg(iv + k); ci = ld1_b32(P.irr_col + k, pol); }
    for (int ch = 0; ch < nfull; ++ch) {
        if (ch > 0) { ld4_b32(rv + ch * 256 + lane * 8, pol, va); ld8_b32(rc + ch * 256 + lane * 8, pol, ca); }
#pragma unroll
        for (int j = 0; j < 4; ++j) block(va[j], ca[2 * j], ca[2 * j + 1]);
    }
#pragma unroll
    for (int j = 0; j < 3; ++j)
        if (j < rem) block(vr[j], cr[2 * j], cr[2 * j + 1]);   // rem is warp-uniform
    if constexpr (VAR == VAR_MMA) {
        const float d = diag_to_quad(c0, c1, lane);
        part = t == 0 ? d : 0.f;
    }
    part = fmaf(h2f(vi), h2f(gxh(x, ci)), part);
    for (k += 4; k < ie; k += 4)
        part = fmaf(h2f(__ldg(iv + k)), h2f(gxh(x, ld1_b32(P.irr_col + k, pol))), part);
    part += __shfl_xor_sync(FULL, part, 1);
    part += __shfl_xor_sync(FULL, part, 2);
    if (t == 0) store_y<1>(P, orow, part);
}

// ------------------------------------------------------------------------------------------
// short rows (Alg. 4) and singles (Alg. 5): one tile of 32 four-slot rows.
// Results are transposed with shuffles so that lane L writes outputs L and L+32 of the tile:
// the output map is read with two coalesced loads issued at the start of the tile.
// ------------------------------------------------------------------------------------------
// cat 0 = 1&3 (seg0 = slot 0, seg1 = slots 1-3), 1 = len-4, 2 = 2&2 (slots 0-1 | 2-3)
__device__ __forceinline__ int seg_of(int cat, int slot) { return cat == 0 ? (slot > 0) : (cat == 2 ? (slot >> 1) : 0); }

template <int VAR>
__device__ __forceinline__ void short_tile_f64(const MainParams& P, int cat, int64_t tile, int64_t obase, int lane,
                                               uint64_t pol) {
    const int g = lane >> 2, t = lane & 3;
    const int nseg = cat == 1 ? 1 : 2;
    double v[4];
    uint32_t c[4];
    ld4_f64(static_cast<const double*>(P.short_val) + tile * 128 + lane * 4, pol, v);
    ld4_b32(P.short_col + tile * 128 + lane * 4, pol, c);
    const int32_t o0 = __ldg(P.short_out + obase + lane);                        // outputs L, L+32
    const int32_t o1 = nseg == 2 ? __ldg(P.short_out + obase + 32 + lane) : -1;
    const double* x = static_cast<const double*>(P.x);
    double xv[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) xv[j] = gx(x, c[j]);
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
                dmma(cc0, cc1, v[j], myseg == s ? xv[j] : 0.0);
                val = __shfl_sync(FULL, (g & 1) ? cc1 : cc0, src + ((lane & 7) >> 1));
            } else {
                double p = myseg == s ? v[j] * xv[j] : 0.0;
                p += __shfl_xor_sync(FULL, p, 1);
                p += __shfl_xor_sync(FULL, p, 2);
                val = __shfl_sync(FULL, p, src);
            }
            const int blk = nseg == 2 ? 2 * j + s : j;   // this result fills outputs 8*blk .. 8*blk+7
            if ((lane >> 3) == blk) r0 = val;
            if ((lane >> 3) == blk - 4) r1 = val;
        }
    }
    store_y<0>(P, o0, r0);
    if (nseg == 2) store_y<0>(P, o1, r1);
}

template <int VAR>
__device__ __forceinline__ void short_tile_f16(const MainParams& P, int cat, int64_t tile, int64_t obase, int lane,
                                               uint64_t pol) {
    const int g = lane >> 2, t = lane & 3;
    const int nseg = cat == 1 ? 1 : 2;
    uint32_t a0, a2, c[4];
    ld2_b32(static_cast<const uint16_t*>(P.short_val) + tile * 128 + lane * 4, pol, a0, a2);
    ld4_b32(P.short_col + tile * 128 + lane * 4, pol, c);
    const int32_t o0 = __ldg(P.short_out + obase + lane);
    const int32_t o1 = nseg == 2 ? __ldg(P.short_out + obase + 32 + lane) : -1;
    const uint16_t* x = static_cast<const uint16_t*>(P.x);
    uint16_t xh[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) xh[e] = gxh(x, c[e]);
    // element e: four-slot row group q = (e<2 ? 0 : 2) + (t>>1), slot 2(t&1) + (e&1); elements
    // 0,1 are this lane's slots of m16n8k8 block 0 (rows 0-15), elements 2,3 of block 1 (16-31)
    const int seg0 = seg_of(cat, 2 * (t & 1)), seg1 = seg_of(cat, 2 * (t & 1) + 1);
    const int gs = lane & 7;                              // row g' whose result this lane collects
    float r0 = 0.f, r1 = 0.f;
    float slo[2], shi[2];
    if constexpr (VAR == VAR_CUDACORE) {
        const float2 vl = u2f2(a0), vh = u2f2(a2);
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
                hmma(cc0, cc1, (q >> 1) ? a2 : a0, b0);
                val = __shfl_sync(FULL, (g & 1) ? cc1 : cc0, 4 * gs + (gs >> 1));
            } else {
                val = __shfl_sync(FULL, q < 2 ? slo[s] : shi[s], 4 * gs + 2 * (q & 1));
            }
            const int blk = nseg == 2 ? 2 * q + s : q;
            if ((lane >> 3) == blk) r0 = val;
            if ((lane >> 3) == blk - 4) r1 = val;
        }
    }
    store_y<1>(P, o0, r0);
    if (nseg == 2) store_y<1>(P, o1, r1);
}

// singles (Alg. 5): lane handles 4 consecutive len-1 rows on CUDA cores
template <int DT>
__device__ __forceinline__ void singles_tile(const MainParams& P, int64_t tile, int64_t obase, int lane, uint64_t pol) {
    uint32_t c[4], o[4];
    ld4_b32(P.short_col + tile * 128 + lane * 4, pol, c);
    ld4_b32(P.short_out + obase + lane * 4, pol, o);
    if constexpr (DT == 0) {
        double v[4];
        ld4_f64(static_cast<const double*>(P.short_val) + tile * 128 + lane * 4, pol, v);
#pragma unroll
        for (int j = 0; j < 4; ++j) store_y<0>(P, static_cast<int32_t>(o[j]), v[j] * gx(static_cast<const double*>(P.x), c[j]));
    } else {
        uint32_t a0, a2;
        ld2_b32(static_cast<const uint16_t*>(P.short_val) + tile * 128 + lane * 4, pol, a0, a2);
        float2 lo = u2f2(a0);
        float2 hi = u2f2(a2);
        const float v[4] = {lo.x, lo.y, hi.x, hi.y};
        const uint16_t* x = static_cast<const uint16_t*>(P.x);
#pragma unroll
        for (int j = 0; j < 4; ++j) store_y<1>(P, static_cast<int32_t>(o[j]), v[j] * h2f(gxh(x, c[j])));
    }
}

// ------------------------------------------------------------------------------------------
// the fused main kernel
// ------------------------------------------------------------------------------------------
#ifndef DASP_MIN_BLOCKS
#define DASP_MIN_BLOCKS 4   // caps registers at 64: >= 32 resident warps per SM, no spills
#endif
template <int DT, int VAR>
__global__ void __launch_bounds__(MAIN_THREADS, DASP_MIN_BLOCKS) dasp_main_kernel(const MainParams P) {
    const int lane = threadIdx.x & 31;
    // role of this warp inside its panel; the descriptor fields are loaded only on the branch
    // that needs them so they do not stay live (register pressure = occupancy)
    const PanelDesc* D = P.panels + __ldg(P.blk_panel + blockIdx.x);
    int64_t w = (static_cast<int64_t>(blockIdx.x) - __ldg(&D->blk0)) * WARPS_PER_BLOCK + (threadIdx.x >> 5);
    const uint64_t pol = stream_policy();
    const int64_t nunits = __ldg(&D->nunits);
    if (w < nunits) {                                    // long rows, phase 1
        if (!(P.class_mask & 1)) return;
        const int64_t u = __ldg(P.unit_order + __ldg(&D->unit0) + w);
        if constexpr (DT == 0) long_unit_f64<VAR>(P, u, lane, pol);
        else long_unit_f16<VAR>(P, u, lane, pol);
        return;
    }
    w -= nunits;
    const int64_t nmw = __ldg(&D->nmw);
    if (w < nmw) {                                       // medium rows
        if (!(P.class_mask & 2)) return;
        const int64_t rbp0 = __ldg(&D->rb0);
        const int64_t rb0 = rbp0 + w * P.rbw;
        const int64_t rb1 = min(rb0 + P.rbw, rbp0 + __ldg(&D->nrb));
        for (int64_t rb = rb0; rb < rb1; ++rb) {
            if constexpr (DT == 0) medium_rb_f64<VAR>(P, rb, lane, pol);
            else medium_rb_f16<VAR>(P, rb, lane, pol);
        }
        return;
    }
    const int64_t t = w - nmw;                           // short tiles: [1&3][len4][2&2][singles]
    const int64_t t13 = __ldg(&D->t13), t4 = __ldg(&D->t4), t22 = __ldg(&D->t22);
    if (t >= t13 + t4 + t22 + __ldg(&D->ts) || !(P.class_mask & 4)) return;
    const int64_t tile = __ldg(&D->tile0) + t;
    const int64_t out0 = __ldg(&D->out0);
    int cat;
    int64_t obase;
    if (t < t13) { cat = 0; obase = out0 + t * 64; }
    else if (t < t13 + t4) { cat = 1; obase = out0 + 64 * t13 + (t - t13) * 32; }
    else if (t < t13 + t4 + t22) { cat = 2; obase = out0 + 64 * t13 + 32 * t4 + (t - t13 - t4) * 64; }
    else {
        obase = out0 + 64 * t13 + 32 * t4 + 64 * t22 + (t - t13 - t4 - t22) * 128;
        singles_tile<DT>(P, tile, obase, lane, pol);
        return;
    }
    if constexpr (DT == 0) short_tile_f64<VAR>(P, cat, tile, obase, lane, pol);
    else short_tile_f16<VAR>(P, cat, tile, obase, lane, pol);
}

// long phase 2 (Alg. 2 l.17-25): one warp per long row, lane-strided sum of the group partials
// in a fixed order, butterfly reduction (deterministic, R19); then the empty rows (R1).
template <int DT>
__global__ void __launch_bounds__(256) dasp_finish_kernel(const FinishParams P) {
    using A = typename Tr<DT>::A;
    using Y = typename Tr<DT>::Y;
    const int lane = threadIdx.x & 31;
    const int64_t w = (static_cast<int64_t>(blockIdx.x) * 256 + threadIdx.x) / 32;
    Y* y = static_cast<Y*>(P.y);
    if (w < P.row_long) {
        const A* part = static_cast<const A*>(P.partial);
        A s = 0;
        for (int64_t k = P.group_ptr[w] + lane; k < P.group_ptr[w + 1]; k += 32) s += part[k];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(FULL, s, o);
        if (lane == 0) {
            const int32_t row = P.long_out[w];
            Y r = static_cast<Y>(P.alpha) * s;
            if (P.beta != 0.0) r += static_cast<Y>(P.beta) * y[row];
            y[row] = r;
        }
        return;
    }
    const int64_t e = (w - P.row_long) * 32 + lane;
    if (e < P.n0) {
        const int32_t row = P.empty_rows[e];
        y[row] = P.beta != 0.0 ? static_cast<Y>(P.beta) * y[row] : Y(0);
    }
}

template <int DT>
__global__ void dasp_scale_kernel(void* yv, int64_t m, double beta) {
    using Y = typename Tr<DT>::Y;
    Y* y = static_cast<Y*>(yv);
    for (int64_t i = static_cast<int64_t>(blockIdx.x) * blockDim.x + threadIdx.x; i < m;
         i += static_cast<int64_t>(gridDim.x) * blockDim.x)
        y[i] = beta != 0.0 ? static_cast<Y>(beta) * y[i] : Y(0);
}

}  // namespace

template <typename Kern>
static cudaError_t launch_ex(Kern kernel, unsigned blocks, cudaStream_t s, const void* apw_base, size_t apw_bytes,
                             float apw_hit, const MainParams& p) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(blocks);
    cfg.blockDim = dim3(MAIN_THREADS);
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    if (apw_bytes) {
        attr[0].id = cudaLaunchAttributeAccessPolicyWindow;
        attr[0].val.accessPolicyWindow.base_ptr = const_cast<void*>(apw_base);
        attr[0].val.accessPolicyWindow.num_bytes = apw_bytes;
        attr[0].val.accessPolicyWindow.hitRatio = apw_hit;
        attr[0].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        attr[0].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
    }
    return cudaLaunchKernelEx(&cfg, kernel, p);
}

cudaError_t launch_main(const MainParams& p, int dtype, int variant, int64_t blocks, cudaStream_t s,
                        const void* apw_base, size_t apw_bytes, float apw_hit) {
    if (blocks <= 0) return cudaSuccess;
    if (blocks > 0x7fffffffLL) return cudaErrorInvalidConfiguration;
    const unsigned nb = static_cast<unsigned>(blocks);
    cudaError_t e;
    if (dtype == 0) {
        if (variant == VAR_MMA) e = launch_ex(dasp_main_kernel<0, VAR_MMA>, nb, s, apw_base, apw_bytes, apw_hit, p);
        else e = launch_ex(dasp_main_kernel<0, VAR_CUDACORE>, nb, s, apw_base, apw_bytes, apw_hit, p);
    } else {
        if (variant == VAR_MMA) e = launch_ex(dasp_main_kernel<1, VAR_MMA>, nb, s, apw_base, apw_bytes, apw_hit, p);
        else e = launch_ex(dasp_main_kernel<1, VAR_CUDACORE>, nb, s, apw_base, apw_bytes, apw_hit, p);
    }
    if (e != cudaSuccess) return e;
    return cudaGetLastError();
}

cudaError_t launch_finish(const FinishParams& p, int dtype, cudaStream_t s) {
    const int64_t warps = p.row_long + (p.n0 + 31) / 32;
    if (warps == 0) return cudaSuccess;
    dim3 grid(static_cast<unsigned>((warps * 32 + 255) / 256)), block(256);
    if (dtype == 0) dasp_finish_kernel<0><<<grid, block, 0, s>>>(p);
    else dasp_finish_kernel<1><<<grid, block, 0, s>>>(p);
    return cudaGetLastError();
}

cudaError_t launch_scale(void* y, int64_t m, double beta, int dtype, cudaStream_t s) {
    if (m == 0) return cudaSuccess;
    int64_t blocks = (m + 255) / 256;
    if (blocks > 148 * 16) blocks = 148 * 16;
    if (dtype == 0) dasp_scale_kernel<0><<<static_cast<unsigned>(blocks), 256, 0, s>>>(y, m, beta);
    else dasp_scale_kernel<1><<<static_cast<unsigned>(blocks), 256, 0, s>>>(y, m, beta);
    return cudaGetLastError();
}

}  // namespace dasp
