// hhc_device.cuh -- device helpers shared by the HHC kernels (hhc_kernels.cu,
// wave_kernels.cu, microbench.cu): stencil tables, canonical point updates (reading R4),
// hexagon geometry (readings G1-G3), cp.async, the per-block geometry table.
#pragma once
#include <cuda_runtime.h>

#include <utility>

#include "hhc_internal.h"

namespace hhc {

// ----------------------------------------------------------------- stencil tables
struct Off { int d1, d2, d3; };

__host__ __device__ constexpr int kind_ndims(int kind) { return (kind == 4 || kind == 5) ? 3 : 2; }
__host__ __device__ constexpr bool kind_in_nb(int kind, int nz) {
    return (kind == STENCIL_HEAT2D_9PT || kind == STENCIL_LAPLACIAN3D_27PT) ? true : nz <= 1;
}
// j-th offset of N_kind in lexicographic order over {-1,0,1}^D (reading R4)
__host__ __device__ constexpr Off kind_off(int kind, int j) {
    const int D = kind_ndims(kind);
    int n = 0;
    for (int d1 = -1; d1 <= 1; ++d1)
        for (int d2 = -1; d2 <= 1; ++d2)
            for (int d3 = (D == 3 ? -1 : 0); d3 <= (D == 3 ? 1 : 0); ++d3) {
                const int nz = (d1 != 0) + (d2 != 0) + (d3 != 0);
                if (!kind_in_nb(kind, nz)) continue;
                if (n == j) return Off{d1, d2, d3};
                ++n;
            }
    return Off{0, 0, 0};
}
__host__ __device__ constexpr int kind_npts(int kind) {
    const int D = kind_ndims(kind);
    int n = 0;
    for (int d1 = -1; d1 <= 1; ++d1)
        for (int d2 = -1; d2 <= 1; ++d2)
            for (int d3 = (D == 3 ? -1 : 0); d3 <= (D == 3 ? 1 : 0); ++d3)
                if (kind_in_nb(kind, (d1 != 0) + (d2 != 0) + (d3 != 0))) ++n;
    return n;
}

// ----------------------------------------------------------------- point updates
// Default weights (reading R1) as compile-time constants: with coeffs == NULL
// the weights become FFMA immediates (no register/constant-bank operand).
__host__ __device__ constexpr float kind_default_w(int kind, int nz) {
    return kind == STENCIL_JACOBI2D_5PT ? 0.2f
         : kind == STENCIL_LAPLACIAN2D_5PT ? (nz == 0 ? 0.5f : 0.125f)
         : kind == STENCIL_HEAT2D_9PT ? (nz == 0 ? 0.25f : nz == 1 ? 0.125f : 0.0625f)
         : kind == STENCIL_HEAT3D_7PT ? (nz == 0 ? 0.25f : 0.125f)
         : kind == STENCIL_LAPLACIAN3D_27PT
               ? (nz == 0 ? 0.5f : nz == 1 ? 7.0f / 128.0f : nz == 2 ? 3.0f / 256.0f : 1.0f / 256.0f)
               : 0.0f;
}
template <int KIND, bool DEFW, int J>
__device__ __forceinline__ float wgt(const HexParams& p) {
    if constexpr (DEFW) {
        constexpr Off o = kind_off(KIND, J);
        constexpr float w = kind_default_w(KIND, (o.d1 != 0) + (o.d2 != 0) + (o.d3 != 0));
        return w;
    } else {
        return p.w[J];
    }
}

// 2D rows r0, r1, r2 = x-1, x, x+1, slots s-2 .. s+3 of the previous level.
// Output column k (u = u0+k) reads offset (d1, d2) at row 1+d1, slot k+1+d2.
template <int KIND, int MODE, bool DEFW, int J, int N>
__device__ __forceinline__ float lin_term2(float acc, const float (&r0)[N], const float (&r1)[N],
                                           const float (&r2)[N], int k, const HexParams& p) {
    constexpr Off o = kind_off(KIND, J);
    const float v = o.d1 < 0 ? r0[k + 1 + o.d2] : o.d1 == 0 ? r1[k + 1 + o.d2] : r2[k + 1 + o.d2];
    const float w = wgt<KIND, DEFW, J>(p);
    if constexpr (J == 0) return __fmul_rn(w, v);
    else if constexpr (MODE == STENCIL_MODE_FUSED) return __fmaf_rn(w, v, acc);
    else return __fadd_rn(acc, __fmul_rn(w, v));
}
template <int KIND, int MODE, bool HASC, bool DEFW, int N, int... J>
__device__ __forceinline__ float lin2(const float (&r0)[N], const float (&r1)[N], const float (&r2)[N], int k,
                                      const HexParams& p, std::integer_sequence<int, J...>) {
    float acc = 0.0f;
    ((acc = lin_term2<KIND, MODE, DEFW, J, N>(acc, r0, r1, r2, k, p)), ...);
    if constexpr (HASC) acc = __fadd_rn(acc, p.c);
    return acc;
}

// Gradient-2D (reading R1): gx = .5(e-w), gy = .5(s-n), g2 = (1+gx^2)+gy^2,
// lap = ((n-c)+(s-c))+((e-c)+(w-c)), out = c + (kappa*lap)/sqrt(g2).
template <int MODE, bool DEFW, int N>
__device__ __forceinline__ float grad2(const float (&r0)[N], const float (&r1)[N], const float (&r2)[N], int k,
                                       const HexParams& p) {
    const float n = r0[k + 1], s = r2[k + 1];
    const float w = r1[k], e = r1[k + 2], c = r1[k + 1];
    const float gx = __fmul_rn(0.5f, __fsub_rn(e, w));
    const float gy = __fmul_rn(0.5f, __fsub_rn(s, n));
    float g2;
    if constexpr (MODE == STENCIL_MODE_FUSED) g2 = __fmaf_rn(gy, gy, __fmaf_rn(gx, gx, 1.0f));
    else g2 = __fadd_rn(__fadd_rn(1.0f, __fmul_rn(gx, gx)), __fmul_rn(gy, gy));
    const float lap = __fadd_rn(__fadd_rn(__fsub_rn(n, c), __fsub_rn(s, c)),
                                __fadd_rn(__fsub_rn(e, c), __fsub_rn(w, c)));
    const float kappa = DEFW ? 0.125f : p.kappa;
    const float q = __fdiv_rn(__fmul_rn(kappa, lap), __fsqrt_rn(g2));
    return __fadd_rn(c, q);
}

// Packed pair form of lin2 (K1 pair layout): every row register holds the two
// columns (q, q + D) of one pair, so each stencil term of both points is one
// f32x2 operation on an aligned register pair (FFMA2/FMUL2 on sm_100a).  Each
// half is the same correctly rounded operation sequence as lin2 (reading R4),
// hence bit-identical.  Only for MODE_FUSED: ptxas contracts a packed
// mul.rn + add.rn pair into FFMA2 (observed with CUDA 12.9), so the plain mode
// keeps scalar __fmul_rn/__fadd_rn.
template <int KIND, bool DEFW, int J>
__device__ __forceinline__ float2 lin_term2x2(float2 acc, const float2 (&r0)[6], const float2 (&r1)[6],
                                              const float2 (&r2)[6], int k, const HexParams& p) {
    constexpr Off o = kind_off(KIND, J);
    const float2 v = o.d1 < 0 ? r0[k + 1 + o.d2] : o.d1 == 0 ? r1[k + 1 + o.d2] : r2[k + 1 + o.d2];
    const float w = wgt<KIND, DEFW, J>(p);
    if constexpr (J == 0) return __fmul2_rn(make_float2(w, w), v);
    else return __ffma2_rn(make_float2(w, w), v, acc);
}
template <int KIND, bool HASC, bool DEFW, int... J>
__device__ __forceinline__ float2 lin2x2(const float2 (&r0)[6], const float2 (&r1)[6], const float2 (&r2)[6], int k,
                                         const HexParams& p, std::integer_sequence<int, J...>) {
    float2 acc = make_float2(0.0f, 0.0f);
    ((acc = lin_term2x2<KIND, DEFW, J>(acc, r0, r1, r2, k, p)), ...);
    if constexpr (HASC) acc = __fadd2_rn(acc, make_float2(p.c, p.c));
    return acc;
}

template <int KIND, int MODE, bool HASC, bool DEFW, int N>
__device__ __forceinline__ float point2(const float (&r0)[N], const float (&r1)[N], const float (&r2)[N], int k,
                                        const HexParams& p) {
    if constexpr (KIND == STENCIL_GRADIENT2D) return grad2<MODE, DEFW, N>(r0, r1, r2, k, p);
    else return lin2<KIND, MODE, HASC, DEFW, N>(r0, r1, r2, k, p, std::make_integer_sequence<int, kind_npts(KIND)>{});
}

// 3D rows r0, r1, r2 = x-1, x, x+1; each [l][c]: l = u2-2, u2-1, u2 ; c = slots s-2 .. s+3.
template <int KIND, int MODE, bool DEFW, int J>
__device__ __forceinline__ float lin_term3(float acc, const float (&r0)[3][6], const float (&r1)[3][6],
                                           const float (&r2)[3][6], int k, const HexParams& p) {
    constexpr Off o = kind_off(KIND, J);
    const float v = o.d1 < 0 ? r0[1 + o.d2][k + 1 + o.d3]
                  : o.d1 == 0 ? r1[1 + o.d2][k + 1 + o.d3] : r2[1 + o.d2][k + 1 + o.d3];
    const float w = wgt<KIND, DEFW, J>(p);
    if constexpr (J == 0) return __fmul_rn(w, v);
    else if constexpr (MODE == STENCIL_MODE_FUSED) return __fmaf_rn(w, v, acc);
    else return __fadd_rn(acc, __fmul_rn(w, v));
}
template <int KIND, int MODE, bool HASC, bool DEFW, int... J>
__device__ __forceinline__ float lin3(const float (&r0)[3][6], const float (&r1)[3][6], const float (&r2)[3][6],
                                      int k, const HexParams& p, std::integer_sequence<int, J...>) {
    float acc = 0.0f;
    ((acc = lin_term3<KIND, MODE, DEFW, J>(acc, r0, r1, r2, k, p)), ...);
    if constexpr (HASC) acc = __fadd_rn(acc, p.c);
    return acc;
}

// ----------------------------------------------------------------- helpers
__device__ __forceinline__ void ld6(const float* base, float (&r)[6]) {
    const float2 h = *reinterpret_cast<const float2*>(base - 2);
    const float4 m = *reinterpret_cast<const float4*>(base);
    r[0] = h.x; r[1] = h.y; r[2] = m.x; r[3] = m.y; r[4] = m.z; r[5] = m.w;
}

// Clipped row [l, r) of local level lev (reading G1; radius R: slopes and the
// fixed ring scale by R); empty (l == r) outside [0, nlev).
__device__ __forceinline__ void hex_row(const HexParams& p, int64_t x0, int nlev, int lev,
                                        int64_t& l, int64_t& r) {
    if (lev < 0 || lev >= nlev) { l = r = 0; return; }
    const int tau = p.tau_lo + lev;
    const int mm = p.R * min(tau, p.tT - tau);
    l = max(x0 - mm, (int64_t)p.R);
    r = min(x0 + p.tS1 + mm, p.S1 - p.R);
    if (r < l) r = l;
}

// Footprint of local level lev (values of level lev-1 the block does not hold):
// F = (row(lev) +- R) \ row(lev-1), as two intervals, plus the interval of
// row(lev-1) positions inside row(lev)+-R ("inner").  first = no usable row(lev-1).
struct Foot { int64_t A0, A1, f1a, f1b, f2a, f2b, ia, ib; bool first, empty; };

__device__ __forceinline__ Foot footprint(const HexParams& p, int64_t x0, int nlev, int lev) {
    Foot f;
    int64_t rl, rr, pl, pr;
    hex_row(p, x0, nlev, lev, rl, rr);
    hex_row(p, x0, nlev, lev - 1, pl, pr);
    f.empty = rl >= rr;
    f.A0 = rl - p.R; f.A1 = rr + p.R;
    f.first = (lev == 0) || (pl >= pr);
    if (f.first) {
        f.f1a = f.A0; f.f1b = f.A1; f.f2a = f.f2b = f.A1; f.ia = f.ib = f.A1;
    } else {
        f.f1a = f.A0; f.f1b = max(f.A0, min(f.A1, pl));
        f.f2a = min(f.A1, max(pr, f.A0)); f.f2b = f.A1;
        if (f.f2a < f.f1b) f.f2a = f.f1b;
        f.ia = max(f.A0, pl); f.ib = min(f.A1, pr);
        if (f.ib < f.ia) f.ib = f.ia;
    }
    return f;
}

// Asynchronous 4-byte global -> shared copy (LDGSTS); the footprint rows are
// issued back to back and waited for once per sub-tile.
__device__ __forceinline__ void cp_async4(float* dst, const float* src) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(dst);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(s), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;\n" ::: "memory"); }

// Four consecutive floats src[0..3] -> dst[0..3] (dst 16-B aligned) with the
// widest cp.async the source alignment allows (16, 8 or 4 bytes per copy); the
// skew makes the source alignment level-dependent (3D footprint lines).
__device__ __forceinline__ void cp_async_f4(float* dst, const float* src) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(dst);
    const unsigned a = (unsigned)(uintptr_t)src & 15u;
    if (a == 0) {
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(src) : "memory");
    } else if ((a & 7u) == 0) {
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(s), "l"(src) : "memory");
        asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(s + 8), "l"(src + 2) : "memory");
    } else {
#pragma unroll
        for (int j = 0; j < 4; ++j)
            asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(s + 4 * j), "l"(src + j) : "memory");
    }
}

// Non-facet interval [lo, hi) of smem rows at one level (reading G3): rows whose
// every reader at the next level, x' in [x-R, x+R] within the interior
// [R, S1-1-R], lies inside this block's next row [nl, nr).  Empty -> write all.
__device__ __forceinline__ void facet_gap(int64_t nl, int64_t nr, int64_t S1, bool final_level, int64_t xs,
                                          int NX, int R, int& lo, int& hi) {
    lo = hi = 0;
    if (final_level || nl >= nr) return;
    const int64_t xl = nl <= R ? (int64_t)-4 + xs : nl + R;         // max(x-R,R) >= nl
    const int64_t xh = nr >= S1 - R ? xs + NX + 4 : nr - R;        // min(x+R,S1-1-R) < nr
    if (xl >= xh) return;
    lo = (int)max(xl - xs, (int64_t)-2);
    hi = (int)min(xh - xs, (int64_t)NX + 2);
}

// Per-level geometry of the block's hexagon, in smem rows pp = x - xs, computed
// once per block (identical for every sub-tile); kGeo ints per level:
//  0..5 footprint intervals f1, f2, inner; 6 first; 7 empty;
//  8, 9 the row [rl, rr); 10, 11 the non-facet gap [lo, hi); 12 rows per x-group.
constexpr int kGeo = 16;
__device__ __forceinline__ void build_geo(const HexParams& p, int64_t x0, int64_t xs, int nlev, int* geo) {
    const int NX = p.tS1 + p.R * p.tT + 2 * p.R;
    const int64_t tb = p.t0 + p.tau_lo;
    for (int lev = threadIdx.x; lev < nlev; lev += blockDim.x) {
        const Foot f = footprint(p, x0, nlev, lev);
        int* g = geo + lev * kGeo;
        g[0] = (int)(f.f1a - xs); g[1] = (int)(f.f1b - xs);
        g[2] = (int)(f.f2a - xs); g[3] = (int)(f.f2b - xs);
        g[4] = (int)(f.ia - xs);  g[5] = (int)(f.ib - xs);
        g[6] = f.first ? 1 : 0;   g[7] = f.empty ? 1 : 0;
        int64_t rl, rr, nl, nr;
        hex_row(p, x0, nlev, lev, rl, rr);
        hex_row(p, x0, nlev, lev + 1, nl, nr);
        g[8] = (int)(rl - xs); g[9] = (int)(rr - xs);
        int lo, hi;
        facet_gap(nl, nr, p.S1, tb + lev == p.T, xs, NX, p.R, lo, hi);
        g[10] = lo; g[11] = hi;
        g[12] = (int)((rr - rl + p.G - 1) / p.G);
    }
}

// Flat list of the footprint rows of all levels (F(lev), full rows), built once
// per block by one thread: entry = pp | lev << 13.  Returns the count.
__device__ __forceinline__ int build_foot_list(const int* geo, int nlev, int* list) {
    int n = 0;
    for (int lev = 0; lev < nlev; ++lev) {
        const int* g = geo + lev * kGeo;
        if (g[7]) continue;
        for (int pp = g[0]; pp < g[1]; ++pp) list[n++] = pp | (lev << 13);
        for (int pp = g[2]; pp < g[3]; ++pp) list[n++] = pp | (lev << 13);
    }
    return n;
}

}  // namespace hhc
