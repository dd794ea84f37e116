// hhc_kernels_pair.cu -- K1P: 2D HHC kernel with two levels per shared-memory pass
// (DESIGN.md §Kernels).
//
// Same tiling, schedule and global I/O as K1 (§3.1, Fig. 2; readings
// G1-G3).  The rows of a hexagon are computed two levels at a time: a pass
// reads level l-1 from a shared-memory plane, computes level l into a rolling
// 3-row register window and, one row behind, level l+1 from those registers,
// and writes only level l+1 back (temporal blocking in registers: half the
// shared-memory traffic, half the barriers and per-level setup of K1).
//
// The S2 neighbours of level l come from the left lane by warp shuffle.  To
// need no synchronisation between warps inside a pass, each warp computes 4
// columns of overlap: lane 0 recomputes the last 4 columns of the warp to its
// left (or of the previous sub-tile) at level l and only serves as the shuffle
// source of lane 1; it never stores.  A warp therefore owns 124 new columns and
// tS2 = 124 * (warps per x-group).  The rows of a level are split over G
// x-groups; a group computes the two level-l rows just outside its level-(l+1)
// segment redundantly (no exchange between groups inside a pass).  Levels that
// cannot be paired (odd tails, a second level that is the first of the hexagon)
// are done by single-level passes with the same layout.
#include "hhc_device.cuh"

namespace hhc {

constexpr int kCW = 124;                                   // new columns per warp
constexpr unsigned kFullMask = 0xffffffffu;

// Per-block schedule of passes: sched[l] = type | pass << 4, type 1 = single,
// 2 = first level of a pair, 0 = second level of a pair.  Pass k reads plane
// (k+1)&1 and writes plane k&1.
__device__ __forceinline__ void build_sched(const int* geo, int nlev, int* sched) {
    int k = 0;
    for (int l = 0; l < nlev; ++k) {
        const int* g = geo + l * kGeo;
        const int* gn = geo + (l + 1) * kGeo;
        if (l + 1 < nlev && !g[7] && !gn[7] && !gn[6]) {
            sched[l] = 2 | (k << 4);
            sched[l + 1] = 0 | (k << 4);
            l += 2;
        } else {
            sched[l] = 1 | (k << 4);
            l += 1;
        }
    }
}

template <int KIND, int MODE, bool HASC, bool DEFW>
__global__ void __launch_bounds__(512) hex2d_pair_kernel(const __grid_constant__ HexParams p) {
    extern __shared__ __align__(16) float sm[];
    const int tT = p.tT, tS1 = p.tS1, tS2 = p.tS2;
    const int NX = tS1 + tT + 2;
    const int RS = tS2 + 8;                            // slots: 2 pad, 6 halo, tS2 window
    const int nthr = blockDim.x, tid = threadIdx.x;
    const int lane = tid & 31, warp = tid >> 5;
    const int nw = tS2 / kCW;                          // warps per x-group
    const int wg = warp % nw, grp = warp / nw;         // warp within the group, group
    const int gtid = tid % (32 * nw);                  // thread index within the group
    const int G = p.G;
    const int64_t S1 = p.S1, S2 = p.S2;
    const int S2i = (int)S2;
    const int64_t x0 = p.xbase + (int64_t)blockIdx.x * p.P;
    const int64_t xs = x0 - tT / 2 - 1;
    const int nlev = p.tau_hi - p.tau_lo;
    const int64_t tb = p.t0 + p.tau_lo;
    // two planes of NX rows, each with one guard row before and after (the rolling
    // window of a pass may touch row -1 or NX; those values are never used)
    float* const pl0 = sm + RS;
    float* const pl1 = sm + (NX + 2) * RS + RS;
    float* const face = sm + 2 * (NX + 2) * RS;        // [2][tT + 1][NX][6]
    const int FS = (tT + 1) * NX * 6;
    float* const stage = face + 2 * FS;                // [2][4][tS2 + 4]
    const int SR = tS2 + 4;
    int* const geo = reinterpret_cast<int*>(stage + 2 * 4 * SR);   // [tT][kGeo]
    int* const sched = geo + kGeo * tT;                            // [tT]
    build_geo(p, x0, xs, nlev, geo);
    __syncthreads();
    if (tid == 0) build_sched(geo, nlev, sched);
    __syncthreads();

    const int colbase = kCW * wg + 4 * lane;           // u0 - (a - 4)
    const int s = colbase + 4;                         // smem slot of column k = 0
    const bool store_lane = lane != 0;                 // lane 0 is the overlap lane

    for (int j2 = 0; j2 < p.n2; ++j2) {
        const int64_t a = 1 + (int64_t)j2 * tS2;
        const int64_t u0 = a - 4 + colbase;
        float* const fcur = face + (j2 & 1) * FS;      // [l][pp][6]: level l-1, last 6 columns
        float* const fnxt = face + ((j2 + 1) & 1) * FS;

        // ---- footprint of every pass-start level (values of level l-1 made elsewhere),
        //      and the stage of the first pair's second level
        if (!p.compute_only) {
            const int W = tS2 + 6;                     // columns u' in [a-6, a+tS2)
            for (int l = 0; l < nlev; ++l) {
                const int* g = geo + l * kGeo;
                const int type = sched[l] & 15, k = sched[l] >> 4;
                if (g[7] || type == 0) continue;
                const bool halo_all = g[6] || j2 == 0;
                const float* src = p.plane[(tb + l - 1) & 1];
                float* const dpl = ((k + 1) & 1) ? pl1 : pl0;
                const int64_t ybase = a - 5 - l;      // y of footprint column c: u' - (l-1), u' = a-6+c
                for (int seg = 0; seg < 3; ++seg) {
                    const int pa = g[2 * seg], pb = g[2 * seg + 1];
                    const bool full = seg < 2;
                    if (!full && !halo_all) break;
                    for (int pp = pa + grp; pp < pb; pp += G) {
                        const int64_t x = xs + pp;
                        if (l > 0 && (x == 0 || x == S1 - 1)) continue;   // ring rows: per-pass fill
                        const float* row = src + x * S2;
                        // halo columns (c < 6) only in the first sub-tile: later ones take
                        // them from the face, because global memory may already hold level
                        // l+1 there (written by the previous sub-tile of this block)
                        for (int c = gtid + (j2 > 0 ? 6 : 0); c < (full ? W : 6); c += 32 * nw) {
                            const int64_t y = ybase + c;
                            if (y < 0 || y >= S2) continue;
                            float* d = (c >= 6 || l == 0) ? dpl + pp * RS + c + 2 : fcur + (l * NX + pp) * 6 + c;
                            cp_async4(d, row + y);
                        }
                    }
                }
            }
            // stage for the pair that starts at level 0 (if any)
            if ((sched[0] & 15) == 2) {
                const int* gn = geo + 1 * kGeo;
                const float* src = p.plane[(tb + 0) & 1];
                float* const st = stage;               // pair parity 0
                int slot = 0;
                for (int seg = 0; seg < 2; ++seg)
                    for (int X = gn[2 * seg]; X < gn[2 * seg + 1]; ++X, ++slot) {
                        const int64_t x = xs + X;
                        if (x == 0 || x == S1 - 1) continue;
                        const float* row = src + x * S2;
                        for (int c = tid; c < SR; c += nthr) {
                            const int64_t y = a - 4 + c - 0;
                            if (y >= 0 && y < S2) cp_async4(st + slot * SR + c, row + y);
                        }
                    }
            }
            cp_async_wait_all();
        }
        if (j2 > 0) {                                   // halo of the first pass from the face
            float* const R0 = (((sched[0] >> 4) + 1) & 1) ? pl1 : pl0;
            for (int i = tid; i < NX * 6; i += nthr) {
                const int pp = i / 6, c = i - pp * 6;
                R0[pp * RS + 2 + c] = fcur[pp * 6 + c];  // level 0 entry, ring rows included
            }
        }
        __syncthreads();

        int npair = 0;                                  // pairs done in this sub-tile (stage parity)
        for (int l = 0; l < nlev;) {
            const int type = sched[l] & 15, k = sched[l] >> 4;
            const float* const R = ((k + 1) & 1) ? pl1 : pl0;   // level l-1
            float* const Wp = (k & 1) ? pl1 : pl0;            // level l (single) or l+1 (pair)
            const int lout = type == 2 ? l + 1 : l;     // level stored by this pass
            const int* g = geo + l * kGeo;
            // halo slots of the next pass's read plane (= Wp), from the face of level lout+1
            // and the face of level l (its last 6 columns of level l-1) for the next sub-tile
            for (int i = tid; i < NX * 6; i += nthr) {
                const int pp = i / 6, c = i - pp * 6;
                const int64_t xr = xs + pp;
                fnxt[(l * NX + pp) * 6 + c] = R[pp * RS + tS2 + 2 + c];
                if (lout + 1 < nlev && xr != 0 && xr != S1 - 1)
                    Wp[pp * RS + 2 + c] = fcur[((lout + 1) * NX + pp) * 6 + c];
            }
            // ring rows of Wp at the skew of level lout
            if (xs <= 0 || xs + NX > S1 - 1) {
                for (int i = tid; i < 2 * (tS2 + 6); i += nthr) {
                    const int64_t xr = (i < tS2 + 6) ? 0 : S1 - 1;
                    const int slot = 2 + (i % (tS2 + 6));
                    const int pp = (int)(xr - xs);
                    if (pp < 0 || pp >= NX) continue;
                    const int64_t y = a + slot - 8 - lout;
                    Wp[pp * RS + slot] = (y >= 0 && y < S2) ? __ldcg(p.in + xr * S2 + y) : 0.0f;
                }
            }
            // prefetch the stage of the next pair (values of its first level, rows F(second))
            if (!p.compute_only) {
                const int ln = lout + 1;
                if (ln + 1 < nlev && (sched[ln] & 15) == 2) {
                    const int* gn = geo + (ln + 1) * kGeo;
                    const float* src = p.plane[(tb + ln) & 1];
                    float* const st = stage + ((npair + (type == 2 ? 1 : 0)) & 1) * 4 * SR;
                    int slot = 0;
                    for (int seg = 0; seg < 2; ++seg)
                        for (int X = gn[2 * seg]; X < gn[2 * seg + 1]; ++X, ++slot) {
                            const int64_t x = xs + X;
                            if (x == 0 || x == S1 - 1) continue;
                            const float* row = src + x * S2;
                            for (int c = tid; c < SR; c += nthr) {
                                const int64_t y = a - 4 + c - ln;
                                if (y >= 0 && y < S2) cp_async4(st + slot * SR + c, row + y);
                            }
                        }
                }
            }

            if (!g[7]) {
                if (type == 1) {
                    // ---------------- single-level pass (K1 body, K1P layout)
                    const int seg = g[12];
                    const int pa = g[8] + grp * seg;
                    const int pe = min(g[9], pa + seg);
                    if (pa < pe) {
                        const int y0 = (int)(u0 - l);
                        const bool allvalid = (y0 >= 1) && (y0 + 3 <= S2i - 2);
                        const unsigned nwlo = (unsigned)g[10], nwlen = (unsigned)(g[11] - g[10]);
                        float* gp = p.plane[(tb + l) & 1] + (xs + pa) * S2 + y0;
                        const float* __restrict__ rp = R + (pa - 1) * RS + s;
                        float* __restrict__ wp = Wp + pa * RS + s;
                        int pp = pa;
                        auto step = [&](const float(&r0)[6], const float(&r1)[6], float(&r2)[6]) {
                            ld6(rp, r2);
                            rp += RS;
                            float o[4];
#pragma unroll
                            for (int kk = 0; kk < 4; ++kk) o[kk] = point2<KIND, MODE, HASC, DEFW, 6>(r0, r1, r2, kk, p);
                            if (!allvalid) {
                                const float* inrow = p.in + (xs + pp) * S2;
#pragma unroll
                                for (int kk = 0; kk < 4; ++kk) {
                                    const int y = y0 + kk;
                                    if ((y == 0 || y == S2i - 1) && !p.compute_only) o[kk] = __ldcg(inrow + y);
                                    else if (y < 1 || y > S2i - 2) o[kk] = 0.0f;
                                }
                            }
                            if (store_lane) *reinterpret_cast<float4*>(wp) = make_float4(o[0], o[1], o[2], o[3]);
                            wp += RS;
                            if (store_lane && (unsigned)(pp - (int)nwlo) >= nwlen && !p.compute_only) {
#pragma unroll
                                for (int kk = 0; kk < 4; ++kk)
                                    if (allvalid || (y0 + kk >= 1 && y0 + kk <= S2i - 2)) gp[kk] = o[kk];
                            }
                            gp += S2;
                            ++pp;
                        };
                        float A[6], B[6], C[6];
                        ld6(rp, A);
                        rp += RS;
                        ld6(rp, B);
                        rp += RS;
                        int n = pe - pa;
                        for (; n >= 3; n -= 3) {
                            step(A, B, C);
                            step(B, C, A);
                            step(C, A, B);
                        }
                        if (n >= 1) step(A, B, C);
                        if (n >= 2) step(B, C, A);
                    }
                } else {
                    // ---------------- pair pass: levels l (registers) and l+1 (stored)
                    const int* gn = geo + (l + 1) * kGeo;
                    const int rl = g[8], rr = g[9];                       // level l rows
                    const int rln = gn[8], rrn = gn[9];                   // level l+1 rows
                    const int segn = (rrn - rln + G - 1) / G;
                    const int a1 = rln + grp * segn;
                    const int e1 = min(rrn, a1 + segn);
                    if (a1 < e1) {
                        // level-l rows this group produces: [a1-1, e1+1); rows it owns (facets):
                        const int own_lo = grp == 0 ? -1000 : a1;
                        const int own_hi = (a1 + segn >= rrn) ? 1000 : e1;
                        const int y0 = (int)(u0 - l);                     // level l, column 0
                        const int y1 = y0 - 1;                            // level l+1
                        const bool allv0 = (y0 >= 1) && (y0 + 3 <= S2i - 2);
                        const bool allv1 = (y1 >= 1) && (y1 + 3 <= S2i - 2);
                        const unsigned nwlo0 = (unsigned)g[10], nwlen0 = (unsigned)(g[11] - g[10]);
                        const unsigned nwlo1 = (unsigned)gn[10], nwlen1 = (unsigned)(gn[11] - gn[10]);
                        const int f1a = gn[0], f1n = gn[1] - gn[0], f2a = gn[2];
                        const float* const st = stage + (npair & 1) * 4 * SR + colbase;
                        float* const gpl0 = p.plane[(tb + l) & 1];
                        float* const gpl1 = p.plane[(tb + l + 1) & 1];
                        const float* __restrict__ rp = R + (a1 - 2) * RS + s;       // level l-1 row x-1 at x = a1-1
                        int x = a1 - 1;
                        // one step: level l at row x (from level l-1 rows x-1..x+1 = P0, P1, P2),
                        // then level l+1 at row x-1 (from level l rows x-2..x = L0, L1, L2)
                        auto pstep = [&](const float(&P0)[6], const float(&P1)[6], float(&P2)[6],
                                         const float(&L0)[6], const float(&L1)[6], float(&L2)[6]) {
                            ld6(rp, P2);
                            rp += RS;
                            float o[4];
                            const int64_t xg = xs + x;
                            if (x >= rl && x < rr) {
#pragma unroll
                                for (int kk = 0; kk < 4; ++kk) o[kk] = point2<KIND, MODE, HASC, DEFW, 6>(P0, P1, P2, kk, p);
                                if (!allv0) {
                                    const float* inrow = p.in + xg * S2;
#pragma unroll
                                    for (int kk = 0; kk < 4; ++kk) {
                                        const int y = y0 + kk;
                                        if ((y == 0 || y == S2i - 1) && !p.compute_only) o[kk] = __ldcg(inrow + y);
                                        else if (y < 1 || y > S2i - 2) o[kk] = 0.0f;
                                    }
                                }
                                if (store_lane && x >= own_lo && x < own_hi &&
                                    (unsigned)(x - (int)nwlo0) >= nwlen0 && !p.compute_only) {
                                    float* gp = gpl0 + xg * S2 + y0;
#pragma unroll
                                    for (int kk = 0; kk < 4; ++kk)
                                        if (allv0 || (y0 + kk >= 1 && y0 + kk <= S2i - 2)) gp[kk] = o[kk];
                                }
                            } else if (xg == 0 || xg == S1 - 1) {           // ring row at the skew of level l
                                const float* inrow = p.in + xg * S2;
#pragma unroll
                                for (int kk = 0; kk < 4; ++kk) {
                                    const int y = y0 + kk;
                                    o[kk] = (y >= 0 && y < S2i && !p.compute_only) ? __ldcg(inrow + y) : 0.0f;
                                }
                            } else {                                         // footprint row of level l+1
                                const int slot = (x >= f1a && x - f1a < f1n) ? x - f1a : f1n + (x - f2a);
                                const float4 q4 = *reinterpret_cast<const float4*>(st + slot * SR);
                                o[0] = q4.x; o[1] = q4.y; o[2] = q4.z; o[3] = q4.w;
                            }
                            L2[0] = __shfl_up_sync(kFullMask, o[2], 1);
                            L2[1] = __shfl_up_sync(kFullMask, o[3], 1);
                            L2[2] = o[0]; L2[3] = o[1]; L2[4] = o[2]; L2[5] = o[3];
                            const int xm = x - 1;
                            if (xm >= a1) {
                                float q[4];
#pragma unroll
                                for (int kk = 0; kk < 4; ++kk) q[kk] = point2<KIND, MODE, HASC, DEFW, 6>(L0, L1, L2, kk, p);
                                const int64_t xmg = xg - 1;
                                if (!allv1) {
                                    const float* inrow = p.in + xmg * S2;
#pragma unroll
                                    for (int kk = 0; kk < 4; ++kk) {
                                        const int y = y1 + kk;
                                        if ((y == 0 || y == S2i - 1) && !p.compute_only) q[kk] = __ldcg(inrow + y);
                                        else if (y < 1 || y > S2i - 2) q[kk] = 0.0f;
                                    }
                                }
                                if (store_lane)
                                    *reinterpret_cast<float4*>(Wp + xm * RS + s) = make_float4(q[0], q[1], q[2], q[3]);
                                if (store_lane && (unsigned)(xm - (int)nwlo1) >= nwlen1 && !p.compute_only) {
                                    float* gp = gpl1 + xmg * S2 + y1;
#pragma unroll
                                    for (int kk = 0; kk < 4; ++kk)
                                        if (allv1 || (y1 + kk >= 1 && y1 + kk <= S2i - 2)) gp[kk] = q[kk];
                                }
                            }
                            ++x;
                        };
                        float PA[6], PB[6], PC[6], LA[6], LB[6], LC[6];
                        ld6(rp, PA);
                        rp += RS;
                        ld6(rp, PB);
                        rp += RS;
#pragma unroll
                        for (int kk = 0; kk < 6; ++kk) { LA[kk] = 0.0f; LB[kk] = 0.0f; }
                        int n = e1 - a1 + 2;                                 // steps x = a1-1 .. e1
                        for (; n >= 3; n -= 3) {                             // rotating names, no moves
                            pstep(PA, PB, PC, LA, LB, LC);
                            pstep(PB, PC, PA, LB, LC, LA);
                            pstep(PC, PA, PB, LC, LA, LB);
                        }
                        if (n >= 1) pstep(PA, PB, PC, LA, LB, LC);
                        if (n >= 2) pstep(PB, PC, PA, LB, LC, LA);
                    }
                }
            }
            if (!p.compute_only) cp_async_wait_all();
            __syncthreads();
            if (type == 2) ++npair;
            l += (type == 2) ? 2 : 1;
        }
    }
}

// ----------------------------------------------------------------- dispatch
template <int KIND, int MODE>
static hex_kernel_t pick_pair_mode(bool has_c, bool defw) {
    if (defw) return hex2d_pair_kernel<KIND, MODE, false, true>;
    if (KIND != STENCIL_GRADIENT2D && has_c) return hex2d_pair_kernel<KIND, MODE, true, false>;
    return hex2d_pair_kernel<KIND, MODE, false, false>;
}

template <int KIND>
static hex_kernel_t pick_pair_kind(int mode, bool has_c, bool defw) {
    return mode == STENCIL_MODE_FUSED ? pick_pair_mode<KIND, 1>(has_c, defw) : pick_pair_mode<KIND, 0>(has_c, defw);
}

hex_kernel_t get_hex_pair_kernel(int kind, int mode, bool has_c, bool defw) {
    switch (kind) {
    case STENCIL_JACOBI2D_5PT: return pick_pair_kind<STENCIL_JACOBI2D_5PT>(mode, has_c, defw);
    case STENCIL_HEAT2D_9PT: return pick_pair_kind<STENCIL_HEAT2D_9PT>(mode, has_c, defw);
    case STENCIL_GRADIENT2D: return pick_pair_kind<STENCIL_GRADIENT2D>(mode, false, defw);
    case STENCIL_LAPLACIAN2D_5PT: return pick_pair_kind<STENCIL_LAPLACIAN2D_5PT>(mode, has_c, defw);
    default: return nullptr;
    }
}

}  // namespace hhc
