// hhc_kernels_reg.cu -- K1R: the register-resident 2D HHC kernel.
//
// Same tiling, schedule and global I/O as K1 (hex2d_kernel): one thread block
// per hexagonal prism, sub-tiles of tS2 skewed columns swept
// in order, rows of the hexagon bottom to top with one barrier per level
// (Eq. 15's tau_sync per row).  What changes is where the hexagon lives: each
// thread owns 4 consecutive skewed columns of EVERY hexagon row in registers
// (v[NR][4], NR >= tS1+tT+2), so a level is computed in place from registers
// (SURVEY §8(a) a5).  The S1 neighbours are the thread's own registers; the
// two S2 neighbours to the left come from the left lane by warp shuffle, and
// lane 0 reads them from a small shared-memory exchange written by the left
// warp's lane 31 at the previous level (or from the previous sub-tile's face,
// or from global memory for rows the block did not compute).  Footprint rows
// (values produced by other hexagons, readings G3) are staged one level ahead
// with cp.async; facet rows are stored straight from registers.
#include "hhc_device.cuh"

namespace hhc {

namespace {
constexpr unsigned kFull = 0xffffffffu;

// Rows are compile-time register indices: a tiny integral-constant helper.
template <int R>
using IC = std::integral_constant<int, R>;

template <typename F, int... R>
__device__ __forceinline__ void for_rows(F&& f, std::integer_sequence<int, R...>) {
    (f(IC<R>{}), ...);
}
}  // namespace

template <int KIND, int MODE, bool DEFW, int NR>
__global__ void __launch_bounds__(256, 1) hex2d_reg_kernel(const __grid_constant__ HexParams p) {
    extern __shared__ __align__(16) float sm[];
    const int tT = p.tT, tS1 = p.tS1, tS2 = p.tS2;
    const int NX = tS1 + tT + 2;                       // <= NR (host check)
    const int nthr = blockDim.x;                       // = tS2 / 4
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nw = nthr >> 5;
    const int64_t S1 = p.S1, S2 = p.S2;
    const int S2i = (int)S2;
    const int64_t x0 = p.xbase + (int64_t)blockIdx.x * p.P;
    const int64_t xs = x0 - tT / 2 - 1;                // register row 0 is x = xs
    const int nlev = p.tau_hi - p.tau_lo;
    const int64_t tb = p.t0 + p.tau_lo;
    float* const stage = sm;                           // [2][4][tS2]   footprint rows of the next level
    float* const xch = stage + 2 * 4 * tS2;            // [2][nw][NR][2] lane 31 -> lane 0 of the next warp
    float* const face = xch + 2 * nw * NR * 2;         // [2][tT+1][NR][2] last lane -> next sub-tile
    int* const geo = reinterpret_cast<int*>(face + 2 * (tT + 1) * NR * 2);   // [tT][kGeo]
    build_geo(p, x0, xs, nlev, geo);
    __syncthreads();

    float v[NR][4];
#pragma unroll
    for (int r = 0; r < NR; ++r)
#pragma unroll
        for (int k = 0; k < 4; ++k) v[r][k] = 0.0f;

    for (int j2 = 0; j2 < p.n2; ++j2) {
        const int64_t a = 1 + (int64_t)j2 * tS2;
        const int64_t u0 = a + 4 * tid;                // skewed column of this thread's k = 0
        float* const fcur = face + (j2 & 1) * (tT + 1) * NR * 2;
        float* const fnxt = face + ((j2 + 1) & 1) * (tT + 1) * NR * 2;

        // first sub-tile: the halo of warp 0 lane 0 is the ring / level -1 input
        if (j2 == 0 && !p.compute_only) {
            for (int i = tid; i < nlev * NX * 2; i += nthr) {
                const int lev = i / (NX * 2), X = (i / 2) % NX, c = i & 1;
                const float* src = p.plane[(tb + lev - 1) & 1];
                const int64_t x = xs + X, y = a - 1 + c - lev;
                fcur[(lev * NR + X) * 2 + c] =
                    (x >= 0 && x < S1 && y >= 0 && y < S2) ? __ldcg(src + x * S2 + y) : 0.0f;
            }
            __syncthreads();
        }

        for (int lev = 0; lev < nlev; ++lev) {
            const int* g = geo + lev * kGeo;
            if (g[7]) {                                 // empty level (hexagon clipped here)
                __syncthreads();
                continue;
            }
            const bool first = g[6] != 0;
            const int rl = g[8], rr = g[9];
            const unsigned nwlo = (unsigned)g[10], nwlen = (unsigned)(g[11] - g[10]);
            const unsigned long long fmask = (unsigned long long)(unsigned)g[13] |
                                             ((unsigned long long)(unsigned)g[14] << 32);
            const int f1a = g[0], f1n = g[1] - g[0], f2a = g[2];
            const float* const srcp = p.plane[(tb + lev - 1) & 1];     // values of level lev-1
            // lane-0 halo source of this level (values of level lev-1)
            float* const rd = warp == 0 ? fcur + lev * NR * 2 : xch + ((((lev - 1) & 1) * nw + warp - 1) * NR) * 2;
            const int64_t yprev = u0 - (lev - 1);      // y of column k = 0 at level lev-1

            // (1) first level of the hexagon in this sub-tile: rows row +- 1 straight from global
            if (first && !p.compute_only) {
                const int A0 = g[0], A1 = g[1];
                for_rows([&](auto Rc) {
                    constexpr int R = decltype(Rc)::value;
                    if (R >= A0 && R < A1) {
                        const int64_t x = xs + R;
                        const float* row = srcp + x * S2;
#pragma unroll
                        for (int k = 0; k < 4; ++k) {
                            const int64_t y = yprev + k;
                            v[R][k] = (y >= 0 && y < S2) ? __ldcg(row + y) : 0.0f;
                        }
                        if (lane == 0) {
#pragma unroll
                            for (int c = 0; c < 2; ++c) {
                                const int64_t y = yprev - 2 + c;
                                rd[R * 2 + c] = (y >= 0 && y < S2) ? __ldcg(row + y) : 0.0f;
                            }
                        }
                    }
                }, std::make_integer_sequence<int, NR>{});
            }
            // (2) ring rows x = 0, S1-1 hold the ring at this level's skew
            if ((xs <= 0 || xs + NX > S1 - 1) && !p.compute_only) {
                for_rows([&](auto Rc) {
                    constexpr int R = decltype(Rc)::value;
                    const int64_t x = xs + R;
                    if (x == 0 || x == S1 - 1) {
                        const float* row = p.in + x * S2;
#pragma unroll
                        for (int k = 0; k < 4; ++k) {
                            const int64_t y = yprev + k;
                            v[R][k] = (y >= 0 && y < S2) ? __ldcg(row + y) : 0.0f;
                        }
                        if (lane == 0) {
#pragma unroll
                            for (int c = 0; c < 2; ++c) {
                                const int64_t y = yprev - 2 + c;
                                rd[R * 2 + c] = (y >= 0 && y < S2) ? __ldcg(row + y) : 0.0f;
                            }
                        }
                    }
                }, std::make_integer_sequence<int, NR>{});
            }
            // (3) prefetch the footprint rows of level lev+1 (values of level lev, at most 4 rows)
            if (!p.compute_only && lev + 1 < nlev) {
                const int* gn = geo + (lev + 1) * kGeo;
                if (!gn[6] && !gn[7]) {
                    const float* src = p.plane[(tb + lev) & 1];
                    float* const st = stage + ((lev + 1) & 1) * 4 * tS2 + 4 * tid;
                    float* const rdn = warp == 0 ? fcur + (lev + 1) * NR * 2
                                                 : xch + (((lev & 1) * nw + warp - 1) * NR) * 2;
                    const int64_t ycur = u0 - lev;
                    int slot = 0;
                    for (int seg = 0; seg < 2; ++seg) {
                        for (int X = gn[2 * seg]; X < gn[2 * seg + 1]; ++X, ++slot) {
                            const int64_t x = xs + X;
                            if (x == 0 || x == S1 - 1) continue;   // ring rows: step (2)
                            const float* row = src + x * S2;
#pragma unroll
                            for (int k = 0; k < 4; ++k) {
                                const int64_t y = ycur + k;
                                if (y >= 0 && y < S2) cp_async4(st + slot * tS2 + k, row + y);
                            }
                            if (lane == 0) {
#pragma unroll
                                for (int c = 0; c < 2; ++c) {
                                    const int64_t y = ycur - 2 + c;
                                    if (y >= 0 && y < S2) cp_async4(rdn + X * 2 + c, row + y);
                                }
                            }
                        }
                    }
                }
            }

            // (4) the rows of this level, bottom to top, in place
            const float* const stg = stage + (lev & 1) * 4 * tS2 + 4 * tid;
            const int y0 = (int)(u0 - lev);            // y of column k = 0 at level lev
            const bool allvalid = (y0 >= 1) && (y0 + 3 <= S2i - 2);
            float* const gbase = p.plane[(tb + lev) & 1] + xs * S2 + y0;
            float* const xw = xch + (((lev & 1) * nw + warp) * NR) * 2;
            float* const fw = fnxt + (lev + 1) * NR * 2;
            const bool last_warp = warp == nw - 1;
            float po[4], hp0 = 0.0f, hp1 = 0.0f, hc0 = 0.0f, hc1 = 0.0f;
#pragma unroll
            for (int k = 0; k < 4; ++k) po[k] = 0.0f;

            auto fetch_f = [&](auto Xc) {               // footprint row X (if any) from the stage
                constexpr int X = decltype(Xc)::value;
                if ((fmask >> X) & 1ull) {
                    const int slot = (X - f1a < f1n && X >= f1a) ? X - f1a : f1n + (X - f2a);
                    const float4 q = *reinterpret_cast<const float4*>(stg + slot * tS2);
                    v[X][0] = q.x; v[X][1] = q.y; v[X][2] = q.z; v[X][3] = q.w;
                }
            };
            auto halo = [&](auto Xc, float& h0, float& h1) {
                constexpr int X = decltype(Xc)::value;
                h0 = __shfl_up_sync(kFull, v[X][2], 1);
                h1 = __shfl_up_sync(kFull, v[X][3], 1);
                if (lane == 0) {
                    const float2 q = *reinterpret_cast<const float2*>(rd + X * 2);
                    h0 = q.x;
                    h1 = q.y;
                }
            };

            for_rows([&](auto Rc) {
                constexpr int R = decltype(Rc)::value;
                if constexpr (R >= 1 && R + 1 < NR) {
                    if ((unsigned)(R - rl) < (unsigned)(rr - rl)) {
                        if (R == rl) {
                            if (!first) {
                                fetch_f(IC<R - 1>{});
                                fetch_f(IC<R>{});
                            }
#pragma unroll
                            for (int k = 0; k < 4; ++k) po[k] = v[R - 1][k];
                            halo(IC<R - 1>{}, hp0, hp1);
                            halo(IC<R>{}, hc0, hc1);
                        }
                        if (!first) fetch_f(IC<R + 1>{});
                        float hn0, hn1;
                        halo(IC<R + 1>{}, hn0, hn1);
                        const float r0[6] = {hp0, hp1, po[0], po[1], po[2], po[3]};
                        const float r1[6] = {hc0, hc1, v[R][0], v[R][1], v[R][2], v[R][3]};
                        const float r2[6] = {hn0, hn1, v[R + 1][0], v[R + 1][1], v[R + 1][2], v[R + 1][3]};
                        float o[4];
#pragma unroll
                        for (int k = 0; k < 4; ++k) o[k] = point2<KIND, MODE, false, DEFW, 6>(r0, r1, r2, k, p);
                        if (!allvalid) {
                            const float* inrow = p.in + (xs + R) * S2;
#pragma unroll
                            for (int k = 0; k < 4; ++k) {
                                const int y = y0 + k;
                                if ((y == 0 || y == S2i - 1) && !p.compute_only) o[k] = __ldcg(inrow + y);
                                else if (y < 1 || y > S2i - 2) o[k] = 0.0f;
                            }
                        }
                        if ((unsigned)(R - (int)nwlo) >= nwlen && !p.compute_only) {   // facet row (G3)
                            float* gp = gbase + (int64_t)R * S2;
#pragma unroll
                            for (int k = 0; k < 4; ++k)
                                if (allvalid || (y0 + k >= 1 && y0 + k <= S2i - 2)) gp[k] = o[k];
                        }
                        if (lane == 31) {
                            *reinterpret_cast<float2*>(xw + R * 2) = make_float2(o[2], o[3]);
                            if (last_warp) *reinterpret_cast<float2*>(fw + R * 2) = make_float2(o[2], o[3]);
                        }
#pragma unroll
                        for (int k = 0; k < 4; ++k) {
                            po[k] = v[R][k];
                            v[R][k] = o[k];
                        }
                        hp0 = hc0; hp1 = hc1;
                        hc0 = hn0; hc1 = hn1;
                    }
                }
            }, std::make_integer_sequence<int, NR>{});

            if (!p.compute_only) cp_async_wait_all();
            __syncthreads();
        }
    }
}

// ----------------------------------------------------------------- dispatch
template <int KIND, int MODE>
static hex_kernel_t pick_nr(int nr) {
    switch (nr) {
    case 16: return hex2d_reg_kernel<KIND, MODE, true, 16>;
    case 24: return hex2d_reg_kernel<KIND, MODE, true, 24>;
    case 32: return hex2d_reg_kernel<KIND, MODE, true, 32>;
    case 40: return hex2d_reg_kernel<KIND, MODE, true, 40>;
    default: return nullptr;
    }
}

template <int KIND>
static hex_kernel_t pick_reg_mode(int mode, int nr) {
    return mode == STENCIL_MODE_FUSED ? pick_nr<KIND, 1>(nr) : pick_nr<KIND, 0>(nr);
}

int reg_rows_for(int NX) {
    for (int nr : {16, 24, 32, 40})
        if (NX <= nr) return nr;
    return 0;
}

hex_kernel_t get_hex_reg_kernel(int kind, int mode, int nr) {
    switch (kind) {
    case STENCIL_JACOBI2D_5PT: return pick_reg_mode<STENCIL_JACOBI2D_5PT>(mode, nr);
    case STENCIL_HEAT2D_9PT: return pick_reg_mode<STENCIL_HEAT2D_9PT>(mode, nr);
    case STENCIL_GRADIENT2D: return pick_reg_mode<STENCIL_GRADIENT2D>(mode, nr);
    case STENCIL_LAPLACIAN2D_5PT: return pick_reg_mode<STENCIL_LAPLACIAN2D_5PT>(mode, nr);
    default: return nullptr;
    }
}

}  // namespace hhc
