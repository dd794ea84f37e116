// wave_kernels.cu -- wavefront-parallel Jacobi-1D (K3).
//
// The paper's generality claim: "Consider, wavefront parallel
// Jacobi1D stencil.  The total execution time is the sum of the times for each
// wavefront ... equation 6 holds for wavefront parallel codes."  This is that
// second schedule on the same Eq. 1 update and the same oracle:
// parallelogram tiles of tT levels x tS columns in skewed coordinates
// x' = x + t (classic time skewing), one launch per anti-diagonal i + j = d
// (the wavefront), one thread block per tile.  DESIGN.md reading W1.
//
// In skewed coordinates the update of (t, x') reads (t-1, x'-2), (t-1, x'-1)
// and (t-1, x'), so a tile needs the bottom row of its band (level t0, written
// by band i-1 as its top rows) and two halo columns per level from its left
// neighbour (i, j-1), both finished by earlier wavefronts.  A tile writes to
// global memory only what later tiles read: its two rightmost columns of every
// level and its top row.  Two parity planes (level t in plane[t & 1]); no
// value a later reader needs is overwritten early because a write of
// (t+2, x) belongs to a tile at the same or a later wavefront than every
// reader of (t, x) (reading W1).
#include <cuda_runtime.h>

#include "hhc_internal.h"

namespace hhc {

// VEC (tS % 4 == 0): each thread computes aligned groups of 4 slots (one LDS.128 + one
// LDS.64 of the level below, one STS.128), with a branch-free body when the whole
// level lies inside the interior; rows start 2 floats into a 16-B line so that
// slot 2 (the tile's first own column) is 16-B aligned.
template <int MODE, bool HASC, bool DEFW, bool VEC>
__global__ void __launch_bounds__(256) wave1d_kernel(const __grid_constant__ WaveParams p) {
    extern __shared__ __align__(16) float smw[];
    const int tS = p.tS, tT = p.tT;
    const int RW = tS + 2;                                   // slots k: x' = j*tS - 2 + k
    const int RWP = (RW + 2 + 3) & ~3;                       // padded row: slot k at row[2 + k]
    float* const buf0 = smw + 2;
    float* const buf1 = smw + RWP + 2;
    float* const halo = smw + 2 * RWP;                       // [tT][2]: columns k = 0, 1 of level t0 + l
    const int nthr = blockDim.x, tid = threadIdx.x;
    const int64_t i = p.ia + blockIdx.x, j = p.d - i;
    const int64_t t0 = i * tT;                               // input level of the band
    const int nlev = (int)min((int64_t)tT, p.T - t0);
    const int64_t xb = j * tS - 2;                           // skewed column of slot 0
    const int64_t S = p.S;
    const float third = 1.0f / 3.0f;
    const float w0 = DEFW ? third : p.w[0], w1 = DEFW ? third : p.w[1], w2 = DEFW ? third : p.w[2];
    {
        const float* src = p.plane[t0 & 1];
        const int64_t x0 = xb - t0;                          // x of slot 0 at level t0
        if (x0 >= 0 && x0 + RW <= S) {                       // the whole bottom row is in the array:
            const float* s0 = src + x0;                      // unchecked, unrolled for loads in flight
#pragma unroll 8
            for (int k = tid; k < RW; k += nthr) buf0[k] = __ldcg(s0 + k);
        } else {
            for (int k = tid; k < RW; k += nthr) {
                const int64_t x = x0 + k;
                buf0[k] = (x >= 0 && x < S) ? __ldcg(src + x) : 0.0f;
            }
        }
        for (int e = tid; e < 2 * (nlev - 1); e += nthr) {
            const int l = 1 + (e >> 1), k = e & 1;
            const int64_t t = t0 + l;
            const int64_t x = xb + k - t;
            halo[2 * l + k] = (x >= 0 && x < S) ? __ldcg(p.plane[t & 1] + x) : 0.0f;
        }
    }
    __syncthreads();
    auto pt = [&](float a, float b, float c) {                // canonical order d1 = -1, 0, 1 (R4)
        float acc;
        if constexpr (MODE == STENCIL_MODE_FUSED) {
            acc = __fmul_rn(w0, a);
            acc = __fmaf_rn(w1, b, acc);
            acc = __fmaf_rn(w2, c, acc);
        } else {
            acc = __fmul_rn(w0, a);
            acc = __fadd_rn(acc, __fmul_rn(w1, b));
            acc = __fadd_rn(acc, __fmul_rn(w2, c));
        }
        if constexpr (HASC) acc = __fadd_rn(acc, p.c);
        return acc;
    };
    for (int l = 1; l <= nlev; ++l) {
        const int64_t t = t0 + l;
        const float* const prev = (l & 1) ? buf0 : buf1;
        float* const cur = (l & 1) ? buf1 : buf0;
        float* const dst = p.plane[t & 1];
        if (tid < 2 && l < nlev) cur[tid] = halo[2 * l + tid];
        const bool top = l == nlev;
        if constexpr (VEC) {
            // slots 2 .. RW-1 in aligned groups of 4; x of slot k is xb + k - t
            const int64_t xlo = xb + 2 - t, xhi = xb + RW - 1 - t;
            if (xlo >= 1 && xhi <= S - 2) {                      // the whole level is interior
                for (int k = 2 + 4 * tid; k < RW; k += 4 * nthr) {
                    const float2 lo = *reinterpret_cast<const float2*>(prev + k - 2);
                    const float4 v = *reinterpret_cast<const float4*>(prev + k);
                    const float4 o = make_float4(pt(lo.x, lo.y, v.x), pt(lo.y, v.x, v.y), pt(v.x, v.y, v.z),
                                                 pt(v.y, v.z, v.w));
                    *reinterpret_cast<float4*>(cur + k) = o;
                    if (top) {
                        float* g = dst + (xb + k - t);
                        g[0] = o.x; g[1] = o.y; g[2] = o.z; g[3] = o.w;
                    } else if (k + 4 >= RW) {                    // the group holding slots tS, tS+1
                        dst[xb + tS - t] = o.z;
                        dst[xb + tS + 1 - t] = o.w;
                    }
                }
                __syncthreads();
                continue;
            }
        }
        for (int k = 2 + tid; k < RW; k += nthr) {
            const int64_t x = xb + k - t;
            // interior: Eq. 1; the ring (x = 0, S-1) keeps its value, which sits
            // one slot to the left one level below; farther out is never read
            const bool in = x >= 1 && x <= S - 2;
            const float v = in ? pt(prev[k - 2], prev[k - 1], prev[k]) : prev[k - 1];
            cur[k] = v;
            if (in && (top || k >= tS)) dst[x] = v;
        }
        __syncthreads();
    }
}

static void (*pick_wave1d(int mode, bool has_c, bool defw, bool vec))(WaveParams) {
    void (*k)(WaveParams);
    if (vec) {
        if (mode == STENCIL_MODE_FUSED)
            k = defw ? wave1d_kernel<1, false, true, true> : has_c ? wave1d_kernel<1, true, false, true> : wave1d_kernel<1, false, false, true>;
        else
            k = defw ? wave1d_kernel<0, false, true, true> : has_c ? wave1d_kernel<0, true, false, true> : wave1d_kernel<0, false, false, true>;
    } else {
        if (mode == STENCIL_MODE_FUSED)
            k = defw ? wave1d_kernel<1, false, true, false> : has_c ? wave1d_kernel<1, true, false, false> : wave1d_kernel<1, false, false, false>;
        else
            k = defw ? wave1d_kernel<0, false, true, false> : has_c ? wave1d_kernel<0, true, false, false> : wave1d_kernel<0, false, false, false>;
    }
    return k;
}

// the kernel's dynamic shared-memory limit, set outside any stream capture
int prepare_wave1d(int mode, bool has_c, bool defw, int tT, int tS) {
    auto k = pick_wave1d(mode, has_c, defw, tS % 4 == 0);
    const int64_t smem = wave1d_smem_bytes(tT, tS);
    cudaError_t e = cudaFuncSetAttribute((const void*)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    return e == cudaSuccess ? STENCIL_OK : STENCIL_ECUDA;
}

int launch_wave1d(int mode, bool has_c, bool defw, const WaveParams& p, int64_t nblocks, void* stream) {
    auto k = pick_wave1d(mode, has_c, defw, p.tS % 4 == 0);
    const int64_t smem = wave1d_smem_bytes(p.tT, p.tS);
    void* args[] = {const_cast<WaveParams*>(&p)};
    cudaError_t e = cudaLaunchKernel((const void*)k, dim3((unsigned)nblocks), dim3(256), args, (size_t)smem,
                                     (cudaStream_t)stream);
    return e == cudaSuccess ? STENCIL_OK : STENCIL_ECUDA;
}

}  // namespace hhc
