// Isolated K1 main loop (pair layout, Heat-2D fused FFMA2, software-pipelined
// 4-row window) without barriers: cycles per warp-step.
#include <cstdio>
#include <cuda_runtime.h>
#include "../../paper_conf_ppopp_prajapatirradg17_b200/csrc/hhc_device.cuh"
using namespace hhc;
__device__ __forceinline__ int chunk_off(int c) { return 4 * (c ^ ((c >> 3) & 1)); }
__device__ __forceinline__ void ldpairs(const float* row, int oh, int od0, int od1, float2 (&r)[6]) {
    const float4 h = *reinterpret_cast<const float4*>(row + oh);
    const float4 m = *reinterpret_cast<const float4*>(row + od0);
    const float4 q = *reinterpret_cast<const float4*>(row + od1);
    r[0] = make_float2(h.x, h.y); r[1] = make_float2(h.z, h.w);
    r[2] = make_float2(m.x, m.y); r[3] = make_float2(m.z, m.w);
    r[4] = make_float2(q.x, q.y); r[5] = make_float2(q.z, q.w);
}
template <int VAR>
__global__ void __launch_bounds__(384, 1) loop(const __grid_constant__ HexParams p, int nsteps, int rows, long long* cyc, float* sink) {
    extern __shared__ __align__(16) float sm[];
    const int tS2 = 512, RS = tS2 + 8, D = 256;
    const int ncol = 64, col = threadIdx.x % ncol, grp = threadIdx.x / ncol;
    const int oh = chunk_off(2 * col), od0 = chunk_off(2 * col + 1), od1 = chunk_off(2 * col + 2);
    float* prev = sm;
    float* cur = sm + rows * RS;
    for (int i = threadIdx.x; i < 2 * rows * RS; i += blockDim.x) sm[i] = i * 1e-6f;
    __syncthreads();
    const bool last_col = col == ncol - 1;
    int nwlo = -100, nwhi = 1000;
    const unsigned nwlen = nwhi - nwlo;
    float* gp = sink + threadIdx.x;
    __shared__ volatile int done[16];
    if (threadIdx.x < 16) done[threadIdx.x] = 0;
    __syncthreads();
    const int G = blockDim.x / ncol;
    int lev = 0;
    long long t0 = clock64();
    for (int rep = 0; rep < nsteps; rep += rows - 2) {
        if (VAR == 4 && (threadIdx.x & 31) == 0) {
            // wait for the neighbour groups to finish the previous level
            while ((grp > 0 && done[grp - 1] < lev) || (grp + 1 < G && done[grp + 1] < lev)) {}
        }
        if (VAR == 4) { __syncwarp(); __threadfence_block(); }
        const float* rp = prev + grp * 0 * RS;
        float* wp = cur + RS;
        int pp = 1;
        auto step = [&](const float2(&r0)[6], const float2(&r1)[6], const float2(&r2)[6], float2(&r3)[6]) {
            ldpairs(rp, oh, od0, od1, r3);
            rp += RS;
            float2 o[4];
#pragma unroll
            for (int k = 0; k < 4; ++k)
                o[k] = lin2x2<STENCIL_HEAT2D_9PT, false, true>(r0, r1, r2, k, p, std::make_integer_sequence<int, 9>{});
            *reinterpret_cast<float4*>(wp + od0) = make_float4(o[0].x, o[0].y, o[1].x, o[1].y);
            *reinterpret_cast<float4*>(wp + od1) = make_float4(o[2].x, o[2].y, o[3].x, o[3].y);
            if (VAR >= 1 && last_col) { wp[1] = o[2].x; wp[3] = o[3].x; }
            wp += RS;
            if (VAR >= 2 && (unsigned)(pp - nwlo) >= nwlen) {
#pragma unroll
                for (int k = 0; k < 4; ++k) { gp[k] = o[k].x; gp[D + k] = o[k].y; }
            }
            gp += 1024;
            ++pp;
        };
        float2 A[6], Bv[6], C[6], E[6];
        ldpairs(rp, oh, od0, od1, A); rp += RS;
        ldpairs(rp, oh, od0, od1, Bv); rp += RS;
        ldpairs(rp, oh, od0, od1, C); rp += RS;
        int n = rows - 4;
        for (; n >= 4; n -= 4) {
            step(A, Bv, C, E); step(Bv, C, E, A); step(C, E, A, Bv); step(E, A, Bv, C);
        }
        if (n >= 1) step(A, Bv, C, E);
        if (n >= 2) step(Bv, C, E, A);
        if (n >= 3) step(C, E, A, Bv);
        float* t = prev; prev = cur; cur = t;
        if (VAR == 3) __syncthreads();
        else if (VAR == 4) {
            asm volatile("bar.sync %0, %1;" :: "r"(1 + grp), "r"(ncol) : "memory");
            if (col == 0) { __threadfence_block(); done[grp] = lev + 1; }
        } else __syncwarp();
        ++lev;
    }
    long long t1 = clock64();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
int main() {
    HexParams p{};
    float* sink; cudaMalloc(&sink, 64 << 20);
    long long* cyc; cudaMalloc(&cyc, 8 * 1024);
    for (int var = 1; var < 5; ++var)
        for (int thr : {384})
            for (int rows : {7, 8, 9, 12, 20}) {
                if (var == 2) continue;
                auto k = var == 1 ? loop<1> : var == 3 ? loop<3> : loop<4>;
                int smem = 2 * rows * 520 * 4;
                cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
                const int nsteps = 4000;
                k<<<148, thr, smem>>>(p, nsteps, rows, cyc, sink);
                cudaDeviceSynchronize();
                long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
                int reps = (nsteps + rows - 3) / (rows - 2);
                double wsteps = (double)reps * (rows - 4) * thr / 32;   // warp-steps per block
                printf("var %d thr %d rows %2d: %.1f cycles per warp-step per SM, %.2f pts/clk/SM (FP bound 14.2) err=%s\n", var, thr, rows,
                       c / wsteps, wsteps * 256 / c, cudaGetErrorString(cudaGetLastError()));
            }
}
