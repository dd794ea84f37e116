// FFMA2 / FFMA dependent-chain latency and per-warp throughput vs number of
// independent chains (one CTA of W warps per SM).
#include <cstdio>
#include <cuda_runtime.h>
template <int K, bool PACKED>
__global__ void k(float* out, int iters) {
    float2 a[K];
    for (int i = 0; i < K; ++i) a[i] = make_float2(threadIdx.x * 1e-7f + i, i + 0.5f);
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 8; ++r)
#pragma unroll
            for (int i = 0; i < K; ++i) {
                if (PACKED) a[i] = __ffma2_rn(a[i], make_float2(0.999f, 0.999f), make_float2(0.5f, 0.5f));
                else { a[i].x = __fmaf_rn(a[i].x, 0.999f, 0.5f); }
            }
    }
    long long t1 = clock64();
    float s = 0;
    for (int i = 0; i < K; ++i) s += a[i].x + a[i].y;
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0 && blockIdx.x == 0) out[0] = (float)(t1 - t0);
}
template <int K, bool P>
void run(float* out, int warps) {
    const int iters = 2000;
    k<K, P><<<1, 32 * warps>>>(out, iters);
    cudaDeviceSynchronize();
    float c; cudaMemcpy(&c, out, 4, cudaMemcpyDeviceToHost);
    double per = c / (iters * 8.0 * K);
    printf("%s K=%d warps=%2d: %.2f cycles per instr per warp  (%.2f instr/cycle/SM)\n", P ? "FFMA2" : "FFMA ", K, warps,
           per, warps / per);
}
int main() {
    float* out; cudaMalloc(&out, 1 << 20);
    for (int w : {1, 4, 8, 16}) {
        run<1, true>(out, w); run<2, true>(out, w); run<4, true>(out, w); run<8, true>(out, w);
        run<1, false>(out, w); run<4, false>(out, w); run<8, false>(out, w);
    }
}
