// Micro-benchmark: FP32 FMA issue throughput on sm_100a, scalar FFMA vs packed
// FFMA2 (fma.rn.f32x2), immediate and register weight forms.
#include <cstdio>
#include <cuda_runtime.h>
#define N_ACC 16
template <int MODE>
__global__ void k(float* out, float w, int iters) {
    float a[N_ACC];
    unsigned long long p[N_ACC];
    for (int i = 0; i < N_ACC; ++i) { a[i] = threadIdx.x * 1e-7f + i; p[i] = (unsigned long long)__float_as_uint(a[i]) | ((unsigned long long)__float_as_uint(a[i] + 1) << 32); }
    const unsigned long long w2 = (unsigned long long)__float_as_uint(w) | ((unsigned long long)__float_as_uint(w) << 32);
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int i = 0; i < N_ACC; ++i) {
            if (MODE == 0) a[i] = __fmaf_rn(a[i], 0.999f, 0.5f);                 // imm form
            if (MODE == 1) a[i] = __fmaf_rn(a[i], w, a[(i + 1) % N_ACC]);      // 3-reg
            if (MODE == 2) asm volatile("fma.rn.f32x2 %0, %0, %1, %0;" : "+l"(p[i]) : "l"(0x3f7fbe773f7fbe77ull));
            if (MODE == 3) asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(p[i]) : "l"(w2), "l"(p[(i + 1) % N_ACC]));
        }
    }
    float s = 0;
    for (int i = 0; i < N_ACC; ++i) s += a[i] + __uint_as_float((unsigned)p[i]) + __uint_as_float((unsigned)(p[i] >> 32));
    out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
int main() {
    float* out; cudaMalloc(&out, 148 * 8 * 1024 * 4);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    const int iters = 4096;
    for (int mode = 0; mode < 4; ++mode)
        for (int thr : {256, 512, 1024}) {
            auto f = mode == 0 ? k<0> : mode == 1 ? k<1> : mode == 2 ? k<2> : k<3>;
            f<<<sms * 2, thr>>>(out, 0.999f, 16);
            cudaEventRecord(e0);
            f<<<sms * 2, thr>>>(out, 0.999f, iters);
            cudaEventRecord(e1); cudaEventSynchronize(e1);
            float ms; cudaEventElapsedTime(&ms, e0, e1);
            double fmas = (double)sms * 2 * thr * iters * N_ACC * (mode >= 2 ? 2 : 1);
            printf("mode %d (%s) thr %4d: %.3f ms  %.2f TFLOP/s  FMA/clk/SM(@1.965GHz) %.1f\n", mode,
                   mode == 0 ? "FFMA imm" : mode == 1 ? "FFMA reg" : mode == 2 ? "FFMA2 imm" : "FFMA2 reg", thr, ms,
                   2 * fmas / ms / 1e9, fmas / (ms * 1e-3) / sms / 1.965e9);
        }
    printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
}
