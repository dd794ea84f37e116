// Minimal TMA check: 3D box load with the descriptor in param space (grid constant) or global memory.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cstdlib>
typedef CUresult (*enc_t)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
struct P { const float* x; int pad; CUtensorMap tm[2]; int mode; };
__device__ unsigned su(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__global__ void k(const __grid_constant__ P p, const CUtensorMap* gtm, float* out, int variant) {
    extern __shared__ __align__(128) float s[];
    __shared__ __align__(8) uint64_t bar;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        const void* tm = variant == 0 ? (const void*)&p.tm[p.mode] : (const void*)gtm;
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(&bar)), "r"(36 * 5 * 4) : "memory");
        if (variant == 2)
            asm volatile("cp.async.bulk.tensor.3d.shared::cta.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                         ::"r"(su(s)), "l"(tm), "r"(-3), "r"(-1), "r"(2), "r"(su(&bar)) : "memory");
        else
            asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                         ::"r"(su(s)), "l"(tm), "r"(-3), "r"(-1), "r"(2), "r"(su(&bar)) : "memory");
    }
    asm volatile("{\n.reg .pred P;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W;\n}" ::"r"(su(&bar)) : "memory");
    for (int i = threadIdx.x; i < 36 * 5; i += blockDim.x) out[i] = s[i];
}
int main(int argc, char** argv) {
    const int only = argc > 1 ? atoi(argv[1]) : -1;
    const int S1 = 20, S2 = 22, S3 = 40;
    std::vector<float> h(S1 * S2 * S3);
    for (size_t i = 0; i < h.size(); ++i) h[i] = (float)i;
    float *d, *o; CUtensorMap* g;
    cudaMalloc(&d, h.size() * 4); cudaMalloc(&o, 36 * 5 * 4); cudaMalloc(&g, 128);
    cudaMemcpy(d, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    void* f = nullptr; cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
    enc_t enc = (enc_t)f;
    P p{}; p.x = d; p.mode = 0;
    cuuint64_t gd[3] = {S3, S2, S1}, gs[2] = {S3 * 4, S2 * S3 * 4};
    cuuint32_t box[3] = {36, 5, 1}, es[3] = {1, 1, 1};
    CUresult r = enc(&p.tm[0], CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, d, gd, gs, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    printf("encode %d q %d sizeof(P) %zu off %zu\n", (int)r, (int)q, sizeof(P), (size_t)((char*)&p.tm[0] - (char*)&p));
    cudaMemcpy(g, &p.tm[0], 128, cudaMemcpyHostToDevice);
    for (int v = 2; v >= 0; --v) {
        if (only >= 0 && v != only) continue;
        cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 4096);
        k<<<1, 64, 4096>>>(p, g, o, v);
        cudaError_t e = cudaDeviceSynchronize();
        std::vector<float> ho(36 * 5);
        cudaMemcpy(ho.data(), o, ho.size() * 4, cudaMemcpyDeviceToHost);
        printf("variant %d: %s  s[0..5]=%g %g %g %g %g %g  s[36+3]=%g (expect %g)\n", v, cudaGetErrorString(e), ho[0], ho[1], ho[2],
               ho[3], ho[4], ho[5], ho[39], (float)(2 * S2 * S3 + 0 * S3 + 0));
        if (e != cudaSuccess) return 1;
    }
    return 0;
}
