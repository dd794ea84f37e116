// TMA variants: argv = notile(0/1) boxx boxy c0 c1 c2 desc(0 param,1 global)
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
typedef CUresult (*enc_t)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
struct P { CUtensorMap tm; };
__device__ unsigned su(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__global__ void k(const __grid_constant__ P p, const CUtensorMap* gtm, float* out, int nb, int c0, int c1, int c2, int notile, int desc) {
    extern __shared__ __align__(1024) float s[];
    uint64_t* bar = reinterpret_cast<uint64_t*>(s + 8192);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su(bar)));
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        const void* tm = desc == 0 ? (const void*)&p.tm : (const void*)gtm;
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(bar)), "r"(nb) : "memory");
        if (notile)
            asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                         ::"r"(su(s)), "l"(tm), "r"(c0), "r"(c1), "r"(c2), "r"(su(bar)) : "memory");
        else
            asm volatile("cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];"
                         ::"r"(su(s)), "l"(tm), "r"(c0), "r"(c1), "r"(c2), "r"(su(bar)) : "memory");
    }
    asm volatile("{\n.reg .pred P;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W;\n}" ::"r"(su(bar)) : "memory");
    for (int i = threadIdx.x; i < nb / 4; i += blockDim.x) out[i] = s[i];
}
int main(int argc, char** argv) {
    const int notile = atoi(argv[1]), bx = atoi(argv[2]), by = atoi(argv[3]);
    const int c0 = atoi(argv[4]), c1 = atoi(argv[5]), c2 = atoi(argv[6]), desc = atoi(argv[7]);
    const int S1 = 20, S2 = 22, S3 = 40;
    std::vector<float> h(S1 * S2 * S3);
    for (size_t i = 0; i < h.size(); ++i) h[i] = (float)i;
    float *d, *o; CUtensorMap* g;
    cudaMalloc(&d, h.size() * 4); cudaMalloc(&o, 65536); cudaMalloc(&g, 128);
    cudaMemcpy(d, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
    void* f = nullptr; cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
    enc_t enc = (enc_t)f;
    P p{};
    cuuint64_t gd[3] = {S3, S2, S1}, gs[2] = {S3 * 4, S2 * S3 * 4};
    cuuint32_t box[3] = {(cuuint32_t)bx, (cuuint32_t)by, 1}, es[3] = {1, 1, 1};
    CUresult r = enc(&p.tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, d, gd, gs, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    cudaMemcpy(g, &p.tm, 128, cudaMemcpyHostToDevice);
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 8192 * 4 + 64);
    const int nb = bx * by * 4;
    k<<<1, 64, 8192 * 4 + 64>>>(p, g, o, nb, c0, c1, c2, notile, desc);
    cudaError_t e = cudaDeviceSynchronize();
    std::vector<float> ho(nb / 4);
    cudaMemcpy(ho.data(), o, nb, cudaMemcpyDeviceToHost);
    const int i1 = bx + 1;   // (line 1, col 1)
    const float exp1 = (float)((c2 * S2 + c1 + 1) * S3 + c0 + 1);
    printf("notile=%d box=%dx%d c=(%d,%d,%d) desc=%d enc=%d: %s  s[0]=%g s[bx+1]=%g (expect %g)\n", notile, bx, by, c0, c1,
           c2, desc, (int)r, cudaGetErrorString(e), ho[0], ho[i1], exp1);
    return e != cudaSuccess;
}
