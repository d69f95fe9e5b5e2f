// Standalone check of a u8 4-D TMA tile load (box W x 3 x 3 x 1) -- variants via argv:
//   tma_u8_test <boxw> <x0> <y0> <planes>
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <cstdlib>
typedef CUresult (*PFN)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *, const cuuint64_t *,
                        const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
__global__ void k(const __grid_constant__ CUtensorMap m, int x0, int y0, uint32_t bytes, uint8_t *out) {
    __shared__ __align__(128) uint8_t buf[4096];
    __shared__ __align__(8) uint64_t bar;
    uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar), d = (uint32_t)__cvta_generic_to_shared(buf);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(b));
        asm volatile("fence.mbarrier_init.release.cluster;");
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes));
        asm volatile("cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];"
                     ::"r"(d), "l"(&m), "r"(x0), "r"(0), "r"(y0), "r"(0), "r"(b) : "memory");
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p;}" : "=r"(ok) : "r"(b));
        for (uint32_t i = 0; i < bytes; i++) out[i] = buf[i];
    }
}
int main(int argc, char **argv) {
    int boxw = atoi(argv[1]), x0 = atoi(argv[2]), y0 = atoi(argv[3]), planes = atoi(argv[4]);
    int wp = 32, H = 16, nb = 16;
    uint8_t *g; cudaMalloc(&g, (size_t)wp * 3 * H * nb);
    cudaMemset(g, 7, (size_t)wp * 3 * H * nb);
    void *p; cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
    CUtensorMap m;
    cuuint64_t dims[4] = {(cuuint64_t)wp, 3, (cuuint64_t)H, (cuuint64_t)nb};
    cuuint64_t strides[3] = {(cuuint64_t)wp, (cuuint64_t)wp * 3, (cuuint64_t)wp * 3 * H};
    cuuint32_t box[4] = {(cuuint32_t)boxw, (cuuint32_t)planes, 3, 1};
    cuuint32_t es[4] = {1, 1, 1, 1};
    CUresult r = ((PFN)p)(&m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, g, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                          CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    uint8_t *out; cudaMallocManaged(&out, 4096);
    k<<<1, 32>>>(m, x0, y0, (uint32_t)boxw * planes * 3, out);
    cudaError_t e = cudaDeviceSynchronize();
    printf("boxw %d x0 %d y0 %d planes %d: encode %d  kernel %s  out[0..3] %d %d %d %d\n", boxw, x0, y0, planes, (int)r,
           cudaGetErrorString(e), out[0], out[1], out[2], out[3]);
    return 0;
}
