// ubench.cu -- microbenchmarks that decide the SR conv design:
//   1. tcgen05.mma kind::f16 SS throughput (A, B in SMEM) for M=128 and
//      N in {16, 32, 64, 96, 144, 256}: cycles per MMA (K = 16).
//   2. tcgen05.mma with A in TMEM (".kind::f16 [d], [a], b") for N = 32.
//   3. tcgen05.ld 32x32b.x32 throughput: bytes per cycle per SM.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ubench tools/ubench.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "../paper_conf_sigcomm_yeolkjyh22_b200/csrc/ptx.cuh"

using namespace ns;

__device__ __forceinline__ void umma_ts(uint32_t d, uint32_t a_tmem, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d),
        "r"(a_tmem), "l"(bdesc), "r"(idesc), "r"(acc)
        : "memory");
}

template <int N, bool TS, int NACC = 1>
__global__ void k_mma(int iters, long long *cycles) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tm;
    const int warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(smem)[i] = 0x3f803f80u;
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
    fence_proxy_async_smem();
    if (warp == 0) tmem_alloc(&tm, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t t = tm;
    if (threadIdx.x == 0) {
        const uint32_t idesc = idesc_bf16_f32(128, N);
        const uint32_t a = smem_u32(smem), b = smem_u32(smem + 32768);
        long long c0 = clock64();
        for (int i = 0; i < iters; i++) {
            const uint64_t bd = smem_desc(b + (i & 3) * 256, N * 16, 128);
            const uint32_t dcol = t + 256 - (N <= 64 ? 0 : 0) + (uint32_t)((i % NACC) * (N <= 64 ? 64 : 0));
            if (TS) {
                umma_ts(dcol, t, bd, idesc, i >= NACC);
            } else {
                const uint64_t ad = smem_desc(a + (i & 7) * 16, 130 * 16, 128);
                umma_bf16(dcol, ad, bd, idesc, i >= NACC);
            }
        }
        umma_commit(&bar);
        mbar_wait(&bar, 0);
        long long c1 = clock64();
        cycles[blockIdx.x] = c1 - c0;
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tmem_dealloc(t, 512);
}

__global__ void k_tld(int iters, long long *cycles, uint32_t *sink) {
    __shared__ uint32_t tm;
    const int warp = threadIdx.x >> 5;
    if (warp == 0) tmem_alloc(&tm, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t t = tm + ((uint32_t)((warp & 3) * 32) << 16);
    uint32_t acc = 0;
    long long c0 = clock64();
    for (int i = 0; i < iters; i++) {
        uint32_t r[32];
        tmem_ld32(t + (i & 7) * 32, r);
        tmem_wait_ld();
#pragma unroll
        for (int k = 0; k < 32; k++) acc += r[k];
    }
    long long c1 = clock64();
    __syncthreads();
    if (threadIdx.x == 0) cycles[blockIdx.x] = c1 - c0;
    sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tmem_dealloc(tm, 512);
}

template <int N, bool TS, int NACC = 1>
void run_mma(long long *d) {
    const int iters = 4096;
    cudaFuncSetAttribute(k_mma<N, TS, NACC>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
    k_mma<N, TS, NACC><<<148, 128, 64 * 1024>>>(iters, d);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < 148; i++) avg += h[i];
    avg /= 148;
    const double cyc = avg / iters;
    const double ideal = 128.0 * N / 256.0;
    printf("acc%d mma %s M=128 N=%3d K=16: %6.1f cycles/MMA (floor %5.1f) -> %5.1f%% of tensor peak, smem %5.1f B/clk  [%s]\n",
           NACC, TS ? "TS" : "SS", N, cyc, ideal, 100.0 * ideal / cyc, (TS ? N * 32.0 : (128 * 32.0 + N * 32.0)) / cyc,
           cudaGetErrorString(e));
}

// tcgen05.cp smem -> tmem, 128x256b shape (128 lanes x 256 bits = 4 KB per op)
__global__ void k_cp(int iters, long long *cycles) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tm;
    const int warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
    if (warp == 0) tmem_alloc(&tm, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t t = tm;
    if (threadIdx.x == 0) {
        const uint32_t a = smem_u32(smem);
        long long c0 = clock64();
        for (int i = 0; i < iters; i++) {
            const uint64_t ad = smem_desc(a + (i & 7) * 1024, 16, 128);
            asm volatile("tcgen05.cp.cta_group::1.128x256b [%0], %1;" ::"r"(t + (uint32_t)((i & 7) * 8)), "l"(ad) : "memory");
        }
        umma_commit(&bar);
        mbar_wait(&bar, 0);
        cycles[blockIdx.x] = clock64() - c0;
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tmem_dealloc(t, 512);
}

int main() {
    long long *d;
    uint32_t *sink;
    cudaMalloc(&d, 148 * sizeof(long long));
    cudaMalloc(&sink, 148 * 512 * 4);
    run_mma<16, false>(d);
    run_mma<32, false>(d);
    run_mma<64, false>(d);
    run_mma<96, false>(d);
    run_mma<144, false>(d);
    run_mma<256, false>(d);
    run_mma<32, true>(d);
    run_mma<96, true>(d);
    run_mma<16, false, 4>(d);
    run_mma<32, false, 2>(d);
    run_mma<32, false, 4>(d);
    run_mma<64, false, 4>(d);
    run_mma<32, true, 4>(d);
    {
        const int iters = 4096;
        cudaFuncSetAttribute(k_cp, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
        k_cp<<<148, 128, 64 * 1024>>>(iters, d);
        cudaError_t e = cudaDeviceSynchronize();
        long long h[148];
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < 148; i++) avg += h[i];
        avg /= 148;
        printf("tcgen05.cp 128x256b: %6.1f cycles/op -> %6.1f B/clk  [%s]\n", avg / iters, 4096.0 * iters / avg,
               cudaGetErrorString(e));
    }
    for (int warps : {4, 8, 16}) {
        const int iters = 2048;
        k_tld<<<148, warps * 32>>>(iters, d, sink);
        cudaError_t e = cudaDeviceSynchronize();
        long long h[148];
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < 148; i++) avg += h[i];
        avg /= 148;
        const double bytes = (double)iters * warps * 32 * 32 * 4;
        printf("tcgen05.ld 32x32b.x32 (+wait) %2d warps: %7.1f B/clk/SM  [%s]\n", warps, bytes / avg,
               cudaGetErrorString(e));
    }
    return 0;
}
