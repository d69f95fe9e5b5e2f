// ubench.cu -- microbenchmarks that decide the SR conv design:
//   1. tcgen05.mma kind::f16 SS throughput (A, B in SMEM) for M=128 and
//      N in {16, 32, 64, 96, 144, 256}: cycles per MMA (K = 16).
//   2. tcgen05.mma with A in TMEM (".kind::f16 [d], [a], b") for N = 32.
//   3. tcgen05.ld 32x32b.x32 throughput: bytes per cycle per SM.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ubench tools/ubench.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>
#include "../paper_conf_sigcomm_yeolkjyh22_b200/csrc/ptx.cuh"

using namespace ns;
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

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

// The res-block conv1 group exactly: 3 dx x 2 kc MMAs, M=128 N=96 K=16, A = h slot
// (LBO kHalo*16, dx shift 16 B), B = rot strip (LBO 5*32*16), window start
// rotating with the step, commit per group; RANDOM=1 fills SMEM with random
// bf16 (data-dependent power), 0 with 1.0.
template <bool RANDOM, bool WAIT, int DMODE = 0, int BMODE = 0, int AMODE = 0>
__global__ void k_rot(int groups, long long *cycles) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t bar;
    __shared__ uint32_t tm;
    const int warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 96 * 1024 / 4; i += blockDim.x) {
        uint32_t h = (uint32_t)i * 2654435761u + 12345u;
        h ^= h >> 13; h *= 0x5bd1e995u; h ^= h >> 15;
        // random bf16 in about [-2, 2]: sign, exponent 126..128, random mantissa
        const uint32_t lo = ((h & 0x8000u) | ((126u + (h >> 16) % 3u) << 7) | (h & 0x7Fu));
        const uint32_t hi = (((h >> 8) & 0x8000u) | ((126u + (h >> 20) % 3u) << 7) | ((h >> 9) & 0x7Fu));
        reinterpret_cast<uint32_t *>(smem)[i] = RANDOM ? (lo | (hi << 16)) : 0x3f803f80u;
    }
    __shared__ uint64_t bars[2];
    if (threadIdx.x == 0) { mbar_init(&bar, 1); mbar_init(&bars[0], 1); mbar_init(&bars[1], 1); fence_mbar_init(); }
    fence_proxy_async_smem();
    if (warp == 0) tmem_alloc(&tm, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t t = tm;
    if (threadIdx.x == 0) {
        constexpr int NB = 32, KC = 2;
        const uint32_t idesc = idesc_bf16_f32(128, 3 * NB);
        const uint32_t a = smem_u32(smem), b = smem_u32(smem + 32768);
        long long c0 = clock64();
        for (int g = 0; g < groups; g++) {
            // AMODE 0: 2 A slots; 1: 5 slots of 9216 B (the h ring)
            const uint32_t aoff = AMODE == 0 ? (g & 1) * 8448 : (uint32_t)(g % 3) * 9216;
            // BMODE 0: one strip; 1: alternate two strips (conv1 / conv2 weights) 15 KB apart
            const uint32_t boff = BMODE == 0 ? 0 : (g & 1) * 15360;
            // DMODE 0: D at 0 / 192; 1: cycle 0, 192, 96, 288 (conv1 A, conv1 B, conv2 A, conv2 B)
            const uint32_t dcol = DMODE != 1 ? (g & 1) * 192 : (uint32_t)((g & 1) * 192 + ((g >> 1) & 1) * 96);
            const uint64_t ad0 = smem_desc(a + aoff, 130 * 16, 128);
            const uint64_t bd0 = smem_desc(b + boff + (uint32_t)(g % 3) * NB * 16, 5 * NB * 16, 128);
            for (int dx = 0; dx < 3; dx++)
                for (int kc = 0; kc < KC; kc++)
                    umma_bf16(t + dcol, ad0 + (uint64_t)((2 * kc * 130 * 16 + dx * 16) >> 4),
                              bd0 + (uint64_t)(((dx * KC + kc) * 2 * 5 * NB * 16) >> 4), idesc, 1u);
            if (WAIT || DMODE == 2) umma_commit(&bars[g & 1]);  // DMODE 2: commit per group, no wait
            if (WAIT) mbar_wait(&bars[g & 1], (g >> 1) & 1);
        }
        if (!WAIT) { umma_commit(&bar); mbar_wait(&bar, 0); }
        cycles[blockIdx.x] = clock64() - c0;
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tmem_dealloc(t, 512);
}

template <bool RANDOM, bool WAIT, int DMODE = 0, int BMODE = 0, int AMODE = 0>
void run_rot(long long *d) {
    const int groups = 1024;
    cudaFuncSetAttribute(k_rot<RANDOM, WAIT, DMODE, BMODE, AMODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, 96 * 1024);
    k_rot<RANDOM, WAIT, DMODE, BMODE, AMODE><<<148, 128, 96 * 1024>>>(groups, d);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < 148; i++) avg += h[i];
    avg /= 148;
    printf("res-block group (6 MMA M128 N96 K16, rot strip) data=%s %s dmode %d bmode %d amode %d: %6.1f cycles/MMA  [%s]\n",
           RANDOM ? "random" : "1.0", WAIT ? "wait-per-group" : "streamed", DMODE, BMODE, AMODE, avg / groups / 6,
           cudaGetErrorString(e));
}

// MMA stream (res-block group pattern) while the other warps of the CTA spin on
// an mbarrier that completes only at the end.  POLL 0: plain try_wait, 1:
// try_wait with suspend hint, 2: lane 0 polls (hint) then __syncwarp.
template <int POLL>
__global__ void k_rot_poll(int groups, long long *cycles) {
    extern __shared__ __align__(1024) uint8_t smem[];
    __shared__ uint64_t bar, done;
    __shared__ uint32_t tm;
    const int warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 96 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(smem)[i] = 0x3f813f7fu ^ (i * 2654435761u & 0x00ff00ffu);
    if (threadIdx.x == 0) { mbar_init(&bar, 1); mbar_init(&done, 1); fence_mbar_init(); }
    fence_proxy_async_smem();
    if (warp == 0) tmem_alloc(&tm, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t t = tm;
    if (warp == 0) {
        if (threadIdx.x == 0) {
            constexpr int NB = 32, KC = 2;
            const uint32_t idesc = idesc_bf16_f32(128, 3 * NB);
            const uint32_t a = smem_u32(smem), b = smem_u32(smem + 32768);
            long long c0 = clock64();
            for (int g = 0; g < groups; g++) {
                const uint64_t ad0 = smem_desc(a + (uint32_t)(g % 3) * 9216, 130 * 16, 128);
                const uint64_t bd0 = smem_desc(b + (g & 1) * 15360 + (uint32_t)(g % 3) * NB * 16, 5 * NB * 16, 128);
                for (int dx = 0; dx < 3; dx++)
                    for (int kc = 0; kc < KC; kc++)
                        umma_bf16(t + (g & 1) * 192, ad0 + (uint64_t)((2 * kc * 130 * 16 + dx * 16) >> 4),
                                  bd0 + (uint64_t)(((dx * KC + kc) * 2 * 5 * NB * 16) >> 4), idesc, 1u);
            }
            umma_commit(&bar);
            mbar_wait(&bar, 0);
            cycles[blockIdx.x] = clock64() - c0;
            mbar_arrive(&done);
        }
    } else {
        if (POLL == 0) { while (!mbar_try_wait(&done, 0)) {} }
        else if (POLL == 1) { while (!mbar_try_wait_sleep(&done, 0)) {} }
        else { if ((threadIdx.x & 31) == 0) { while (!mbar_try_wait_sleep(&done, 0)) {} } __syncwarp(); }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tmem_dealloc(t, 512);
}
template <int POLL>
void run_rot_poll(long long *d, int threads) {
    const int groups = 1024;
    cudaFuncSetAttribute(k_rot_poll<POLL>, cudaFuncAttributeMaxDynamicSharedMemorySize, 96 * 1024);
    k_rot_poll<POLL><<<148, threads, 96 * 1024>>>(groups, d);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < 148; i++) avg += h[i];
    avg /= 148;
    printf("MMA stream + %2d polling warps, poll mode %d: %6.1f cycles/MMA  [%s]\n", threads / 32 - 1, POLL,
           avg / groups / 6, cudaGetErrorString(e));
}

// mbarrier ping-pong between warp 0 and warp 1: round-trip cycles.  HINT 0:
// plain try_wait loop, 1: try_wait with the suspend-time hint.
template <int HINT>
__global__ void k_pingpong(int iters, long long *cycles) {
    __shared__ uint64_t b0, b1;
    const int warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) { mbar_init(&b0, 32); mbar_init(&b1, 32); fence_mbar_init(); }
    __syncthreads();
    auto wait = [&](uint64_t *b, uint32_t par) {
        if (HINT) { while (!mbar_try_wait_sleep(b, par)) {} }
        else { while (!mbar_try_wait(b, par)) {} }
    };
    long long c0 = clock64();
    for (int i = 0; i < iters; i++) {
        if (warp == 0) { mbar_arrive(&b0); wait(&b1, i & 1); }
        else if (warp == 1) { wait(&b0, i & 1); mbar_arrive(&b1); }
    }
    if (threadIdx.x == 0) cycles[blockIdx.x] = clock64() - c0;
}
template <int HINT>
void run_pingpong(long long *d) {
    const int iters = 4096;
    k_pingpong<HINT><<<148, 64>>>(iters, d);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < 148; i++) avg += h[i];
    avg /= 148;
    printf("mbarrier ping-pong round trip, %s: %6.1f cycles  [%s]\n", HINT ? "try_wait + suspend hint" : "plain try_wait",
           avg / iters, cudaGetErrorString(e));
}

int main() {
    long long *d;
    uint32_t *sink;
    cudaMalloc(&d, 148 * sizeof(long long));
    cudaMalloc(&sink, 148 * 512 * 4);
    run_rot<false, false>(d);
    run_rot<true, false>(d);
    run_rot<true, true>(d);
    run_rot<true, false, 1, 0, 0>(d);
    run_rot<true, false, 0, 1, 0>(d);
    run_rot<true, false, 0, 0, 1>(d);
    run_rot<true, false, 1, 1, 1>(d);
    run_rot<true, false, 2, 0, 0>(d);
    run_pingpong<0>(d);
    run_pingpong<1>(d);
    for (int th : {32, 128, 576}) { run_rot_poll<0>(d, th); run_rot_poll<1>(d, th); run_rot_poll<2>(d, th); }
    if (getenv("ROT_ONLY")) return 0;
    run_mma<16, false>(d);
    run_mma<32, false>(d);
    run_mma<64, false>(d);
    run_mma<96, false>(d);
    run_mma<144, false>(d);
    run_mma<256, false>(d);
    run_mma<32, true>(d);
    run_mma<96, true>(d);
    run_mma<128, false>(d);
    run_mma<128, true>(d);
    run_mma<192, true>(d);
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
