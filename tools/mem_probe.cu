// mem_probe.cu -- does the reconstruction kernel's store pattern make the L2
// read DRAM?  Writes S frames of 3 x 2160 x 3840 bytes with the recon CTA shape
// (32 x 4 threads, 6 rows per thread, 24 B per thread-row) in two ways:
//   mode 0: each thread stores its 24 B per row as 3 x 8-B stores (k_recon_step);
//   mode 1: each warp stores its 768-B row segment as contiguous 16-B chunks.
// Run under ncu with dram__bytes_read.sum / dram__bytes_write.sum.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/bin/mem_probe tools/mem_probe.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int H = 2160, W = 3840, RPT = 6, TX = 32, TY = 4;

__global__ void k_store(uint8_t *base, size_t frame, int mode) {
    uint8_t *out = base + (size_t)blockIdx.z * frame;
    const int x0 = blockIdx.x * TX * 24, y0 = (blockIdx.y * TY + threadIdx.y) * RPT;
    for (int c = 0; c < 3; c++)
        for (int r = 0; r < RPT; r++) {
            uint8_t *row = out + (size_t)c * H * W + (size_t)(y0 + r) * W + x0;
            const uint32_t v = (uint32_t)(r * 131 + c * 7 + threadIdx.x);
            if (mode == 0) {
                uint8_t *p = row + 24 * threadIdx.x;
#pragma unroll
                for (int q = 0; q < 3; q++) *reinterpret_cast<uint2 *>(p + 8 * q) = make_uint2(v, v + q);
            } else {
                for (int i = threadIdx.x; i < 48; i += 32)
                    *reinterpret_cast<uint4 *>(row + 16 * i) = make_uint4(v, v, v, v);
            }
        }
}

// Read side: each thread stages its reference window rows (RPT + 1 rows of
// 4 aligned 8-B words at x = 24 t + dx) like k_recon_step (mode 0), or only
// RPT rows (mode 1), or each warp loads its band of the row as contiguous
// 16-B chunks (mode 2).
__global__ void k_read(const uint8_t *base, size_t frame, int mode, int dx, int dy) {
    __shared__ uint2 sm[TY * TX * (RPT + 1) * 4];
    const uint8_t *ref = base + (size_t)blockIdx.z * frame;
    const int tid = threadIdx.y * TX + threadIdx.x;
    const int x0 = blockIdx.x * TX * 24, y0 = (blockIdx.y * TY + threadIdx.y) * RPT;
    for (int c = 0; c < 3; c++) {
        const int rows = mode == 1 ? RPT : RPT + 1;
        for (int r = 0; r < rows; r++) {
            const int yy = min(max(y0 + r + dy, 0), H - 1);
            const uint8_t *row = ref + (size_t)c * H * W + (size_t)yy * W;
            if (mode <= 1) {
                const int xb = min(max((x0 + 24 * (int)threadIdx.x + dx) & ~7, 0), W - 32);
#pragma unroll
                for (int i = 0; i < 4; i++) {
                    const uint32_t d = (uint32_t)__cvta_generic_to_shared(&sm[(r * 4 + i) * TY * TX + tid]);
                    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(d), "l"(row + xb + 8 * i) : "memory");
                }
            } else {
                const int xb = min(max((x0 + dx) & ~15, 0), W - 784);
                for (int i = threadIdx.x; i < 49; i += 32) {
                    const uint32_t d = (uint32_t)__cvta_generic_to_shared(&sm[(r * 4 * TY * TX + threadIdx.y * 98 + 2 * i) % (TY * TX * (RPT + 1) * 4)]);
                    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(row + xb + 16 * i) : "memory");
                }
            }
            asm volatile("cp.async.commit_group;" ::: "memory");
        }
        asm volatile("cp.async.wait_all;" ::: "memory");
    }
}

int main(int argc, char **argv) {
    const int S = 64;
    const size_t frame = (size_t)3 * H * W;
    uint8_t *buf = nullptr;
    if (cudaMalloc(&buf, frame * S) != cudaSuccess) return 1;
    dim3 g(W / (TX * 24), H / (TY * RPT), S), b(TX, TY);
    for (int mode = 0; mode < 2; mode++)
        for (int it = 0; it < 3; it++) k_store<<<g, b>>>(buf, frame, mode);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    for (int mode = 0; mode < 2; mode++) {
        cudaEventRecord(e0);
        for (int it = 0; it < 10; it++) k_store<<<g, b>>>(buf, frame, mode);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        printf("mode %d: %.3f ms per launch, %.0f GB/s written\n", mode, ms / 10, frame * S / (ms / 10 * 1e6));
    }
    for (int mode = 0; mode < 3; mode++) {
        for (int it = 0; it < 2; it++) k_read<<<g, b>>>(buf, frame, mode, 5, 2);
        cudaEventRecord(e0);
        for (int it = 0; it < 10; it++) k_read<<<g, b>>>(buf, frame, mode, 5, 2);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        printf("read mode %d: %.3f ms per launch, %.0f GB/s (frame bytes)\n", mode, ms / 10, frame * S / (ms / 10 * 1e6));
    }
    cudaFree(buf);
    return 0;
}
