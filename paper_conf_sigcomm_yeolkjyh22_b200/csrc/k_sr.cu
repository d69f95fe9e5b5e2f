// k_sr.cu -- anchor SR DNN (NAS "high" EDSR-style net, 8
// residual blocks, 32 channels, x3) as implicit-GEMM 3x3 convolutions on the
// 5th-generation tensor cores (tcgen05.mma, accumulators in TMEM), fed by TMA.
//
// Formulation: one UMMA M tile = 128 consecutive
// output pixels of one row; N = output channels; K = 9 taps x Cin.  Input rows
// live in shared memory as K-major "interleaved" core matrices
// [Cin/8][130 px][8 ch] bf16 (exactly the TMA box of the activation layout
// [job][H][C/8][W][8]); the 3x3 taps are pure descriptor offsets: tap (dy, dx)
// reads ring slot (row y+dy-1) at start + dx*16 B, because consecutive pixels
// are 16 B apart inside a channel group (SBO = 128 B per 8 rows).  No im2col,
// zero padding comes from TMA out-of-bounds fill.  A CTA walks a strip of rows
// with a 6-slot TMA ring, double-buffered TMEM accumulators, and a fused
// epilogue (bias, ReLU, residual add, pixel shuffle, or the HR tail with the
// integer bilinear skip, round and clamp to u8).
#include <cuda_bf16.h>
#include <cstdio>
#include "ns_internal.h"
#include "ptx.cuh"

namespace ns {

#ifdef NS_TRACE
// debug-only timeline of CTA (0,0,0): per-role regions of {clock64, tag << 32 | step},
// plain stores (no atomics on the traced threads' critical path)
__device__ unsigned long long g_trace[16 * 2 * 1024];
#define NS_TR(tag, q)                                                                            \
    do {                                                                                         \
        if (blockIdx.x == 0 && blockIdx.y == 0 && blockIdx.z == 0 && _trn < 1024) {              \
            g_trace[2 * (_trr * 1024 + _trn)] = clock64();                                       \
            g_trace[2 * (_trr * 1024 + _trn) + 1] = ((unsigned long long)(tag) << 32) | (unsigned)(q); \
            _trn++;                                                                              \
        }                                                                                        \
    } while (0)
#define NS_TR_ROLE(r) int _trr = (r), _trn = 0
#else
#define NS_TR(tag, q) \
    do {              \
    } while (0)
#define NS_TR_ROLE(r)
#endif

// EPI_HEAD: the store epilogue of the head conv, whose input x = LR - 128 has 3
// real channels: only channel group 0 (8 channels, 16 B/px) is stored and
// loaded by TMA; group 1 of every ring slot is a zero region written once.
enum { EPI_STORE = 0, EPI_RELU = 1, EPI_RESID = 2, EPI_HEAD = 5 };

struct ConvArgs {
    int H, W;               // conv spatial dims (input == output)
    int n_xtiles, rows_per_cta;
    int j0;                 // first job of the batch
    const SrJob *jobs;
    const int32_t *job_count;
    size_t b_off, bias_off; // this launch's B operand / bias offsets in the packed model
    const uint16_t *in;     // bf16 activation in [job][H][CIN/8][W][8] (k_conv_rot, k_uptail2: bulk-copied rows)
    uint16_t *out;          // bf16 activation out (EPI_STORE/RELU/RESID)
    const uint16_t *resid;  // EPI_RESID
    int C;                  // channels of the output activation (shuffle: per sub-pixel)
    int s;                  // scale (shuffle / tail)
    int sub0;               // shuffle: first sub-pixel of this launch
    int lr_h, lr_w;         // tail: LR dims of the bilinear skip
    float *ring;            // uptail: fp32 t of the HR frame-border ring [job][nring][3]
    uint8_t *lr8;           // u8 copy of the net's input planes [job][H][3][wp] (k_prep_lr), k_uptail's skip taps
    int wp;
    uint8_t *hr_tmp;        // NS_FMT_I420 batches: the HR output goes here ([slot][3][H][W]) and is packed
    size_t hr_tmp_frame;    // to 4:2:0 into jobs[].hr afterwards (k_pack420); NULL: straight to jobs[].hr
};

__host__ __device__ constexpr uint32_t round_up(uint32_t v, uint32_t a) { return (v + a - 1) / a * a; }
__host__ __device__ constexpr uint32_t tmem_cols_for(uint32_t c) {
    return c <= 32 ? 32 : c <= 64 ? 64 : c <= 128 ? 128 : c <= 256 ? 256 : 512;
}


__device__ __forceinline__ uint32_t pack_bf16(float a, float b) {
    __nv_bfloat162 v = __floats2bfloat162_rn(a, b);
    return *reinterpret_cast<uint32_t *>(&v);
}
__device__ __forceinline__ float bf_lo(uint32_t u) { return __uint_as_float(u << 16); }
__device__ __forceinline__ float bf_hi(uint32_t u) { return __uint_as_float(u & 0xFFFF0000u); }

// O6 tap of the fixed-point bilinear upsample (half-pixel centres, Q7).
__device__ __forceinline__ void up_tap(int X, int s, int len, int &i0, int &i1, int &w1) {
    int u = 2 * X + 1 - s;
    int x0 = (u >= 0) ? u / (2 * s) : -((-u + 2 * s - 1) / (2 * s));
    int rem = u - 2 * s * x0;
    w1 = (128 * rem + s) / (2 * s);
    i0 = min(max(x0, 0), len - 1);
    i1 = min(max(x0 + 1, 0), len - 1);
}

// ------------------------------------------------------------------ rotated-accumulator conv
// Measured on B200 (tools/ubench.cu): a K=16 tcgen05.mma with A from shared
// memory costs max(64, N/2) cycles -- the 4 KB A tile is read at ~64 B/clk --
// so a 32-channel conv (N = 32) can use at most 25% of the tensor cores.
// Here each input row is read ONCE per 3x3 tap column dx and multiplied by the
// weights of all three kernel rows at once: N = 3 x Cout.  The three partial
// products land in three TMEM accumulator blocks that belong to the three
// output rows the input row contributes to (y+1 via dy=0, y via dy=1, y-1 via
// dy=2).  Output row r lives in block r mod 3; the B operand is a 5-block
// strip [W_dy2; W_dy1; W_dy0; W_dy2; W_dy1] and the window start (1 - y mod 3)
// mod 3 rotates the kernel rows onto the right blocks.  After input row y the
// block of row y-1 is complete: the epilogue reads it, applies the fused
// epilogue, and zeroes it for row y+2.  No im2col, no lane shifts, 128-pixel
// tiles, N = 96 (C = 32) -> up to 3x the MMA efficiency of N = 32.
// (A head that builds its own input rows from the u8 LR planes in a builder
// warp -- no prep pass -- was parity green and measured neutral.)
template <int CIN, int NB>
struct RotCfg {
    static constexpr int KC = CIN / 16;
    static constexpr uint32_t B_BYTES = 30u * CIN * NB;     // 3 dx x KC x 2 kh x 5NB rows x 16 B
    static constexpr uint32_t BIAS_BYTES = NB * 4u;
    static constexpr uint32_t W_REGION = round_up(B_BYTES + BIAS_BYTES, 1024);
    static constexpr uint32_t SLOT_BYTES = kHalo * CIN * 2u;
    // 128-B slots (bulk-copy rows need 16 B): with 1-KB rounding the C = 32
    // conv (the end conv) took 59.5 KB and 3 CTAs per SM; 56.8 KB fits 4,
    // as many as its TMEM (128 columns each) allows
    static constexpr uint32_t SLOT = round_up(SLOT_BYTES, 128);
    static constexpr int NSLOT = 3;  // input ring; the barrier array is laid out [0,3) ring, 3 weights, 4 MMA
    static constexpr uint32_t TMEM_COLS = tmem_cols_for(3 * NB);
    static constexpr uint32_t SMEM = W_REGION + NSLOT * SLOT + 128;
    static_assert((3 * NB) % 16 == 0 && 3 * NB <= 256, "N = 3 NB");
    static_assert(SMEM <= 232448, "shared memory");
};

__device__ __forceinline__ int mod3(int v) { return ((v % 3) + 3) % 3; }
__host__ __device__ constexpr int fdiv_sr(int a, int b) { return a >= 0 ? a / b : -((-a + b - 1) / b); }
template <int S>
__host__ __device__ constexpr int tap_d_sr(int k) { return fdiv_sr(2 * k + 1 - S, 2 * S); }
template <int S>
__host__ __device__ constexpr int tap_w1_sr(int k) {
    return (128 * ((2 * k + 1 - S) - 2 * S * tap_d_sr<S>(k)) + S) / (2 * S);
}

template <int NB>
__device__ __forceinline__ void tmem_zero(uint32_t taddr) {
    if constexpr (NB == 32) {
        asm volatile(
            "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,"
            "%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1};" ::"r"(taddr), "r"(0u) : "memory");
    } else {
        asm volatile(
            "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1};" ::"r"(
                taddr), "r"(0u) : "memory");
    }
}
// Stores 32 / 16 per-column values (the same for every lane of the warp's quarter).
template <int NB>
__device__ __forceinline__ void tmem_st_vals(uint32_t taddr, const float (&b)[NB]) {
#define NS_F(i) "f"(b[i])
    if constexpr (NB == 32) {
        asm volatile(
            "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
            "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
            NS_F(0), NS_F(1), NS_F(2), NS_F(3), NS_F(4), NS_F(5), NS_F(6), NS_F(7), NS_F(8), NS_F(9), NS_F(10),
            NS_F(11), NS_F(12), NS_F(13), NS_F(14), NS_F(15), NS_F(16), NS_F(17), NS_F(18), NS_F(19), NS_F(20),
            NS_F(21), NS_F(22), NS_F(23), NS_F(24), NS_F(25), NS_F(26), NS_F(27), NS_F(28), NS_F(29), NS_F(30),
            NS_F(31) : "memory");
    } else {
        static_assert(NB == 16, "");
        asm volatile(
            "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::
                "r"(taddr), NS_F(0), NS_F(1), NS_F(2), NS_F(3), NS_F(4), NS_F(5), NS_F(6), NS_F(7), NS_F(8), NS_F(9),
            NS_F(10), NS_F(11), NS_F(12), NS_F(13), NS_F(14), NS_F(15) : "memory");
    }
#undef NS_F
}
// ReLU + round-to-nearest bf16 of a pair, one instruction: low half = lo.
__device__ __forceinline__ uint32_t pack_bf16_relu(float lo, float hi) {
    uint32_t r;
    asm("cvt.rn.relu.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(hi), "f"(lo));
    return r;
}
__device__ __forceinline__ void tmem_st1(uint32_t taddr, float v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "f"(v) : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
// N consecutive columns from v[0..N) in at most two stores (.x8 / .x4 / .x2 / .x1).
template <int N>
__device__ __forceinline__ void tmem_st_run(uint32_t taddr, const float *v) {
    if constexpr (N >= 8) {
        asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr), "f"(v[0]),
                     "f"(v[1]), "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7]) : "memory");
        tmem_st_run<N - 8>(taddr + 8, v + 8);
    } else if constexpr (N >= 4) {
        asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1,%2,%3,%4};" ::"r"(taddr), "f"(v[0]), "f"(v[1]),
                     "f"(v[2]), "f"(v[3]) : "memory");
        tmem_st_run<N - 4>(taddr + 4, v + 4);
    } else if constexpr (N >= 2) {
        asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1,%2};" ::"r"(taddr), "f"(v[0]), "f"(v[1]) : "memory");
        tmem_st_run<N - 2>(taddr + 2, v + 2);
    } else if constexpr (N == 1) {
        tmem_st1(taddr, v[0]);
    }
}

__device__ __forceinline__ int mod5(int v) { return ((v % 5) + 5) % 5; }

template <int NB>
__device__ __forceinline__ void tmem_ldN(uint32_t a, uint32_t (&v)[NB]) {
    if constexpr (NB == 16) {
        tmem_ld16(a, v);
    } else if constexpr (NB == 32) {
        tmem_ld32(a, v);
    } else {
        static_assert(NB == 48, "");
        uint32_t (&v0)[32] = *reinterpret_cast<uint32_t(*)[32]>(v);
        uint32_t (&v1)[16] = *reinterpret_cast<uint32_t(*)[16]>(v + 32);
        tmem_ld32(a, v0);
        tmem_ld16(a + 32, v1);
    }
}
template <int NB>
__device__ __forceinline__ void tmem_zeroN(uint32_t a) {
    if constexpr (NB == 48) {
        tmem_zero<32>(a);
        tmem_zero<16>(a + 32);
    } else {
        tmem_zero<NB>(a);
    }
}



// (k_uptail2 with bulk-copied rows measured neutral to slightly slower on the
// same box -- 20.3 vs 19.2-20.3 ms -- so it keeps its tensor box; double-
// buffered output staging rows measured neutral too.)  uptail2's retired
// accumulator columns are re-initialised by their own epilogue group with
// bias + 1/2 (no 3-group barrier per step).
// Activation rows into a ring slot by one-dimensional bulk copies.  The
// activation layout [job][H][G][W][8] (bf16) holds each channel group's row as
// one contiguous run of 16 B per pixel, so a tile row segment of ncols pixels
// starting at x_start is G contiguous runs; the slot layout is [G][ncols][8]
// (the UMMA K-major core-matrix layout, leading byte offset ncols * 16).  A
// tensor box over the same data has an innermost extent of 16 B (8 channels),
// which the TMA unit serves far more slowly (res-block A/B: body 102.4 -> 96.9
// ms per c4 step).  Columns outside the frame are zeroed once per slot
// (slot_zero_edges); a row outside the frame gets its in-frame columns zeroed
// by the producer (generic stores, proxy fence) and a plain arrive.
__device__ __forceinline__ uint32_t mbar_arrive_state(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
    return 0;
}
template <int G>
__device__ __forceinline__ void slot_zero_edges(uint8_t *slot, int ncols, int W, int x_start, int t, int nt) {
    const int lo = max(0, -x_start), hi = min(ncols, W - x_start);
    for (int i = t; i < G * ncols; i += nt) {
        const int c = i % ncols, g = i / ncols;
        if (c < lo || c >= hi) reinterpret_cast<uint4 *>(slot + g * ncols * 16)[c] = make_uint4(0, 0, 0, 0);
    }
}
template <int G>
__device__ __forceinline__ void row_bulk(uint8_t *slot, int ncols, const uint16_t *in, int job, int H, int W, int y,
                                         int x_start, uint64_t *bar) {
    const int lo = max(0, -x_start), hi = min(ncols, W - x_start);
    if (y < 0 || y >= H) {
        for (int g = 0; g < G; g++)
            for (int c = lo; c < hi; c++) reinterpret_cast<uint4 *>(slot + g * ncols * 16)[c] = make_uint4(0, 0, 0, 0);
        fence_proxy_async_smem();
        mbar_arrive_state(bar);
        return;
    }
    const uint32_t run = (uint32_t)(hi - lo) * 16u;
    mbar_arrive_expect_tx(bar, run * G);
    const uint16_t *src = in + (((size_t)job * H + y) * G * W + (size_t)(x_start + lo)) * 8;
    for (int g = 0; g < G; g++) bulk_load(slot + g * ncols * 16 + lo * 16, src + (size_t)g * W * 8, run, bar);
}

template <int CIN, int NB, int EPI>
__global__ void __launch_bounds__(128)
    k_conv_rot(const __grid_constant__ CUtensorMap tm_in, const ConvArgs a) {
    using Cfg = RotCfg<CIN, NB>;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *s_w = smem;
    const float *s_bias = reinterpret_cast<const float *>(smem + Cfg::B_BYTES);
    uint8_t *s_ring = smem + Cfg::W_REGION;
    // [0,3) ring full, 3 weights, 4 MMA done
    uint64_t *bars = reinterpret_cast<uint64_t *>(s_ring + Cfg::NSLOT * Cfg::SLOT);
    uint32_t *s_tmem = reinterpret_cast<uint32_t *>(bars + 8);

    const int slot_job = blockIdx.z;
    const int job = a.j0 + slot_job;
    if (a.job_count && job >= *a.job_count) return;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int x0 = blockIdx.x * kTile;
    const int y0 = blockIdx.y * a.rows_per_cta;
    const int y1 = min(y0 + a.rows_per_cta, a.H);
    const int n_loads = y1 - y0 + 2;  // input rows y0-1 .. y1

    if (tid == 0) {
        for (int i = 0; i < 8; i++) mbar_init(&bars[i], 1);
        fence_mbar_init();
    }
    if (warp == 0) tmem_alloc(s_tmem, Cfg::TMEM_COLS);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *s_tmem;
    const uint32_t tl = tmem + ((uint32_t)(warp * 32) << 16);  // this warp's TMEM lanes
    const SrJob J = a.jobs[job];
    // EPI_HEAD: TMA fills channel group 0 only; group 1 (at +kHalo*16, the A
    // descriptor's leading byte offset) stays zero for the whole kernel
    constexpr uint32_t LOAD_BYTES = (EPI == EPI_HEAD) ? kHalo * 16u : Cfg::SLOT_BYTES;
    static_assert(EPI != EPI_HEAD || CIN == 16, "head: 3 channels in one group of 8, padded to K = 16");
    if constexpr (EPI == EPI_HEAD) {
        for (int i = tid; i < Cfg::NSLOT * kHalo; i += blockDim.x)
            reinterpret_cast<uint4 *>(s_ring + (i / kHalo) * Cfg::SLOT + kHalo * 16)[i % kHalo] = make_uint4(0, 0, 0, 0);
        fence_proxy_async_smem();
    }
    // rows by bulk copies (row_bulk): G channel groups of 16 B per pixel
    constexpr int G = (EPI == EPI_HEAD) ? 1 : CIN / 8;
    (void)LOAD_BYTES;
    for (int sl = 0; sl < Cfg::NSLOT; sl++)
            slot_zero_edges<G>(s_ring + sl * Cfg::SLOT, kHalo, a.W, x0 - 1, tid, blockDim.x);
    fence_proxy_async_smem();
    __syncthreads();
    if (tid == 0) {
        prefetch_tmap(&tm_in);
        mbar_arrive_expect_tx(&bars[3], Cfg::B_BYTES + Cfg::BIAS_BYTES);
        bulk_load(s_w, J.wts + a.b_off, Cfg::B_BYTES, &bars[3]);
        bulk_load(smem + Cfg::B_BYTES, J.wts + a.bias_off, Cfg::BIAS_BYTES, &bars[3]);
        for (int q = 0; q < Cfg::NSLOT && q < n_loads; q++) {
            row_bulk<G>(s_ring + q * Cfg::SLOT, kHalo, a.in, slot_job, a.H, a.W, y0 - 1 + q, x0 - 1, &bars[q]);
        }
    }
    // the three accumulator blocks start at zero
    tmem_zero<NB>(tl);
    tmem_zero<NB>(tl + NB);
    tmem_zero<NB>(tl + 2 * NB);
    tmem_wait_st();
    mbar_wait(&bars[3], 0);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();

    const uint32_t idesc = idesc_bf16_f32(128, 3 * NB);
    const int p = warp * 32 + lane;
    const int x = x0 + p;
    constexpr int RC = (EPI == EPI_RESID) ? NB / 8 : 1;
    uint4 rnext[RC];  // EPI_RESID: residual row prefetched one step ahead
#pragma unroll
    for (int cg = 0; cg < RC; cg++) rnext[cg] = make_uint4(0, 0, 0, 0);
    for (int q = 0; q < n_loads; q++) {
        const int yin = y0 - 1 + q;
        if (tid == 0) {
            const int sl = q % Cfg::NSLOT;
            mbar_wait(&bars[sl], (q / Cfg::NSLOT) & 1);
            tc_fence_after();
            const uint32_t abase = smem_u32(s_ring + sl * Cfg::SLOT);
            const uint32_t start = (uint32_t)mod3(1 - yin);  // rotation of the kernel rows
            const uint32_t wbase = smem_u32(s_w) + start * NB * 16;
#pragma unroll
            for (int dx = 0; dx < 3; dx++) {
#pragma unroll
                for (int kc = 0; kc < Cfg::KC; kc++) {
                    const uint64_t ad = smem_desc(abase + (uint32_t)(2 * kc * kHalo * 16 + dx * 16), kHalo * 16, 128);
                    const uint64_t bd =
                        smem_desc(wbase + (uint32_t)((dx * Cfg::KC + kc) * 2 * 5 * NB * 16), 5 * NB * 16, 128);
                    umma_bf16(tmem, ad, bd, idesc, 1u);
                }
            }
            umma_commit(&bars[4]);
        }
        __syncwarp();
        const int r = yin - 1;  // output row completed by this input row
        const bool valid = r >= y0 && x < a.W;
        uint4 rres[RC];
        if constexpr (EPI == EPI_RESID) {
            // the residual of this row was fetched one step ago; fetch the next
            // row's now, so its latency is covered by a whole step (ncu: the
            // same-step load left the end conv 60% long-scoreboard stalls)
#pragma unroll
            for (int cg = 0; cg < RC; cg++) rres[cg] = rnext[cg];
            const int rn = yin;
            if (rn >= y0 && rn < y1 && x < a.W) {
                const size_t rb = ((size_t)slot_job * a.H + rn) * (NB / 8);
#pragma unroll
                for (int cg = 0; cg < RC; cg++)
                    rnext[cg] = __ldg(reinterpret_cast<const uint4 *>(a.resid + ((rb + cg) * a.W + x) * 8));
            }
        }
        mbar_wait(&bars[4], q & 1);
        tc_fence_after();
        if (tid == 0 && q + Cfg::NSLOT < n_loads) {  // the slot MMA(q) read is free again
            const int sl = q % Cfg::NSLOT, qn = q + Cfg::NSLOT;
            row_bulk<G>(s_ring + sl * Cfg::SLOT, kHalo, a.in, slot_job, a.H, a.W, y0 - 1 + qn, x0 - 1, &bars[sl]);
        }
        const uint32_t acc = tl + (uint32_t)(mod3(r) * NB);
        uint32_t v[NB];
        if constexpr (NB == 32) {
            uint32_t (&vv)[32] = *reinterpret_cast<uint32_t(*)[32]>(v);
            tmem_ld32(acc, vv);
        } else {
            uint32_t (&vv)[16] = *reinterpret_cast<uint32_t(*)[16]>(v);
            tmem_ld16(acc, vv);
        }
        tmem_wait_ld();
        tmem_zero<NB>(acc);  // row r's block becomes row r+3's
        if (valid) {
            {
                const size_t rowbase = ((size_t)slot_job * a.H + r) * (NB / 8);
#pragma unroll
                for (int cg = 0; cg < NB / 8; cg++) {
                    float f[8];
#pragma unroll
                    for (int i = 0; i < 8; i++) {
                        f[i] = __uint_as_float(v[cg * 8 + i]) + s_bias[cg * 8 + i];
                        if (EPI == EPI_RELU) f[i] = fmaxf(f[i], 0.f);
                    }
                    if constexpr (EPI == EPI_RESID) {
                        const uint4 rr = rres[cg];
                        f[0] += bf_lo(rr.x); f[1] += bf_hi(rr.x);
                        f[2] += bf_lo(rr.y); f[3] += bf_hi(rr.y);
                        f[4] += bf_lo(rr.z); f[5] += bf_hi(rr.z);
                        f[6] += bf_lo(rr.w); f[7] += bf_hi(rr.w);
                    }
                    uint4 o;
                    o.x = pack_bf16(f[0], f[1]); o.y = pack_bf16(f[2], f[3]);
                    o.z = pack_bf16(f[4], f[5]); o.w = pack_bf16(f[6], f[7]);
                    *reinterpret_cast<uint4 *>(a.out + ((rowbase + cg) * a.W + x) * 8) = o;
                }
            }
        }
        tmem_wait_st();
        tc_fence_before();
        __syncthreads();
        tc_fence_after();
    }
    if (warp == 0) tmem_dealloc(tmem, Cfg::TMEM_COLS);
}

// ------------------------------------------------------------------ fused residual block
constexpr int kRbMmaWarps = 4;
// h ring depth per tile: the slot of row q+NH is freed by E2(q+2), so the row
// load gets NH-3 steps of slack.  A/B on B200 (tools/build_variant.sh, body ms
// per c4 step): with tensor-box rows (~2,600-3,200 cycles issue -> landed on the
// clock64 timeline) NH 5 / 6 / 7 -> 114.6 / 105.1 / 109.6; with bulk-copied
// rows (~1,400-1,600 cycles) NH 5 / 6 / 7 -> 106.1 / 98.1 / 95.9.  7 is the
// most that fits (shared memory).
// Each h row of a tile arrives as C/8 one-dimensional bulk copies
// (one contiguous 16-B x 130-px run per channel group) instead of one tensor
// box whose innermost extent is 16 B (8 channels); the out-of-frame columns of
// a tile are zeroed once, out-of-frame rows by the producer.

constexpr int kRbThreads = 32 * (1 + kRbMmaWarps + 16);
// h_out = h + conv2(ReLU(conv1(h) + b1)) + b2 (EDSR block) in one kernel:
// h rows arrive once by TMA, t = ReLU(conv1) never leaves shared memory (it is
// written in the UMMA A-operand layout and consumed by conv2's MMAs), and the
// residual h is read back from the same ring.  Both convs use the rotated
// accumulators of k_conv_rot.  conv1 computes t for 128 positions x0-1 ..
// x0+126, so conv2 yields 126 valid outputs: tiles advance by 126 px.  Each CTA
// ping-pongs two x-tiles so one tile's epilogue overlaps the other's MMAs.
constexpr int kRbOut = kTile - 2;
struct RbArgs {
    int H, W, n_tiles, rows_per_cta, j0;
    const uint16_t *in;     // h [job][H][C/8][W][8] (rows by 1-D bulk copies)
    const SrJob *jobs;
    const int32_t *job_count;
    size_t b1_off, bias1_off, b2_off, bias2_off;
    uint16_t *out;
};
template <int C>
struct RbCfg {
    static constexpr int NB = C, KC = C / 16;
    static constexpr uint32_t B_BYTES = 30u * C * C;
    static constexpr uint32_t BIAS_BYTES = C * 4u;
    static constexpr uint32_t W_CONV = round_up(B_BYTES + BIAS_BYTES, 1024);
    static constexpr uint32_t SLOT_BYTES = kHalo * C * 2u;
    static constexpr uint32_t SLOT = round_up(SLOT_BYTES, 128);  // TMA destination: 128-B aligned
    static constexpr int NH = 7;                                 // h ring per tile
    static constexpr int NTS = 2;                                // t slots per tile (<= 4: e1t rotates over 4; 3 measured slower)
    static constexpr uint32_t TILE_BYTES = (NH + NTS) * SLOT;
    static constexpr uint32_t TCOLS = 2 * 3 * NB;                // conv1 + conv2 rings per tile
    static constexpr uint32_t TMEM_COLS = tmem_cols_for(2 * TCOLS);
    static constexpr int BPT = 2 * NH + 8 + NTS;                 // barriers per tile
    static constexpr int NBAR = 2 * BPT + 1;
    static constexpr uint32_t SMEM = 2 * W_CONV + 2 * TILE_BYTES + NBAR * 8 + 64;
    static_assert(SMEM <= 232448, "shared memory");
};
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void named_bar_sync(int id, int n) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
// Epilogue-group synchronisation of the fused res-block.  Every mbarrier poll
// and arrive is a shared-memory access, and a sleeping waiter re-polls on every
// barrier update of the CTA: with 128 threads arriving and 4 warps polling per
// group, ncu counted ~23M SYNCS polls per launch, ~18% of all shared-memory
// wavefronts of a kernel that is shared-memory-bandwidth bound (the MMA operand
// reads take the rest).  Tried: one arrive per warp (counts 4), after
// __syncwarp; and one warp of the group polls, the group follows on a
// named barrier (no shared-memory traffic).  A/B on B200 (tools/ab_libs.sh,
// body ms per c4 step): neither 104.5, ARRIVE1 105.4, GWAIT 108.1, both 110:
// the polls do not compete with the operand reads enough to matter, and the
// named-barrier hop lengthens the epilogue chain -- both off.
// NS_RB_BIAS_INIT: a retired accumulator block is re-initialised with the
// conv's bias instead of zero, so the epilogues add no bias (E1 becomes one
// cvt.rn.relu.bf16x2 per channel pair).
constexpr uint32_t kRbArriveCount = 128;
__device__ __forceinline__ void rb_arrive(uint64_t *bar) {
    mbar_arrive(bar);
}
__device__ __forceinline__ void rb_group_wait(uint64_t *bar, uint32_t phase, int group) {
    (void)group;
    mbar_wait(bar, phase);
}

// Warp roles: warp 0 = TMA producer, warp 1 = MMA issuer, warps 2-17 = four
// epilogue groups (tile 0 E1, tile 0 E2, tile 1 E1, tile 1 E2); warp w owns
// TMEM lanes 32 (w % 4).
// Per tile and input step q (h row y0-2+q): M1(q) conv1 -> E1(q) reads t row
// y0-3+q, writes it (ReLU, bf16) to t slot q%2 -> M2(q) conv2 on it -> E2(q)
// retires output row y0-4+q (+ b2 + h from the ring).  mbarriers only.
// Each epilogue signals twice: as soon as its accumulator block is read and
// zeroed (e1z / e2z: the next MMA group of that conv may start) and when its
// output is written (e1t: conv2 may read the t row).  So the next conv1 group
// never waits for the t row's conversion and stores: the tensor queue keeps
// both tiles' groups while the epilogues run (a drained queue costs the ~300-
// cycle commit round trip, tools/ubench.cu).
template <int C>
__global__ void __launch_bounds__(kRbThreads, 1) k_resblock(const __grid_constant__ CUtensorMap tm_in, const RbArgs a) {
    using Cfg = RbCfg<C>;
    constexpr int NB = Cfg::NB, NH = Cfg::NH;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *s_w1 = smem, *s_w2 = smem + Cfg::W_CONV;
    const float *s_b1 = reinterpret_cast<const float *>(s_w1 + Cfg::B_BYTES);
    const float *s_b2 = reinterpret_cast<const float *>(s_w2 + Cfg::B_BYTES);
    uint8_t *s_tile = smem + 2 * Cfg::W_CONV;
    uint64_t *bars = reinterpret_cast<uint64_t *>(s_tile + 2 * Cfg::TILE_BYTES);
    uint32_t *s_tmem = reinterpret_cast<uint32_t *>(bars + Cfg::NBAR);
    auto hslot = [&](int k, int i) { return s_tile + k * Cfg::TILE_BYTES + i * Cfg::SLOT; };
    auto tslot = [&](int k, int i) { return s_tile + k * Cfg::TILE_BYTES + (NH + i) * Cfg::SLOT; };
    // per tile: hfull[NH], m1, m2, e1z, e2z, e1t[4], tfree[NTS], hfree[NH]
    constexpr int BPT = Cfg::BPT;
    auto hfull = [&](int k, int i) { return &bars[k * BPT + i]; };
    auto m1bar = [&](int k) { return &bars[k * BPT + NH]; };
    auto m2bar = [&](int k) { return &bars[k * BPT + NH + 1]; };
    auto e1z = [&](int k) { return &bars[k * BPT + NH + 2]; };
    auto e2z = [&](int k) { return &bars[k * BPT + NH + 3]; };
    auto e1t = [&](int k, int i) { return &bars[k * BPT + NH + 4 + i]; };
    auto tfree = [&](int k, int i) { return &bars[k * BPT + NH + 8 + i]; };
    auto hfree = [&](int k, int i) { return &bars[k * BPT + NH + 8 + Cfg::NTS + i]; };
    uint64_t *wbar = &bars[2 * BPT];

    const int slot_job = blockIdx.z;
    const int job = a.j0 + slot_job;
    if (a.job_count && job >= *a.job_count) return;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int y0 = blockIdx.y * a.rows_per_cta;
    const int y1 = min(y0 + a.rows_per_cta, a.H);
    const int nq = y1 - y0 + 4;  // h rows y0-2 .. y1+1
    // tile k of this CTA: x0 = (2 blockIdx.x + k) kRbOut (computed, not indexed: no local memory)
    auto x0k = [&](int k) { return (2 * (int)blockIdx.x + k) * kRbOut; };
    auto vk = [&](int k) { return 2 * (int)blockIdx.x + k < a.n_tiles; };

    if (tid == 0) {
        for (int k = 0; k < 2; k++) {
            for (int i = 0; i < NH; i++) mbar_init(hfull(k, i), 1);
            for (int i = 0; i < NH; i++) mbar_init(hfree(k, i), kRbArriveCount);
            mbar_init(m1bar(k), 1);
            mbar_init(m2bar(k), 1);
            mbar_init(e1z(k), kRbArriveCount);
            mbar_init(e2z(k), kRbArriveCount);
            for (int i = 0; i < 4; i++) mbar_init(e1t(k, i), kRbArriveCount);
            for (int i = 0; i < Cfg::NTS; i++) mbar_init(tfree(k, i), 1);
        }
        mbar_init(wbar, 1);
        fence_mbar_init();
    }
    if (warp == 0) tmem_alloc(s_tmem, Cfg::TMEM_COLS);
    for (int i = tid; i < (int)(2 * Cfg::NTS * (Cfg::SLOT / 16)); i += blockDim.x) {  // t slots start at zero
        const int ks = i / (Cfg::SLOT / 16), o = i % (Cfg::SLOT / 16);
        reinterpret_cast<uint4 *>(tslot(ks / Cfg::NTS, ks % Cfg::NTS))[o] = make_uint4(0, 0, 0, 0);
    }
    // h slot column c <-> x = x0k - 2 + c; in-frame columns [c_lo, c_hi)
    auto c_lo = [&](int k) { return max(0, 2 - x0k(k)); };
    auto c_hi = [&](int k) { return min(kHalo, a.W - x0k(k) + 2); };
    for (int i = tid; i < 2 * NH * (C / 8) * kHalo; i += blockDim.x) {  // out-of-frame columns stay zero
        const int c = i % kHalo, cg = (i / kHalo) % (C / 8), sl = (i / (kHalo * (C / 8))) % NH, k = i / (kHalo * (C / 8) * NH);
        if (c < c_lo(k) || c >= c_hi(k))
            reinterpret_cast<uint4 *>(hslot(k, sl) + cg * kHalo * 16)[c] = make_uint4(0, 0, 0, 0);
    }
    fence_proxy_async_smem();
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *s_tmem;
    const SrJob J = a.jobs[job];
    if (warp > kRbMmaWarps) {
        // both accumulator rings start at zero: the blocks of t row y0-1 and of
        // output row y0 are first touched before any retirement could zero them
        // (TMEM keeps whatever an earlier CTA on this SM left unretired)
        const int g = (warp - 1 - kRbMmaWarps) / 4, k = g / 2, role = g % 2;
        const uint32_t tl = tmem + ((uint32_t)((warp % 4) * 32) << 16) + k * Cfg::TCOLS + role * 3 * NB;
#pragma unroll 1
        for (int b = 0; b < 3; b++) tmem_zeroN<NB>(tl + b * NB);
        tmem_wait_st();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();

    if (warp == 0) {
        // ---------------------------------------------------------------- TMA producer
        if (lane == 0) {
            NS_TR_ROLE(0);
            prefetch_tmap(&tm_in);
            mbar_arrive_expect_tx(wbar, 2 * (Cfg::B_BYTES + Cfg::BIAS_BYTES));
            bulk_load(s_w1, J.wts + a.b1_off, Cfg::B_BYTES, wbar);
            bulk_load(s_w1 + Cfg::B_BYTES, J.wts + a.bias1_off, Cfg::BIAS_BYTES, wbar);
            bulk_load(s_w2, J.wts + a.b2_off, Cfg::B_BYTES, wbar);
            bulk_load(s_w2 + Cfg::B_BYTES, J.wts + a.bias2_off, Cfg::BIAS_BYTES, wbar);
            for (int q = 0; q < nq; q++) {
                for (int k = 0; k < 2; k++) {
                    if (!vk(k)) continue;
                    const int sl = q % NH;
                    // slot reuse: h row q-NH was last read by E2 at step q-NH+2, which
                    // arrives on hfree[slot] (one completion per reuse: never runs ahead)
                    if (q >= NH) mbar_wait(hfree(k, sl), ((q / NH) - 1) & 1);
                    const int yy = y0 - 2 + q, lo = c_lo(k), hi = c_hi(k);
                    if (yy < 0 || yy >= a.H) {  // zero padding row: in-frame columns to zero
                        for (int cg = 0; cg < C / 8; cg++)
                            for (int c = lo; c < hi; c++)
                                reinterpret_cast<uint4 *>(hslot(k, sl) + cg * kHalo * 16)[c] = make_uint4(0, 0, 0, 0);
                        fence_proxy_async_smem();
                        mbar_arrive(hfull(k, sl));
                    } else {
                        const uint32_t run = (uint32_t)(hi - lo) * 16u;
                        mbar_arrive_expect_tx(hfull(k, sl), run * (C / 8));
                        const uint16_t *src = a.in + (((size_t)slot_job * a.H + yy) * (C / 8) * a.W +
                                                      (size_t)(x0k(k) - 2 + lo)) * 8;
                        for (int cg = 0; cg < C / 8; cg++)
                            bulk_load(hslot(k, sl) + cg * kHalo * 16 + lo * 16, src + (size_t)cg * a.W * 8, run,
                                      hfull(k, sl));
                    }
                    NS_TR(30 + k, q);
                }
            }
        }
    } else if (warp <= kRbMmaWarps) {
        // ---------------------------------------------------------------- MMA issuers
        // Four independent issuer warps, one per (conv, tile): warp 1 M1(A),
        // 2 M1(B), 3 M2(A), 4 M2(B).  A waiting issuer (each mbarrier hop is
        // ~130 cycles, tools/ubench.cu) no longer stalls the other streams, so
        // the tensor queue is fed while any one of them waits.  Each warp runs
        // its schedule uniformly; one elected lane issues the 6 MMAs + commit.
        //   M1(k,q) needs hfull(k,q) and e1z(k,q-1) (block of row y0-3+q+1 zeroed);
        //   M2(k,q) needs e1t(k,q) (t row written) and e2z(k,q-1), and releases t
        //   slot q%2 through tfree.
        // Bound on how far conv1 runs ahead: M1(q) needs h row q, whose ring slot
        // E2(q-3) frees, so M2(q-3) is complete whenever E1(q) runs; E1 therefore
        // leads conv2's wait by <= 2 steps and e1t rotates over 4 barriers.
        const int mw = warp - 1, conv = mw >> 1, k = mw & 1;
        NS_TR_ROLE(1 + mw);
        if (vk(k)) {
            const uint32_t idesc = idesc_bf16_f32(128, 3 * NB);
            auto mma_rot = [&](uint32_t dcol, const uint8_t *aslot, const uint8_t *wstrip, int yin, uint64_t *bar,
                               uint64_t *bar0) {
                const uint32_t abase = smem_u32(aslot);
                const uint32_t wbase = smem_u32(wstrip) + (uint32_t)mod3(1 - yin) * NB * 16;
                const uint64_t ad0 = smem_desc(abase, kHalo * 16, 128), bd0 = smem_desc(wbase, 5 * NB * 16, 128);
                if (elect_one()) {
#pragma unroll
                    for (int dx = 0; dx < 3; dx++)
#pragma unroll
                        for (int kc = 0; kc < Cfg::KC; kc++)  // descriptor start address is bits 0-13 (>> 4)
                            umma_bf16(dcol, ad0 + (uint64_t)((2 * kc * kHalo * 16 + dx * 16) >> 4),
                                      bd0 + (uint64_t)(((dx * Cfg::KC + kc) * 2 * 5 * NB * 16) >> 4), idesc, 1u);
                    if (bar0) umma_commit(bar0);  // (the issuing thread's commits track its own MMAs)
                    umma_commit(bar);
                }
                __syncwarp();
            };
            mbar_wait(wbar, 0);
            if (conv == 0) {
                for (int q = 0; q < nq; q++) {  // conv1 on h row y0-2+q
                    if (q >= 1) mbar_wait(e1z(k), (q - 1) & 1);
                    mbar_wait(hfull(k, q % NH), (q / NH) & 1);
                    if (lane == 0) NS_TR(1 + k, q);
                    tc_fence_after();
                    mma_rot(tmem + k * Cfg::TCOLS, hslot(k, q % NH), s_w1, y0 - 2 + q, m1bar(k), nullptr);
                    if (lane == 0) NS_TR(3 + k, q);
                }
            } else {
                for (int q = 2; q < nq; q++) {  // conv2 on t row y0-3+q
                    mbar_wait(e1t(k, (q - 2) & 3), ((q - 2) >> 2) & 1);
                    if (q >= 3) mbar_wait(e2z(k), (q - 3) & 1);
                    if (lane == 0) NS_TR(5 + k, q);
                    tc_fence_after();
                    // tfree: t slot q%2 may be overwritten once these MMAs complete
                    mma_rot(tmem + k * Cfg::TCOLS + 3 * NB, tslot(k, q % Cfg::NTS), s_w2, y0 - 3 + q, m2bar(k),
                            tfree(k, q % Cfg::NTS));
                    if (lane == 0) NS_TR(7 + k, q);
                }
            }
        }
    } else {
        // ---------------------------------------------------------------- epilogues
        // warps 5..20: group g -> tile k = g/2, role = g%2 (E1 | E2).
        // E1 (t -> SMEM, needs the async-proxy fence) and E2 (global stores) run
        // in different warps so the fence never waits on in-flight global stores.
        const int g = (warp - 1 - kRbMmaWarps) / 4, k = g / 2, role = g % 2;
        if (vk(k)) {
            const int ew = warp % 4;   // TMEM lane quarter
            const int p = ew * 32 + lane;
            const uint32_t tl = tmem + ((uint32_t)(ew * 32) << 16) + k * Cfg::TCOLS;
            mbar_wait(wbar, 0);
            NS_TR_ROLE(5 + g);
            float bias[NB];  // b1 (E1) or b2 (E2), kept in registers: no shared loads on the critical chain
#pragma unroll
            for (int i = 0; i < NB; i += 4) {
                const float4 b4 = *reinterpret_cast<const float4 *>((role == 0 ? s_b1 : s_b2) + i);
                bias[i] = b4.x; bias[i + 1] = b4.y; bias[i + 2] = b4.z; bias[i + 3] = b4.w;
            }
            if (role == 0) {
                for (int q = 0; q < nq; q++) {  // E1: t = ReLU(conv1 + b1) -> t slot
                    const int yt = y0 - 3 + q;
                    rb_group_wait(m1bar(k), q & 1, g);
                    if (warp % 4 == 2 && lane == 0) NS_TR(10 + k, q);
                    tc_fence_after();
#ifdef NS_TRACE_NOEPI
                    tc_fence_before();
                    rb_arrive(e1z(k));
                    if (q >= 2) rb_arrive(e1t(k, (q - 2) & 3));
                    continue;
#endif
                    const uint32_t acc = tl + (uint32_t)(mod3(yt) * NB);
                    uint32_t v[NB];
                    tmem_ldN<NB>(acc, v);
                    tmem_wait_ld();
                    if (warp % 4 == 2 && lane == 0) NS_TR(40 + k, q);
                    // the retired block becomes row yt+3's: it starts at b1, so the
                    // epilogue adds no bias (the first three rows retire blocks zeroed at
                    // allocation and add it here)
                    if (q < 3) {
#pragma unroll
                        for (int i = 0; i < NB; i++) v[i] = __float_as_uint(__uint_as_float(v[i]) + bias[i]);
                    }
                    tmem_st_vals<NB>(acc, bias);
                    tmem_wait_st();

                    tc_fence_before();
                    rb_arrive(e1z(k));  // the next conv1 group may start
                    // t slot q%2 was last read by M2(q-2) (another warp's MMAs): completion
                    // #((q-4)/2) of tfree[q%2]; M2(q-4) is done, M2(q) cannot be -> exact
                    if (q >= 2 + Cfg::NTS) rb_group_wait(tfree(k, q % Cfg::NTS), ((q - Cfg::NTS - 2) / Cfg::NTS) & 1, g);
                    if (q >= 2) {
                        const int xt = x0k(k) - 1 + p;
                        const bool inside = yt >= 0 && yt < a.H && xt >= 0 && xt < a.W;
                        uint8_t *ts = tslot(k, q % Cfg::NTS);
#pragma unroll
                        for (int cg = 0; cg < NB / 8; cg++) {
                            const uint32_t *w = v + cg * 8;
                            auto pr = [&](int i) {
                                return inside ? pack_bf16_relu(__uint_as_float(w[i]), __uint_as_float(w[i + 1])) : 0u;
                            };
                            const uint4 o = make_uint4(pr(0), pr(2), pr(4), pr(6));
                            *reinterpret_cast<uint4 *>(ts + cg * kHalo * 16 + p * 16) = o;
                        }
                    }
                    if (warp % 4 == 2 && lane == 0) NS_TR(42 + k, q);
                    fence_proxy_async_smem();
                    if (warp % 4 == 2 && lane == 0) NS_TR(46 + k, q);
                    // t rows y0-3, y0-2 (q < 2) feed no conv2 output: no arrival, so
                    // every phase of e1t is waited on by M2 (compute-sanitizer synccheck)
                    if (q >= 2) rb_arrive(e1t(k, (q - 2) & 3));
                    if (warp % 4 == 2 && lane == 0) NS_TR(12 + k, q);
                }
            } else {
                for (int q = 2; q < nq; q++) {  // E2: out = conv2 + b2 + h
                    const int yo = y0 - 4 + q;
                    rb_group_wait(m2bar(k), (q - 2) & 1, g);
                    if (warp % 4 == 2 && lane == 0) NS_TR(20 + k, q);
                    tc_fence_after();
#ifdef NS_TRACE_NOEPI
                    tc_fence_before();
                    rb_arrive(hfree(k, (q - 2) % NH));
                    rb_arrive(e2z(k));
                    continue;
#endif
                    const uint32_t acc = tl + 3 * NB + (uint32_t)(mod3(yo) * NB);
                    uint32_t v[NB];
                    tmem_ldN<NB>(acc, v);
                    tmem_wait_ld();
                    const bool addb = q < 5;  // first three retirements: blocks zeroed at allocation
                    tmem_st_vals<NB>(acc, bias);
                    tmem_wait_st();

                    tc_fence_before();
                    rb_arrive(e2z(k));  // the next conv2 group may start
                    const int x = x0k(k) + p;
                    if (yo >= y0 && yo < y1 && p < kRbOut && x < a.W) {
                        const uint8_t *hs = hslot(k, (q - 2) % NH);  // h row yo (step q-2)
                        const size_t rowbase = ((size_t)slot_job * a.H + yo) * (NB / 8);
#pragma unroll
                        for (int cg = 0; cg < NB / 8; cg++) {
                            const uint4 rr = *reinterpret_cast<const uint4 *>(hs + cg * kHalo * 16 + (p + 2) * 16);
                            float f[8];
#pragma unroll
                            for (int i = 0; i < 8; i++)
                                f[i] = addb ? __uint_as_float(v[cg * 8 + i]) + bias[cg * 8 + i] : __uint_as_float(v[cg * 8 + i]);
                            f[0] += bf_lo(rr.x); f[1] += bf_hi(rr.x);
                            f[2] += bf_lo(rr.y); f[3] += bf_hi(rr.y);
                            f[4] += bf_lo(rr.z); f[5] += bf_hi(rr.z);
                            f[6] += bf_lo(rr.w); f[7] += bf_hi(rr.w);
                            uint4 o;
                            o.x = pack_bf16(f[0], f[1]); o.y = pack_bf16(f[2], f[3]);
                            o.z = pack_bf16(f[4], f[5]); o.w = pack_bf16(f[6], f[7]);
                            *reinterpret_cast<uint4 *>(a.out + ((rowbase + cg) * a.W + x) * 8) = o;
                        }
                    }
                    rb_arrive(hfree(k, (q - 2) % NH));
                    if (warp % 4 == 2 && lane == 0) NS_TR(22 + k, q);
                }
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tmem_dealloc(tmem, Cfg::TMEM_COLS);
}

// ------------------------------------------------------------------ composed upsampler + tail
// tail o pixel-shuffle o upsampler is linear (EDSR has no nonlinearity between
// them), so it equals one 5x5 conv at LR resolution from h (C ch) to s*s*3
// outputs (CompShape).  This executes 2*25*C*3s^2 FLOP per LR pixel instead of
// 18 s^2 C^2 + 54 C s^2 and never materialises the HR feature map u (531 MB per
// 4K anchor).  It equals the definition exactly except on the 1-pixel HR frame
// border (the tail zero-pads u there); k_uptail_border_* recompute that ring.
// Same rotated-accumulator scheme as k_conv_rot with 5 kernel rows: output LR
// row r lives in block r mod 5, the 9-block strip [W4..W0, W4..W1] window start
// is (2 - y mod 5) mod 5, N = 5 nb.  The epilogue adds the integer bilinear
// skip up_s(LR) (O6), rounds, clamps and writes the s x s HR pixels of each
// LR pixel through a shared-memory tile (8-byte stores).
constexpr int kHalo5 = kTile + 4;
constexpr int kLrBoxW = kTile + 32;  // u8 LR box x0-16 .. x0+143: the innermost TMA start must be 16-B aligned
constexpr int kLrBoxX = 16;          // box origin = x0 - kLrBoxX
template <int CIN, int NB, int S>
struct UpCfg {
    static constexpr int KC = CIN / 16;
    static constexpr uint32_t B_BYTES = 5u * KC * 2 * 9 * NB * 16;
    static constexpr uint32_t BIAS_BYTES = NB * 4u;
    static constexpr uint32_t W_REGION = round_up(B_BYTES + BIAS_BYTES, 1024);
    static constexpr uint32_t SLOT_BYTES = kHalo5 * CIN * 2u;
    static constexpr uint32_t SLOT = round_up(SLOT_BYTES, 1024);
    static constexpr int NSLOT = 3;
    static constexpr uint32_t OUT_BYTES = 3u * S * kTile * S;  // HR tile [plane][i][s*128]
    static constexpr uint32_t TMEM_COLS = tmem_cols_for(5 * NB);
    static constexpr uint32_t SMEM = W_REGION + NSLOT * SLOT + round_up(OUT_BYTES, 128) + 128;
    static_assert((5 * NB) % 16 == 0 && 5 * NB <= 256, "N = 5 nb");
    static_assert(SMEM <= 232448, "shared memory");
};

template <int CIN, int NB, int S>
__global__ void __launch_bounds__(128) k_uptail(const __grid_constant__ CUtensorMap tm_in, const ConvArgs a) {
    using Cfg = UpCfg<CIN, NB, S>;
    constexpr int NOUT = S * S * 3;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *s_w = smem;
    const float *s_bias = reinterpret_cast<const float *>(smem + Cfg::B_BYTES);
    uint8_t *s_ring = smem + Cfg::W_REGION;
    uint8_t *s_out = s_ring + Cfg::NSLOT * Cfg::SLOT;
    uint64_t *bars = reinterpret_cast<uint64_t *>(s_out + round_up(Cfg::OUT_BYTES, 128));  // [0,3) ring, 3 w, 4 mma
    uint32_t *s_tmem = reinterpret_cast<uint32_t *>(bars + 6);

    const int slot_job = blockIdx.z;
    const int job = a.j0 + slot_job;
    if (a.job_count && job >= *a.job_count) return;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int x0 = blockIdx.x * kTile;
    const int y0 = blockIdx.y * a.rows_per_cta;
    const int y1 = min(y0 + a.rows_per_cta, a.H);
    const int n_loads = y1 - y0 + 4;  // input rows y0-2 .. y1+1
    const int lh = a.H, lw = a.W;     // LR dims (the conv runs at LR resolution)
    const int HH = lh * S, WW = lw * S;

    if (tid == 0) {
        for (int i = 0; i < 5; i++) mbar_init(&bars[i], 1);
        fence_mbar_init();
    }
    if (warp == 0) tmem_alloc(s_tmem, Cfg::TMEM_COLS);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *s_tmem;
    const uint32_t tl = tmem + ((uint32_t)(warp * 32) << 16);
    const SrJob J = a.jobs[job];
    uint8_t *const hr_dst = a.hr_tmp ? a.hr_tmp + (size_t)slot_job * a.hr_tmp_frame : J.hr;
    if (tid == 0) {
        prefetch_tmap(&tm_in);
        mbar_arrive_expect_tx(&bars[3], Cfg::B_BYTES + Cfg::BIAS_BYTES);
        bulk_load(s_w, J.wts + a.b_off, Cfg::B_BYTES, &bars[3]);
        bulk_load(smem + Cfg::B_BYTES, J.wts + a.bias_off, Cfg::BIAS_BYTES, &bars[3]);
        for (int q = 0; q < Cfg::NSLOT && q < n_loads; q++) {
            mbar_arrive_expect_tx(&bars[q], Cfg::SLOT_BYTES);
            tma_load_5d(s_ring + q * Cfg::SLOT, &tm_in, &bars[q], 0, x0 - 2, 0, y0 - 2 + q, slot_job);
        }
    }
#pragma unroll
    for (int b = 0; b < 5; b++) tmem_zeroN<NB>(tl + b * NB);
    tmem_wait_st();
    mbar_wait(&bars[3], 0);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();

    const uint32_t idesc = idesc_bf16_f32(128, 5 * NB);
    const int p = warp * 32 + lane;
    const int x = x0 + p;
    for (int q = 0; q < n_loads; q++) {
        const int yin = y0 - 2 + q;
        if (tid == 0) {
            const int sl = q % Cfg::NSLOT;
            mbar_wait(&bars[sl], (q / Cfg::NSLOT) & 1);
            tc_fence_after();
            const uint32_t abase = smem_u32(s_ring + sl * Cfg::SLOT);
            const uint32_t start = (uint32_t)mod5(2 - yin);
            const uint32_t wbase = smem_u32(s_w) + start * NB * 16;
#pragma unroll
            for (int dx = 0; dx < 5; dx++) {
#pragma unroll
                for (int kc = 0; kc < Cfg::KC; kc++) {
                    const uint64_t ad =
                        smem_desc(abase + (uint32_t)(2 * kc * kHalo5 * 16 + dx * 16), kHalo5 * 16, 128);
                    const uint64_t bd =
                        smem_desc(wbase + (uint32_t)((dx * Cfg::KC + kc) * 2 * 9 * NB * 16), 9 * NB * 16, 128);
                    umma_bf16(tmem, ad, bd, idesc, 1u);
                }
            }
            umma_commit(&bars[4]);
        }
        __syncwarp();
        const int r = yin - 2;  // LR output row completed by this input row
        const bool valid_row = r >= y0;
        // bilinear-skip taps for this lane (O6, compile-time sub-pixel weights), from
        // the batch's u8 copy of the net's input planes (k_prep_lr: [job][H][3][wp])
        int Lv[3][3][3];
        if (valid_row && x < lw) {
#pragma unroll
            for (int c = 0; c < 3; c++) {
#pragma unroll
                for (int dy = 0; dy < 3; dy++) {
                    const uint8_t *Lr =
                        a.lr8 + (((size_t)slot_job * lh + min(max(r + dy - 1, 0), lh - 1)) * 3 + c) * a.wp;
#pragma unroll
                    for (int dx = 0; dx < 3; dx++) Lv[c][dy][dx] = Lr[min(max(x + dx - 1, 0), lw - 1)];
                }
            }
        }
        mbar_wait(&bars[4], q & 1);
        tc_fence_after();
        if (tid == 0 && q + Cfg::NSLOT < n_loads) {
            const int sl = q % Cfg::NSLOT, qn = q + Cfg::NSLOT;
            mbar_arrive_expect_tx(&bars[sl], Cfg::SLOT_BYTES);
            tma_load_5d(s_ring + sl * Cfg::SLOT, &tm_in, &bars[sl], 0, x0 - 2, 0, y0 - 2 + qn, slot_job);
        }
        const uint32_t acc = tl + (uint32_t)(mod5(r) * NB);
        uint32_t v[NB];
        tmem_ldN<NB>(acc, v);
        tmem_wait_ld();
        tmem_zeroN<NB>(acc);
        if (valid_row) {
            // HR pixels (S r + i, S x + j): clamp(floor(up_s(LR) + t + 0.5)) -> smem tile
#pragma unroll
            for (int i = 0; i < S; i++) {
                const int dya = tap_d_sr<S>(i) + 1, wy = tap_w1_sr<S>(i);
#pragma unroll
                for (int j = 0; j < S; j++) {
                    const int dxa = tap_d_sr<S>(j) + 1, wx = tap_w1_sr<S>(j);
#pragma unroll
                    for (int c = 0; c < 3; c++) {
                        const int n = (i * S + j) * 3 + c;
                        const int vv = (128 - wy) * ((128 - wx) * Lv[c][dya][dxa] + wx * Lv[c][dya][dxa + 1]) +
                                       wy * ((128 - wx) * Lv[c][dya + 1][dxa] + wx * Lv[c][dya + 1][dxa + 1]);
                        const int U = (vv + 8192) >> 14;
                        const float t = __uint_as_float(v[n]) + s_bias[n];
                        const float o = fminf(fmaxf(floorf((float)U + t + 0.5f), 0.f), 255.f);
                        s_out[(c * S + i) * (kTile * S) + p * S + j] = (uint8_t)o;
                    }
                }
            }
            // frame-border ring (rare lanes): keep the fp32 composed t for the exact fix-up
            if (x < lw && (r == 0 || r == lh - 1 || x == 0 || x == lw - 1)) {
                for (int i = 0; i < S; i++)
                    for (int j = 0; j < S; j++) {
                        const int Y = S * r + i, X = S * x + j;
                        if (!(Y == 0 || Y == HH - 1 || X == 0 || X == WW - 1)) continue;
                        const int ri = Y == 0 ? X : Y == HH - 1 ? WW + X
                                     : X == 0 ? 2 * WW + (Y - 1) : 2 * WW + (HH - 2) + (Y - 1);
                        for (int c = 0; c < 3; c++) {
                            const int n = (i * S + j) * 3 + c;
                            a.ring[((size_t)slot_job * (2 * WW + 2 * (HH - 2)) + ri) * 3 + c] =
                                __uint_as_float(v[n]) + s_bias[n];
                        }
                    }
            }
        }
        tmem_wait_st();
        tc_fence_before();
        __syncthreads();
        if (valid_row) {  // coalesced 8-byte stores of the HR tile rows
            const int xs_hr = x0 * S, wv = min(kTile, lw - x0) * S;  // valid HR bytes per row (multiple of 8)
            constexpr int CH = kTile * S / 8;
            for (int e = tid; e < 3 * S * CH; e += 128) {
                const int ch = e % CH, ri = e / CH, c = ri / S, i = ri % S;
                if (ch * 8 < wv)
                    *reinterpret_cast<uint2 *>(hr_dst + (size_t)c * HH * WW + (size_t)(S * r + i) * WW + xs_hr + ch * 8) =
                        *reinterpret_cast<const uint2 *>(s_out + ri * (kTile * S) + ch * 8);
            }
        }
        __syncthreads();
        tc_fence_after();
    }
    if (warp == 0) tmem_dealloc(tmem, Cfg::TMEM_COLS);
    (void)NOUT;
}

// Warp-specialized composed upsampler+tail for s <= 3: warp 0 TMA, warp 1 MMA
// (elect.sync groups), 2 x-tiles per CTA, and per tile S epilogue groups of 4
// warps (group g = HR sub-row i) that read the retired row in parallel.  The
// 5-block accumulator ring (row r -> block r mod 5) is the same as k_uptail;
// the MMA on input row y waits for the epilogue of row y-3 (previous step),
// and the other tile's MMAs cover that wait.  The TMA warp also stages the
// three u8 LR rows r-1..r+1 of each output row r (bilinear skip taps) in a
// separate ring that the epilogue groups release.  Input ring depth: 3 and 4
// measured equal while the epilogue groups met on a per-step barrier; with the
// bias-initialised columns (no barrier): 3 / 4 / 5 / 6 / 7 -> 18.3 / 16.2 /
// 14.8-15.3 / 15.4-15.5 / 15.5-15.6 ms per c4 step.
template <int CIN, int NB, int S>
struct Up2Cfg {
    static constexpr int KC = CIN / 16, NSTRIP = 9;
    static constexpr uint32_t B_BYTES = 5u * KC * 2 * NSTRIP * NB * 16;
    static constexpr uint32_t BIAS_BYTES = NB * 4u;
    static constexpr uint32_t W_REGION = round_up(B_BYTES + BIAS_BYTES, 1024);
    static constexpr uint32_t SLOT_BYTES = kHalo5 * CIN * 2u;
    static constexpr uint32_t SLOT = round_up(SLOT_BYTES, 128);     // TMA destination: 128-B aligned
    static constexpr int NS = 5;                                    // input ring per tile
    static constexpr int NL = 3;                                    // LR ring per tile
    static constexpr uint32_t LR_BYTES = 9u * kLrBoxW;              // [row 3][plane 3][kLrBoxW]
    static constexpr uint32_t LSLOT = round_up(LR_BYTES, 128);
    static constexpr uint32_t TILE_BYTES = NS * SLOT + NL * LSLOT;
    static constexpr uint32_t TCOLS = 5 * NB;
    static constexpr uint32_t TMEM_COLS = tmem_cols_for(2 * TCOLS);
    static constexpr int BPT = 2 * NS + 3 + 2 * NL;                // barriers per tile
    static constexpr int NBAR = 2 * BPT + 1;
    static constexpr int NWARPS = 2 + 2 * S * 4;
    static constexpr uint32_t SMEM = W_REGION + 2 * TILE_BYTES + NBAR * 8 + 64;
    static_assert(5 * NB <= 256, "N = 5 nb");
    static_assert(SMEM <= 232448, "shared memory");
};

__device__ __forceinline__ void named_bar(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory"); }

// Compile-time bilinear tap of HR index S*x + I (same formula as up_tap with
// the x-dependent part split off): source index x + off, weight w1 / 128.
template <int S, int I>
struct UpTapC {
    static constexpr int u = 2 * I + 1 - S;  // |u| < 2S
    static constexpr int off = u < 0 ? -1 : 0;
    static constexpr int w1 = (128 * (u - 2 * S * off) + S) / (2 * S);
};

// Accumulator columns one epilogue group reads: sub-row I uses n in
// [3 S I, 3 S (I+1)); a 16-column window from the 8-aligned base covers it.
template <int NB, int S>
struct UpCols {
    static constexpr int LW = NB < 16 ? NB : 16;
    __host__ __device__ static constexpr int base(int I) { return NB <= 16 ? 0 : 8 * ((3 * S * I) / 8); }
    __host__ __device__ static constexpr bool fits() {
        for (int I = 0; I < S; I++)
            if (3 * S * (I + 1) - base(I) > LW) return false;
        return true;
    }
    static_assert(fits(), "sub-row column window");
};

// floor + clamp to [0, 255] in one conversion
__device__ __forceinline__ uint32_t f2u8_floor_sat(float v) {
    uint32_t o;
    asm("cvt.rmi.sat.u8.f32 %0, %1;" : "=r"(o) : "f"(v));
    return o;
}

// One HR sub-row I of an LR pixel: the s outputs x 3 planes of the composed
// conv + the integer bilinear skip, rounded and clamped into the staging row.
// lr: this step's staged LR rows [3][3][kLrBoxW] (row r-1+i, column x0-kLrBoxX+j);
// ra/rb: staged rows of the vertical taps; cm/c0/cp: staged columns of x-1,
// x, x+1 (clamped as up_tap clamps); bh: bias + 0.5 of this sub-row's outputs.
template <int NB, int S, int I>
__device__ __forceinline__ void uptail_subrow(const uint32_t (&v)[UpCols<NB, S>::LW], const float (&bh)[3 * S],
                                              const uint8_t *lr, int ra, int rb, int cm, int c0, int cp,
                                              uint8_t *so, size_t cstride, int p) {
    constexpr int wy = UpTapC<S, I>::w1;
    constexpr int base = UpCols<NB, S>::base(I);
    // O6 is separable with exact integer weights: the vertical pass first,
    // va[c][t] = (128 - wy) a + wy b per LR column t of the 3 taps, then per output
    // ((128 - wx) va[ox] + wx va[ox + 1] + 8192) >> 14 -- the same sum as
    // horizontal-first (distributivity, no intermediate rounding), 3 column
    // values per plane instead of 2 per output; sub-rows with wy = 0 read one
    // LR row only.
    int va[3][3];
#pragma unroll
    for (int c = 0; c < 3; c++) {
        const uint8_t *La = lr + (ra * 3 + c) * kLrBoxW;
        const int a0 = La[cm], a1 = La[c0], a2 = La[cp];
        if constexpr (wy == 0) {
            va[c][0] = 128 * a0; va[c][1] = 128 * a1; va[c][2] = 128 * a2;
        } else {
            const uint8_t *Lb = lr + (rb * 3 + c) * kLrBoxW;
            va[c][0] = (128 - wy) * a0 + wy * Lb[cm];
            va[c][1] = (128 - wy) * a1 + wy * Lb[c0];
            va[c][2] = (128 - wy) * a2 + wy * Lb[cp];
        }
    }
#pragma unroll
    for (int j = 0; j < S; j++) {
        const int ox = 1 + (2 * j + 1 - S < 0 ? -1 : 0);
        const int wx = (128 * ((2 * j + 1 - S) - 2 * S * (ox - 1)) + S) / (2 * S);
#pragma unroll
        for (int c = 0; c < 3; c++) {
            const int U = (wx ? (128 - wx) * va[c][ox] + wx * va[c][ox + 1] : 128 * va[c][ox]) + 8192 >> 14;
            const int n = (I * S + j) * 3 + c;
            so[c * cstride + p * S + j] = (uint8_t)f2u8_floor_sat((float)U + (__uint_as_float(v[n - base]) + bh[n - 3 * S * I]));
        }
    }
}

// frame-border ring pixels of sub-row I keep their fp32 t = acc + bias for the
// exact fix-up (k_uptail_ring)
template <int NB, int S, int I>
__device__ __forceinline__ void uptail_ring_store(const uint32_t (&v)[UpCols<NB, S>::LW], const float (&be)[3 * S],
                                               const ConvArgs &a, int x, int r, int lh, int lw, int slot_job) {
    constexpr int base = UpCols<NB, S>::base(I);
    const int HH = lh * S, WW = lw * S;
    const int Y = S * r + I;
#pragma unroll
    for (int j = 0; j < S; j++) {
        const int X = S * x + j;
        if (Y == 0 || Y == HH - 1 || X == 0 || X == WW - 1) {
            const int ri = Y == 0 ? X : Y == HH - 1 ? WW + X : X == 0 ? 2 * WW + (Y - 1) : 2 * WW + (HH - 2) + (Y - 1);
#pragma unroll
            for (int c = 0; c < 3; c++) {
                const int n = (I * S + j) * 3 + c;
                // t = acc + bias: be = bias + 1/2 while the block starts at zero, 0 once it
                // starts at bias + 1/2
                a.ring[((size_t)slot_job * (2 * WW + 2 * (HH - 2)) + ri) * 3 + c] =
                    __uint_as_float(v[n - base]) + be[n - 3 * S * I] - 0.5f;
            }
        }
    }
}

template <int NB, int S, int I>
__device__ __forceinline__ void uptail_group_step(const uint32_t (&v)[UpCols<NB, S>::LW], const float (&bh)[3 * S],
                                                  const float *s_bias, const uint8_t *lr, int r, int x, int x0,
                                                  int lh, int lw, const ConvArgs &a, uint8_t *so, size_t cstride, int p,
                                                  int slot_job) {
    constexpr int oy = UpTapC<S, I>::off;
    const int ra = min(max(r + oy, 0), lh - 1) - (r - 1), rb = min(max(r + oy + 1, 0), lh - 1) - (r - 1);
    const int cm = max(x - 1, 0) - (x0 - kLrBoxX), c0 = x - (x0 - kLrBoxX), cp = min(x + 1, lw - 1) - (x0 - kLrBoxX);
    uptail_subrow<NB, S, I>(v, bh, lr, ra, rb, cm, c0, cp, so, cstride, p);
    if (r == 0 || r == lh - 1 || x == 0 || x == lw - 1) uptail_ring_store<NB, S, I>(v, bh, a, x, r, lh, lw, slot_job);
}

template <int CIN, int NB, int S>
__global__ void __launch_bounds__(Up2Cfg<CIN, NB, S>::NWARPS * 32, 1)
    k_uptail2(const __grid_constant__ CUtensorMap tm_in, const __grid_constant__ CUtensorMap tm_lr, const ConvArgs a) {
    using Cfg = Up2Cfg<CIN, NB, S>;
    constexpr int NS = Cfg::NS, NL = Cfg::NL, BPT = Cfg::BPT;
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t *s_w = smem;
    const float *s_bias = reinterpret_cast<const float *>(smem + Cfg::B_BYTES);
    uint8_t *s_tile = smem + Cfg::W_REGION;
    uint64_t *bars = reinterpret_cast<uint64_t *>(s_tile + 2 * Cfg::TILE_BYTES);
    uint32_t *s_tmem = reinterpret_cast<uint32_t *>(bars + Cfg::NBAR);
    auto islot = [&](int k, int i) { return s_tile + k * Cfg::TILE_BYTES + i * Cfg::SLOT; };
    auto lslot = [&](int k, int i) { return s_tile + k * Cfg::TILE_BYTES + NS * Cfg::SLOT + i * Cfg::LSLOT; };
    // per tile: hfull[NS], sfree[NS], mdone[2], edone, lfull[NL], lfree[NL]
    auto hfull = [&](int k, int i) { return &bars[k * BPT + i]; };
    auto sfree = [&](int k, int i) { return &bars[k * BPT + NS + i]; };
    auto mdone = [&](int k, int par) { return &bars[k * BPT + 2 * NS + par]; };
    auto edone = [&](int k) { return &bars[k * BPT + 2 * NS + 2]; };
    auto lfull = [&](int k, int i) { return &bars[k * BPT + 2 * NS + 3 + i]; };
    auto lfree = [&](int k, int i) { return &bars[k * BPT + 2 * NS + 3 + NL + i]; };
    uint64_t *wbar = &bars[2 * BPT];

    const int slot_job = blockIdx.z;
    const int job = a.j0 + slot_job;
    if (a.job_count && job >= *a.job_count) return;
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int y0 = blockIdx.y * a.rows_per_cta;
    const int y1 = min(y0 + a.rows_per_cta, a.H);
    const int nq = y1 - y0 + 4;  // input rows y0-2 .. y1+1
    const int lh = a.H, lw = a.W;
    const int HH = lh * S, WW = lw * S;
    // tile k of this CTA (computed, not indexed: no local memory)
    auto x0k = [&](int k) { return (2 * (int)blockIdx.x + k) * kTile; };
    auto vk = [&](int k) { return (2 * (int)blockIdx.x + k) * kTile < lw; };
    if (tid == 0) {
        for (int k = 0; k < 2; k++) {
            for (int i = 0; i < NS; i++) { mbar_init(hfull(k, i), 1); mbar_init(sfree(k, i), 1); }
            for (int i = 0; i < NL; i++) { mbar_init(lfull(k, i), 1); mbar_init(lfree(k, i), 4 * S); }
            mbar_init(mdone(k, 0), 1);
            mbar_init(mdone(k, 1), 1);
            mbar_init(edone(k), 128 * S);
        }
        mbar_init(wbar, 1);
        fence_mbar_init();
    }
    if (warp == 0) tmem_alloc(s_tmem, Cfg::TMEM_COLS);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = *s_tmem;
    if (warp >= 2 && warp < 2 + 8 * S && ((warp - 2) / 4) % S == 0) {
        // sub-row-0 group of each tile: zero its accumulator ring (the block of
        // row y0 has no earlier owner whose retirement would have zeroed it)
        const int k = (warp - 2) / 4 / S;
        const uint32_t tl = tmem + ((uint32_t)((warp % 4) * 32) << 16) + k * Cfg::TCOLS;
#pragma unroll 1
        for (int b = 0; b < 5; b++) tmem_zeroN<NB>(tl + b * NB);
        tmem_wait_st();
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();

    if (warp == 0) {
        if (lane == 0) {  // ---- TMA producer
            const SrJob J = a.jobs[job];
            prefetch_tmap(&tm_in);
            prefetch_tmap(&tm_lr);
            mbar_arrive_expect_tx(wbar, Cfg::B_BYTES + Cfg::BIAS_BYTES);
            bulk_load(s_w, J.wts + a.b_off, Cfg::B_BYTES, wbar);
            bulk_load(smem + Cfg::B_BYTES, J.wts + a.bias_off, Cfg::BIAS_BYTES, wbar);
            for (int q = 0; q < nq; q++)
                for (int k = 0; k < 2; k++) {
                    if (!vk(k)) continue;
                    const int sl = q % NS;
                    if (q >= NS) mbar_wait(sfree(k, sl), ((q / NS) - 1) & 1);
                    mbar_arrive_expect_tx(hfull(k, sl), Cfg::SLOT_BYTES);
                    tma_load_5d(islot(k, sl), &tm_in, hfull(k, sl), 0, x0k(k) - 2, 0, y0 - 2 + q, slot_job);
                    const int qv = q - 4;  // output row y0 + qv retires at this step
                    if (qv >= 0) {
                        const int ls = qv % NL;
                        if (qv >= NL) mbar_wait(lfree(k, ls), ((qv / NL) - 1) & 1);
                        mbar_arrive_expect_tx(lfull(k, ls), Cfg::LR_BYTES);
                        tma_load_4d(lslot(k, ls), &tm_lr, lfull(k, ls), x0k(k) - kLrBoxX, 0, y0 + qv - 1, slot_job);
                    }
                }
        }
    } else if (warp == 1) {
        // ---- MMA issuer (whole warp, elected lane issues), both tiles; one issuer
        // per tile measured slower
        const uint32_t idesc = idesc_bf16_f32(128, 5 * NB);
        const int kfirst = 0, klast = 1;
        mbar_wait(wbar, 0);
        for (int q = 0; q < nq; q++)
            for (int k = kfirst; k <= klast; k++) {
                if (!vk(k)) continue;
                const int sl = q % NS, yin = y0 - 2 + q;
                mbar_wait(hfull(k, sl), (q / NS) & 1);
                if (q >= 1) mbar_wait(edone(k), (q - 1) & 1);  // E(q-1) retired row yin-3 = the block of yin+2
                tc_fence_after();
                const uint64_t ad0 = smem_desc(smem_u32(islot(k, sl)), kHalo5 * 16, 128);
                const uint64_t bd0 = smem_desc(smem_u32(s_w) + (uint32_t)mod5(2 - yin) * NB * 16,
                                               Cfg::NSTRIP * NB * 16, 128);
                if (elect_one()) {
#pragma unroll
                    for (int dx = 0; dx < 5; dx++)
#pragma unroll
                        for (int kc = 0; kc < Cfg::KC; kc++)
                            umma_bf16(tmem + k * Cfg::TCOLS, ad0 + (uint64_t)((2 * kc * kHalo5 * 16 + dx * 16) >> 4),
                                      bd0 + (uint64_t)(((dx * Cfg::KC + kc) * 2 * Cfg::NSTRIP * NB * 16) >> 4), idesc,
                                      1u);
                    umma_commit(sfree(k, sl));
                    umma_commit(mdone(k, q & 1));
                }
                __syncwarp();
            }
    } else {  // ---- epilogue groups: tile k, HR sub-row g
        const int grp = (warp - 2) / 4, k = grp / S, g = grp % S;
        const int ew = warp % 4;
        const int p = ew * 32 + lane;
        const int x = x0k(k) + p;
        const uint32_t tl = tmem + ((uint32_t)(ew * 32) << 16) + k * Cfg::TCOLS;
        if (vk(k)) {
            mbar_wait(wbar, 0);
            float bh[3 * S];
#pragma unroll
            for (int i = 0; i < 3 * S; i++) bh[i] = s_bias[3 * S * g + i] + 0.5f;
            const uint32_t cbase = (uint32_t)(NB <= 16 ? 0 : 8 * ((3 * S * g) / 8));
            const int xs_hr = x0k(k) * S;
            uint8_t *const hr = (a.hr_tmp ? a.hr_tmp + (size_t)slot_job * a.hr_tmp_frame : a.jobs[job].hr) + xs_hr;
            for (int q = 0; q < nq; q++) {
                const int r = y0 - 4 + q;  // LR output row completed at this step
                mbar_wait(mdone(k, q & 1), (q >> 1) & 1);
                tc_fence_after();
                const uint32_t acc = tl + (uint32_t)(mod5(r) * NB);
                uint32_t v[UpCols<NB, S>::LW];
                tmem_ldN<UpCols<NB, S>::LW>(acc + cbase, v);
                tmem_wait_ld();
                // each group re-initialises its own 3S output columns of the retired
                // block with bias + 1/2 (the rounding term): no cross-group barrier
                // before the block is free, and no bias add below.  The first five
                // retirements read blocks zeroed at allocation and add it here.
                const bool addb = q < 5;
                tmem_st_run<3 * S>(acc + (uint32_t)(3 * S * g), bh);
                tmem_wait_st();
                tc_fence_before();
                mbar_arrive(edone(k));
                float be[3 * S];  // bias + 1/2 still to add (zero once the block started at it)
#pragma unroll
                for (int i = 0; i < 3 * S; i++) be[i] = addb ? bh[i] : 0.f;
                if (r >= y0) {
                    const int qv = r - y0, ls = qv % NL;
                    mbar_wait(lfull(k, ls), (qv / NL) & 1);
                    const uint8_t *lr = lslot(k, ls);
                    // each thread stores its s bytes per plane straight into the HR frame (a
                    // shared-memory staging row copied out in 8-B chunks behind two group
                    // barriers measured 18.4-18.6 vs 17.1-17.2 ms of sr_up per c4 step)
                    uint8_t *const so = hr + (size_t)(S * r + g) * WW;
                    const size_t cst = (size_t)HH * WW;
                    if (x < lw) {
                        if (g == 0) uptail_group_step<NB, S, 0>(v, be, s_bias, lr, r, x, x0k(k), lh, lw, a, so, cst, p, slot_job);
                        else if (S > 1 && g == 1) uptail_group_step<NB, S, (S > 1 ? 1 : 0)>(v, be, s_bias, lr, r, x, x0k(k), lh, lw, a, so, cst, p, slot_job);
                        else if (S > 2 && g == 2) uptail_group_step<NB, S, (S > 2 ? 2 : 0)>(v, be, s_bias, lr, r, x, x0k(k), lh, lw, a, so, cst, p, slot_job);
                        else if (S > 3 && g == 3) uptail_group_step<NB, S, (S > 3 ? 3 : 0)>(v, be, s_bias, lr, r, x, x0k(k), lh, lw, a, so, cst, p, slot_job);
                    }
                    __syncwarp();   // this warp's LR reads are done
                    if (lane == 0) mbar_arrive(lfree(k, ls));
                }
            }
        }
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 0) tmem_dealloc(tmem, Cfg::TMEM_COLS);
}

// ---- exact frame-border ring.  The composed conv evaluates the tail over
// u at the out-of-frame HR positions around the frame (rows -1 and H, cols -1
// and W), where the definition has zeros (tail zero padding).  For every ring
// pixel:  t = bc + sum Wc h (fp32 composed 5x5)  -  sum_{out-of-frame taps}
// W_tail u_ext,  with u_ext = the upsampler evaluated at those positions (its
// own zero padding of h applies).  Out-of-frame index: row -1: X'+1 (X' in
// -1..W), row H: (W+2) + X'+1, col -1: 2(W+2) + Y', col W: 2(W+2) + H + Y'.
__device__ __forceinline__ int ext_index(int Y, int X, int H, int W) {
    if (Y < 0) return X + 1;
    if (Y >= H) return (W + 2) + X + 1;
    if (X < 0) return 2 * (W + 2) + Y;
    return 2 * (W + 2) + H + Y;
}
__device__ __forceinline__ void ext_pos(int e, int H, int W, int &Y, int &X) {
    if (e < W + 2) { Y = -1; X = e - 1; return; }
    e -= W + 2;
    if (e < W + 2) { Y = H; X = e - 1; return; }
    e -= W + 2;
    if (e < H) { Y = e; X = -1; return; }
    Y = e - H; X = W;
}
__device__ __forceinline__ float act_at(const uint16_t *act, int y, int x, int ci, int h, int w, int C) {
    if (y < 0 || y >= h || x < 0 || x >= w) return 0.f;
    return __uint_as_float((uint32_t)act[(((size_t)y * (C / 8) + ci / 8) * w + x) * 8 + ci % 8] << 16);
}

// u_ext along the four bands.  Along a band only one kernel row (row bands:
// ky = 2 at Y = -1, ky = 0 at Y = H) or one kernel column (column bands) of the
// upsampler meets the frame, so u_ext is a 1-D 3-tap conv along the band over
// the frame's first/last h row (column):
//   u_ext[c, sp](p) = b_up + sum_{ci, t} W_up[c s^2 + i s + j][ci][ky][kx] h_line[p + t - 1][ci]
// with (i, j, ky, kx) = (s-1, sp, 2, t) | (0, sp, 0, t) | (sp, s-1, t, 2) | (sp, 0, t, 0)
// for bands row -1 | row H | col -1 | col W, p the LR coordinate along the band,
// and HR coordinate s p + sp along it.  One thread per output (c, sp) keeps its
// 3C weights in registers; the CTA stages 128 + 2 line pixels (fp32,
// channel-major) and each thread sweeps them 4 positions at a time (6 shared
// loads per 12 FMAs, all broadcasts).
template <int C, int S>
__global__ void __launch_bounds__(C * S) k_uptail_ext_u(const SrJob *jobs, int j0, const int32_t *job_count,
                                                       const uint16_t *hact, int h, int w, size_t aux_off,
                                                       float *ext) {
    constexpr int P = 128;                       // LR positions per CTA
    __shared__ __align__(16) float hs[C][P + 4];  // line pixels p0-1 .. p0+P (+ pad)
    const int slot = blockIdx.y, job = j0 + slot, band = blockIdx.z;
    if (job_count && job >= *job_count) return;
    const int H = h * S, W = w * S, next = 2 * (W + 2) + 2 * H;
    const int L = band < 2 ? w : h;              // line length (LR)
    // row bands need p = -1 .. w (HR X = -1 .. W); column bands p = 0 .. h-1
    const int pfirst = band < 2 ? -1 : 0, plast = band < 2 ? w : h - 1;
    const int p0 = pfirst + blockIdx.x * P;
    if (p0 > plast) return;
    const int tid = threadIdx.x, c = tid / S, sp = tid % S;
    int i, j;
    if (band == 0) { i = S - 1; j = sp; }
    else if (band == 1) { i = 0; j = sp; }
    else if (band == 2) { i = sp; j = S - 1; }
    else { i = sp; j = 0; }
    const float *Wup = reinterpret_cast<const float *>(jobs[job].wts + aux_off);
    const float *wrow = Wup + (size_t)(c * S * S + i * S + j) * C * 9;
    float wr[C][3];
#pragma unroll
    for (int ci = 0; ci < C; ci++)
#pragma unroll
        for (int t = 0; t < 3; t++) {
            const int ky = band == 0 ? 2 : band == 1 ? 0 : t, kx = band < 2 ? t : band == 2 ? 2 : 0;
            wr[ci][t] = wrow[ci * 9 + ky * 3 + kx];
        }
    const float bias = Wup[(size_t)S * S * C * C * 9 + c * S * S + i * S + j];
    // stage the line: element e <-> line pixel p0 - 1 + e (zero outside the frame: the upsampler's padding)
    const uint16_t *act = hact + (size_t)slot * h * (C / 8) * w * 8;
    for (int idx = tid; idx < (P + 2) * (C / 8); idx += C * S) {
        const int e = idx % (P + 2), g = idx / (P + 2), pp = p0 - 1 + e;
        float v[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        if (pp >= 0 && pp < L) {
            const int yy = band == 0 ? 0 : band == 1 ? h - 1 : pp, xx = band < 2 ? pp : band == 2 ? 0 : w - 1;
            const uint4 q = *reinterpret_cast<const uint4 *>(act + (((size_t)yy * (C / 8) + g) * w + xx) * 8);
            v[0] = bf_lo(q.x); v[1] = bf_hi(q.x); v[2] = bf_lo(q.y); v[3] = bf_hi(q.y);
            v[4] = bf_lo(q.z); v[5] = bf_hi(q.z); v[6] = bf_lo(q.w); v[7] = bf_hi(q.w);
        }
#pragma unroll
        for (int k = 0; k < 8; k++) hs[g * 8 + k][e] = v[k];
    }
    if (tid < C * 2) hs[tid / 2][P + 2 + tid % 2] = 0.f;
    __syncthreads();
    const int pos_base = band == 0 ? 1 : band == 1 ? (W + 2) + 1 : band == 2 ? 2 * (W + 2) : 2 * (W + 2) + H;
    const int zmin = band < 2 ? -1 : 0, zmax = band < 2 ? W : H - 1;
    float *dst = ext + (size_t)slot * next * C;
#pragma unroll 1
    for (int q = 0; q < P; q += 4) {
        if (p0 + q > plast) break;
        float acc[4] = {bias, bias, bias, bias};
#pragma unroll
        for (int ci = 0; ci < C; ci++) {
            const float4 a4 = *reinterpret_cast<const float4 *>(&hs[ci][q]);
            const float2 b2 = *reinterpret_cast<const float2 *>(&hs[ci][q + 4]);
            const float v[6] = {a4.x, a4.y, a4.z, a4.w, b2.x, b2.y};
#pragma unroll
            for (int k = 0; k < 4; k++)
                acc[k] = fmaf(wr[ci][0], v[k], fmaf(wr[ci][1], v[k + 1], fmaf(wr[ci][2], v[k + 2], acc[k])));
        }
#pragma unroll
        for (int k = 0; k < 4; k++) {
            const int p = p0 + q + k, Z = S * p + sp;
            if (p <= plast && Z >= zmin && Z <= zmax) dst[(size_t)(pos_base + Z) * C + c] = acc[k];
        }
    }
}

// One thread per ring pixel: t = (composed t from the uptail epilogue) minus
// the out-of-frame tail taps, then the bilinear skip, round, clamp, store.
__global__ void k_uptail_ring(const SrJob *jobs, int j0, const int32_t *job_count, int h, int w, int C, int s,
                              size_t aux_off, const float *ext, const float *ring, const uint8_t *lr8, int wp,
                              uint8_t *hr_tmp) {
    __shared__ float swt[3 * 32 * 9];  // W_tail [3][C][9]
    const int slot = blockIdx.y, job = j0 + slot;
    if (job_count && job >= *job_count) return;
    const int H = h * s, W = w * s, next = 2 * (W + 2) + 2 * H, nring = 2 * W + 2 * (H - 2);
    {
        const float *aux = reinterpret_cast<const float *>(jobs[job].wts + aux_off);
        const float *Wt = aux + (size_t)s * s * C * C * 9 + (size_t)s * s * C;
        for (int k = threadIdx.x; k < 3 * C * 9; k += blockDim.x) swt[k] = Wt[k];
        __syncthreads();
    }
    const int e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= nring) return;
    int Y, X;
    if (e < W) { Y = 0; X = e; }
    else if (e < 2 * W) { Y = H - 1; X = e - W; }
    else if (e < 2 * W + (H - 2)) { Y = 1 + (e - 2 * W); X = 0; }
    else { Y = 1 + (e - 2 * W - (H - 2)); X = W - 1; }
    const SrJob J = jobs[job];
    const float *Wt = swt;
    const float *E = ext + (size_t)slot * next * C;
    const float *tr = ring + ((size_t)slot * nring + e) * 3;
    float t[3] = {tr[0], tr[1], tr[2]};
    for (int dY = -1; dY <= 1; dY++)
        for (int dX = -1; dX <= 1; dX++) {
            const int Yn = Y + dY, Xn = X + dX;
            if (Yn >= 0 && Yn < H && Xn >= 0 && Xn < W) continue;  // in-frame: the composed value is right
            const float *u = E + (size_t)ext_index(Yn, Xn, H, W) * C;
            for (int c = 0; c < C; c++) {
                const float uc = u[c];
#pragma unroll
                for (int co = 0; co < 3; co++) t[co] -= Wt[((size_t)co * C + c) * 9 + (dY + 1) * 3 + (dX + 1)] * uc;
            }
        }
    int ya, yb, wy, xa, xb, wx;
    up_tap(Y, s, h, ya, yb, wy);
    up_tap(X, s, w, xa, xb, wx);
    // the skip taps come from the batch's u8 LR copy (k_prep_lr: the net's input
    // planes, i.e. after the 4:2:0 chroma upsample for NS_FMT_I420)
    uint8_t *const dst = hr_tmp ? hr_tmp + (size_t)slot * 3 * H * W : J.hr;
    const uint8_t *L8 = lr8 + (size_t)slot * h * 3 * wp;
    for (int c = 0; c < 3; c++) {
        auto L = [&](int yy, int xx) { return (int)L8[((size_t)yy * 3 + c) * wp + xx]; };
        const int v = (128 - wy) * ((128 - wx) * L(ya, xa) + wx * L(ya, xb)) +
                      wy * ((128 - wx) * L(yb, xa) + wx * L(yb, xb));
        const int U = (v + 8192) >> 14;
        const float o = fminf(fmaxf(floorf((float)U + t[c] + 0.5f), 0.f), 255.f);
        dst[(size_t)c * H * W + (size_t)Y * W + X] = (uint8_t)o;
    }
}

// LR u8 planar [3][h][w] -> bf16 [h][w][8], channel group 0 of the head input:
// channels 0..2 = LR - 128 (Z13), 3..7 = 0 (channels 8..15 are the zero region of
// the head's ring slots, EPI_HEAD).
// NS_FMT_I420: the input is Y [h][w], U, V [h/2][w/2]; the net takes the
// chroma planes at luma resolution, upsampled x2 with the O6 definition
// (integer bilinear, half-pixel centres, Q7 weights, one round-half-up;
// reading R10), computed here on the fly.
__device__ __forceinline__ int up2_px(const uint8_t *P, int ph, int pw, int y, int x) {
    int ya, yb, wy, xa, xb, wx;
    up_tap(y, 2, ph, ya, yb, wy);
    up_tap(x, 2, pw, xa, xb, wx);
    const int v = (128 - wy) * ((128 - wx) * P[(size_t)ya * pw + xa] + wx * P[(size_t)ya * pw + xb]) +
                  wy * ((128 - wx) * P[(size_t)yb * pw + xa] + wx * P[(size_t)yb * pw + xb]);
    return (v + 8192) >> 14;
}

// One thread per 4 consecutive LR pixels (w % 8 == 0): 4-byte loads per plane,
// four 16-B x0 stores and 4-byte lr8 stores (a thread per pixel with byte
// accesses ran at 0.5 of HBM).
__global__ void k_prep_lr(const SrJob *jobs, int j0, const int32_t *job_count, int h, int w, uint16_t *x0,
                          uint8_t *lr8, int wp, int fmt) {
    const int slot = blockIdx.y, job = j0 + slot;
    if (job_count && job >= *job_count) return;
    const int idx4 = blockIdx.x * blockDim.x + threadIdx.x, w4 = w / 4;
    if (idx4 >= h * w4) return;
    const int y = idx4 / w4, x = 4 * (idx4 % w4);
    const uint8_t *L = jobs[job].lr;
    const size_t plane = (size_t)h * w, idx = (size_t)y * w + x;
    uint32_t q[3];
    q[0] = __ldg(reinterpret_cast<const unsigned int *>(L + idx));
    if (fmt == NS_FMT_I420) {
#pragma unroll
        for (int c = 1; c < 3; c++) {
            const uint8_t *P = L + plane + (size_t)(c - 1) * (plane / 4);
            q[c] = 0;
#pragma unroll
            for (int e = 0; e < 4; e++) q[c] |= (uint32_t)up2_px(P, h / 2, w / 2, y, x + e) << (8 * e);
        }
    } else {
        q[1] = __ldg(reinterpret_cast<const unsigned int *>(L + plane + idx));
        q[2] = __ldg(reinterpret_cast<const unsigned int *>(L + 2 * plane + idx));
    }
    uint4 *o = reinterpret_cast<uint4 *>(x0 + (((size_t)slot * h + y) * w + x) * 8);   // channel group 0 only
#pragma unroll
    for (int e = 0; e < 4; e++) {
        const float p0 = (float)((q[0] >> (8 * e)) & 255), p1 = (float)((q[1] >> (8 * e)) & 255),
                    p2 = (float)((q[2] >> (8 * e)) & 255);
        o[e] = make_uint4(pack_bf16(p0 - 128.f, p1 - 128.f), pack_bf16(p2 - 128.f, 0.f), 0u, 0u);
    }
    uint8_t *l8 = lr8 + ((size_t)slot * h + y) * 3 * wp + x;
#pragma unroll
    for (int c = 0; c < 3; c++) *reinterpret_cast<uint32_t *>(l8 + (size_t)c * wp) = q[c];
}

// NS_FMT_I420 output: the net's full-resolution HR [3][H][W] (hr_tmp) -> jobs[].hr
// as 4:2:0: Y as is, U and V by the rounded 2x2 average floor((a+b+c+d+2)/4)
// (reading R10).  One thread per 2x2 quad (4 Y bytes + 1 U + 1 V).
__global__ void k_pack420(const SrJob *jobs, int j0, const int32_t *job_count, int H, int W, const uint8_t *hr_tmp) {
    const int slot = blockIdx.y, job = j0 + slot;
    if (job_count && job >= *job_count) return;
    const int q = blockIdx.x * blockDim.x + threadIdx.x;
    const int QW = W / 2, QH = H / 2;
    if (q >= QW * QH) return;
    const int qy = q / QW, qx = q % QW;
    const size_t P = (size_t)H * W;
    const uint8_t *src = hr_tmp + (size_t)slot * 3 * P;
    uint8_t *dst = jobs[job].hr;
    const size_t i00 = (size_t)(2 * qy) * W + 2 * qx, i10 = i00 + W;
    *reinterpret_cast<uint16_t *>(dst + i00) = *reinterpret_cast<const uint16_t *>(src + i00);
    *reinterpret_cast<uint16_t *>(dst + i10) = *reinterpret_cast<const uint16_t *>(src + i10);
    for (int c = 1; c < 3; c++) {
        const uint8_t *S = src + c * P;
        const int v = S[i00] + S[i00 + 1] + S[i10] + S[i10 + 1] + 2;
        dst[P + (size_t)(c - 1) * (P / 4) + (size_t)qy * QW + qx] = (uint8_t)(v >> 2);
    }
}

// ------------------------------------------------------------------ host side
typedef CUresult (*PFN_encodeTiled)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                     const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                     CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static PFN_encodeTiled get_encode() {
    static PFN_encodeTiled fn = nullptr;
    if (!fn) {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_encodeTiled>(p);
    }
    return fn;
}

// Activation tensor [nb][H][C/8][W][8] bf16 viewed as 5-D (8, W, C/8, H, nb); box (8, box_w, C/8, 1, 1).
static int make_act_map(CUtensorMap *m, uint16_t *base, int H, int W, int C, int nb, int box_w) {
    PFN_encodeTiled enc = get_encode();
    if (!enc) return -1;
    cuuint64_t dims[5] = {8, (cuuint64_t)W, (cuuint64_t)(C / 8), (cuuint64_t)H, (cuuint64_t)nb};
    cuuint64_t strides[4] = {16, (cuuint64_t)W * 16, (cuuint64_t)(C / 8) * W * 16, (cuuint64_t)H * (C / 8) * W * 16};
    cuuint32_t box[5] = {8, (cuuint32_t)box_w, (cuuint32_t)(C / 8), 1, 1};
    cuuint32_t estr[5] = {1, 1, 1, 1, 1};
    CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 5, base, dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? 0 : -2;
}

// u8 LR copy [job][H][3][wp]: box of kLrBoxW px x 3 planes x 3 rows of one job
static int make_lr8_map(CUtensorMap *m, uint8_t *base, int H, int wp, int nb) {
    PFN_encodeTiled enc = get_encode();
    if (!enc) return -1;
    cuuint64_t dims[4] = {(cuuint64_t)wp, 3, (cuuint64_t)H, (cuuint64_t)nb};
    cuuint64_t strides[3] = {(cuuint64_t)wp, (cuuint64_t)wp * 3, (cuuint64_t)wp * 3 * H};
    cuuint32_t box[4] = {kLrBoxW, 3, 3, 1};
    cuuint32_t estr[4] = {1, 1, 1, 1};
    CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, base, dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                     CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? 0 : -2;
}

static size_t band_floats(int h, int w, int C, int s) {  // out-of-frame u positions x C + ring t x 3
    const size_t H = (size_t)h * s, W = (size_t)w * s;
    return (2 * (W + 2) + 2 * H) * C + (2 * W + 2 * (H - 2)) * 3;
}

size_t sr_arena_bytes(int h, int w, int C, int s, int nb, int fmt) {
    const size_t px = (size_t)h * w * nb;
    size_t b = px * 8 * 2;                   // x0 (channel group 0 of the head input)
    b += 3 * px * C * 2;                     // h0, hb, tb
    b += band_floats(h, w, C, s) * 4 * nb;   // border bands
    b += (size_t)h * 3 * ((w + 15) / 16 * 16) * nb;  // lr8
    if (fmt == NS_FMT_I420) b += (size_t)3 * s * s * px;  // hr_tmp
    return b + 7 * 256;
}

int sr_arena_init(SrArena *a, int h, int w, int C, int s, int nb, int fmt, uint8_t *mem) {
    a->h = h; a->w = w; a->C = C; a->s = s; a->nb = nb; a->fmt = fmt;
    const size_t px = (size_t)h * w * nb;
    auto take = [&](size_t bytes) {
        uint8_t *p = mem;
        mem += (bytes + 255) / 256 * 256;
        return p;
    };
    a->x0 = reinterpret_cast<uint16_t *>(take(px * 8 * 2));
    a->h0 = reinterpret_cast<uint16_t *>(take(px * C * 2));
    a->hb = reinterpret_cast<uint16_t *>(take(px * C * 2));
    a->tb = reinterpret_cast<uint16_t *>(take(px * C * 2));
    a->band = reinterpret_cast<float *>(take(band_floats(h, w, C, s) * 4 * nb));
    a->wp = (w + 15) / 16 * 16;
    a->lr8 = take((size_t)h * 3 * a->wp * nb);
    a->hr_tmp = fmt == NS_FMT_I420 ? take((size_t)3 * s * s * px) : nullptr;
    int rc = 0;
    rc |= make_lr8_map(&a->tm_lr8, a->lr8, h, a->wp, nb);
    rc |= make_act_map(&a->tm_x0, a->x0, h, w, 8, nb, kHalo);
    rc |= make_act_map(&a->tm_h0, a->h0, h, w, C, nb, kHalo);
    rc |= make_act_map(&a->tm_hb, a->hb, h, w, C, nb, kHalo);
    rc |= make_act_map(&a->tm_tb, a->tb, h, w, C, nb, kHalo);
    rc |= make_act_map(&a->tm_tb5, a->tb, h, w, C, nb, kHalo5);
    rc |= make_act_map(&a->tm_hb5, a->hb, h, w, C, nb, kHalo5);
    return rc;
}

// (A/B: 64 -> 120 rows 198.8 -> 197.5 ms per c4 step; 120 -> 180 191.9 -> 190.2; 360 no better)
constexpr int kRotRows = 180;  // rows per CTA strip of the rotated conv and uptail2
template <int CIN, int NB, int EPI>
static cudaError_t conv_rot(int fam, const CUtensorMap &tm, ConvArgs args, int nj, cudaStream_t st) {
    using Cfg = RotCfg<CIN, NB>;
    if (cudaError_t e = ensure_kernel_smem<k_conv_rot<CIN, NB, EPI>>(Cfg::SMEM, 100); e != cudaSuccess) return e;
    args.n_xtiles = (args.W + kTile - 1) / kTile;
    args.rows_per_cta = kRotRows;
    dim3 grid(args.n_xtiles, (args.H + kRotRows - 1) / kRotRows, nj);
    KScope ks(fam, st);
    constexpr int threads = 128;
    k_conv_rot<CIN, NB, EPI><<<grid, threads, Cfg::SMEM, st>>>(tm, args);
    return cudaGetLastError();
}

template <int CIN, int NB, int S>
static cudaError_t uptail(const CUtensorMap &tm, ConvArgs args, int nj, cudaStream_t st) {
    using Cfg = UpCfg<CIN, NB, S>;
    if (cudaError_t e = ensure_kernel_smem<k_uptail<CIN, NB, S>>(Cfg::SMEM); e != cudaSuccess) return e;
    args.n_xtiles = (args.W + kTile - 1) / kTile;
    args.rows_per_cta = kRotRows;
    dim3 grid(args.n_xtiles, (args.H + kRotRows - 1) / kRotRows, nj);
    KScope ks(F_SR_UP, st);
    k_uptail<CIN, NB, S><<<grid, 128, Cfg::SMEM, st>>>(tm, args);
    return cudaGetLastError();
}

// Taller strips = fewer halo rows and prologues per CTA; with the two SR streams
// overlapping each batch's last partial wave, the wave count per launch matters
// less.  A/B (ms per c4 step, same box): 120 -> 240 rows 198.8 -> 196.2; 240 ->
// 360 191.9 -> 190.8 (within noise); 720 no better.  240 rows = 3 strips =
// 288 CTAs per 16-job launch, 1.95 waves of 148 SMs, so a launch that runs
// alone (no overlap) wastes little as well: 240.
constexpr int kRbRows = 240;  // rows per CTA strip of the fused res-block

// Jobs (anchors) per SR batch of one frame shape: about two waves of the fused
// residual block, the dominant SR kernel (one CTA per SM; ceil(h / kRbRows)
// strips x ceil(tiles / 2) CTAs per job) -- 16 at 720p (18 CTAs per job, 288
// per launch on 148 SMs), 49 at 360p (6 per job) instead of a fixed 16, whose
// 96-CTA launches left a third of the GPU idle on c5's 360p half -- clamped to
// [16, 64] (arena memory).
int sr_batch_jobs(int h, int w, int sms) {
    const int per_job = ((h + kRbRows - 1) / kRbRows) * ((((w + kRbOut - 1) / kRbOut) + 1) / 2);
    return std::min(64, std::max(16, 2 * sms / std::max(per_job, 1)));
}
template <int C>
static cudaError_t resblock(const CUtensorMap &tm, const RbArgs &args0, int nj, cudaStream_t st) {
    using Cfg = RbCfg<C>;
    if (cudaError_t e = ensure_kernel_smem<k_resblock<C>>(Cfg::SMEM); e != cudaSuccess) return e;
    RbArgs args = args0;
    args.n_tiles = (args.W + kRbOut - 1) / kRbOut;
    args.rows_per_cta = kRbRows;
    dim3 grid((args.n_tiles + 1) / 2, (args.H + kRbRows - 1) / kRbRows, nj);
    KScope ks(F_SR_BODY, st);
    k_resblock<C><<<grid, kRbThreads, Cfg::SMEM, st>>>(tm, args);
    return cudaGetLastError();
}

template <int CIN, int NB, int S>
static cudaError_t uptail2(const CUtensorMap &tm, const CUtensorMap &tm_lr, ConvArgs args, int nj, cudaStream_t st) {
    using Cfg = Up2Cfg<CIN, NB, S>;
    if (cudaError_t e = ensure_kernel_smem<k_uptail2<CIN, NB, S>>(Cfg::SMEM); e != cudaSuccess) return e;
    const int ntiles = (args.W + kTile - 1) / kTile;
    args.rows_per_cta = kRotRows;
    dim3 grid((ntiles + 1) / 2, (args.H + kRotRows - 1) / kRotRows, nj);
    KScope ks(F_SR_UP, st);
    k_uptail2<CIN, NB, S><<<grid, Cfg::NWARPS * 32, Cfg::SMEM, st>>>(tm, tm_lr, args);
    return cudaGetLastError();
}

template <int C>
static cudaError_t run_net(const SrArena *a, int n_blocks, const SrJob *jobs, int j0, int nj,
                           const int32_t *job_count, cudaStream_t st) {
    const int h = a->h, w = a->w, s = a->s;
    cudaError_t e;
    {
        dim3 g((h * (w / 4) + 255) / 256, nj);
        KScope ks(F_SR_PREP, st);
        k_prep_lr<<<g, 256, 0, st>>>(jobs, j0, job_count, h, w, a->x0, a->lr8, a->wp, a->fmt);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
    ConvArgs base{};
    base.H = h; base.W = w; base.j0 = j0; base.jobs = jobs; base.job_count = job_count; base.C = C; base.s = s;
    base.hr_tmp = a->hr_tmp;  // NS_FMT_I420: full-resolution output, packed to 4:2:0 at the end
    base.lr8 = a->lr8;        // the u8 net-input planes (the upsampler's bilinear skip)
    base.wp = a->wp;
    base.hr_tmp_frame = (size_t)3 * h * s * w * s;
    auto L = [&](int l) { return model_layer(n_blocks, C, s, l); };
    {   // head: conv(x; W_head) -> h0
        ConvArgs g = base; LayerShape ls = L(0);
        g.b_off = ls.b_off; g.bias_off = ls.bias_off; g.out = a->h0; g.in = a->x0;
        if ((e = conv_rot<16, C, EPI_HEAD>(F_SR_HEAD, a->tm_x0, g, nj, st)) != cudaSuccess) return e;
    }
    // residual blocks, fused (conv1 + ReLU + conv2 + skip), ping-pong hb / tb
    const CUtensorMap *hin = &a->tm_h0;
    uint16_t *hcur = a->h0;
    for (int b = 0; b < n_blocks; b++) {
        uint16_t *dst = (b % 2 == 0) ? a->hb : a->tb;
        const LayerShape l1 = L(1 + 2 * b), l2 = L(2 + 2 * b);
        RbArgs r{};
        r.H = h; r.W = w; r.j0 = j0; r.jobs = jobs; r.job_count = job_count;
        r.b1_off = l1.b_off; r.bias1_off = l1.bias_off; r.b2_off = l2.b_off; r.bias2_off = l2.bias_off;
        r.out = dst;
        r.in = hcur;
        if ((e = resblock<C>(*hin, r, nj, st)) != cudaSuccess) return e;
        hin = (dst == a->hb) ? &a->tm_hb : &a->tm_tb;
        hcur = dst;
    }
    // end: h0 + conv(h; W_end) -> the other buffer (read next by the 5x5 conv)
    uint16_t *endout = (hcur == a->hb) ? a->tb : a->hb;
    const CUtensorMap &tm5 = (endout == a->tb) ? a->tm_tb5 : a->tm_hb5;
    {
        ConvArgs g = base; LayerShape ls = L(2 * n_blocks + 1);
        g.b_off = ls.b_off; g.bias_off = ls.bias_off; g.out = endout; g.resid = a->h0; g.in = hcur;
        if ((e = conv_rot<C, C, EPI_RESID>(F_SR_END, *hin, g, nj, st)) != cudaSuccess) return e;
    }
    {   // tail o shuffle o upsampler as one 5x5 conv at LR (+ bilinear skip, round, clamp) -> u8 HR
        const CompShape cs = model_comp(n_blocks, C, s);
        ConvArgs g = base;
        g.b_off = cs.b_off; g.bias_off = cs.bias_off; g.in = endout;
        {
            const size_t H = (size_t)h * s, W = (size_t)w * s;
            g.ring = a->band + (size_t)a->nb * (2 * (W + 2) + 2 * H) * C;
        }
        if (s == 2) e = uptail2<C, 16, 2>(tm5, a->tm_lr8, g, nj, st);
        else if (s == 3) e = uptail2<C, 32, 3>(tm5, a->tm_lr8, g, nj, st);
        else e = uptail<C, 48, 4>(tm5, g, nj, st);
        if (e != cudaSuccess) return e;
        // exact frame-border ring (the tail's zero padding of u)
        KScope ks(F_SR_TAIL, st, 2);
        const int H = h * s, W = w * s, next = 2 * (W + 2) + 2 * H, nring = 2 * W + 2 * (H - 2);
        dim3 g1((std::max(w + 2, h) + 127) / 128, nj, 4), g2((nring + 127) / 128, nj);
        if (s == 2) k_uptail_ext_u<C, 2><<<g1, C * 2, 0, st>>>(jobs, j0, job_count, endout, h, w, cs.aux_off, a->band);
        else if (s == 3) k_uptail_ext_u<C, 3><<<g1, C * 3, 0, st>>>(jobs, j0, job_count, endout, h, w, cs.aux_off, a->band);
        else k_uptail_ext_u<C, 4><<<g1, C * 4, 0, st>>>(jobs, j0, job_count, endout, h, w, cs.aux_off, a->band);
        k_uptail_ring<<<g2, 128, 0, st>>>(jobs, j0, job_count, h, w, C, s, cs.aux_off, a->band,
                                          a->band + (size_t)a->nb * next * C, a->lr8, a->wp, a->hr_tmp);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
    if (a->fmt == NS_FMT_I420) {  // full-resolution HR -> 4:2:0 (reading R10)
        KScope ks(F_SR_TAIL, st);
        const int H = h * s, W = w * s;
        dim3 g((H / 2 * (W / 2) + 255) / 256, nj);
        k_pack420<<<g, 256, 0, st>>>(jobs, j0, job_count, H, W, a->hr_tmp);
        if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
    return cudaSuccess;
}

cudaError_t sr_run_batch(const SrArena *a, int n_blocks, const SrJob *jobs, int j0, int nj,
                         const int32_t *job_count, cudaStream_t st) {
    if (a->C == 32) return run_net<32>(a, n_blocks, jobs, j0, nj, job_count, st);
    return run_net<16>(a, n_blocks, jobs, j0, nj, job_count, st);
}

}  // namespace ns

#ifdef NS_TRACE
extern "C" NS_API int ns_trace_read(unsigned long long *out, int max_pairs) {
    const int n = max_pairs < 16 * 1024 ? max_pairs : 16 * 1024;
    cudaMemcpyFromSymbol(out, ns::g_trace, sizeof(unsigned long long) * 2 * n);
    return n;
}
extern "C" NS_API void ns_trace_reset() {
    static unsigned long long z[16 * 2 * 1024];
    cudaMemcpyToSymbol(ns::g_trace, z, sizeof(z));
}
#endif
