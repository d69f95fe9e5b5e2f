// k_recon.cu -- reuse-based reconstruction of non-anchor frames (K9; PAPER.md
// §2 P:89-91 and §6.1), chunk-end reference state, per-stream stats
// (K10) and the model weight repack (model pre-optimisation, §6.2).
#include <cstdint>
#include "ns_internal.h"
#include "ptx.cuh"

namespace ns {

// O6 tap (half-pixel centres, Q7 weight of the right tap, edge clamp).
__device__ __forceinline__ void up_tap_r(int X, int s, int len, int &i0, int &i1, int &w1) {
    const int u = 2 * X + 1 - s;
    const int x0 = (u >= 0) ? u / (2 * s) : -((-u + 2 * s - 1) / (2 * s));
    const int rem = u - 2 * s * x0;
    w1 = (128 * rem + s) / (2 * s);
    i0 = min(max(x0, 0), len - 1);
    i1 = min(max(x0 + 1, 0), len - 1);
}

// gold[s][f] = latest KEY/ALTREF frame < f of stream s, -1 = the incoming
// GOLDEN state; gold[s][n] = the GOLDEN after the chunk.
__global__ void k_golden_index(const StreamDesc *sd, int S, int n, int16_t *gold) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= S) return;
    const uint8_t *T = sd[s].type;
    int g = -1;
    for (int f = 0; f < n; f++) {
        gold[(size_t)s * (n + 1) + f] = (int16_t)g;
        if (T[f] == NS_KEY || T[f] == NS_ALTREF) g = f;
    }
    gold[(size_t)s * (n + 1) + n] = (int16_t)g;
}

cudaError_t launch_golden_index(const StreamDesc *d_sd, int S, int n, int16_t *gold_idx, cudaStream_t st) {
    KScope ks(F_RECON, st);
    k_golden_index<<<(S + 127) / 128, 128, 0, st>>>(d_sd, S, n, gold_idx);
    return cudaGetLastError();
}

// One frame step f for all streams (K9).  A thread owns one LR block column
// (8s HR pixels wide, the motion vector is uniform there) x 8 HR rows x 3
// planes:  anchor -> skip (SR output already in place); KEY frame or INTRA
// block -> up_s(LR[f]); otherwise clamp(warp_{s*mv}(HR[ref]) + up_s(res[f])).
// The warp (O7) runs two pixels per 32-bit register (16-bit lanes; every
// intermediate < 2^16): each horizontal pass over a reference row is shared by
// the two output rows that use it.  up_s (O6) is separable with compile-time
// taps (the thread's first pixel is a multiple of s).  Reference windows are
// read with aligned 64-bit loads (edge blocks fall back to clamped byte loads).
template <int S>
struct ReconCfg {
    static constexpr int BW = 8 * S;               // HR pixels per thread row
    static constexpr int NP = BW / 2;              // 16-bit pairs per row
    static constexpr int WIN = BW + 1;             // reference bytes per row
    static constexpr int NQ = (7 + WIN + 7) / 8;   // aligned 64-bit words per row
    static constexpr int NA32 = (WIN + 3) / 4;     // aligned 32-bit window words
    static constexpr int RPT = (S == 3) ? 6 : 8;   // HR rows per thread: a multiple of S
                                                   // or of 8s/.. so that Y0 mod S == 0
    // resident CTAs per SM: s = 3 fits 128 registers without spills and its
    // 56 KB of staging exactly fills 4 CTAs' worth of shared memory (latency-
    // bound kernel: occupancy 3 -> 4 CTAs); s = 2, 4 would spill at 128
    static constexpr int MINB = (S == 3) ? 4 : 3;
};

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel) {
    uint32_t r;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
    return r;
}

// Stage the raw aligned 64-bit words covering reference bytes xs .. xs+BW of
// one row into shared memory: dst[i * stride] is word i (struct-of-arrays
// across the CTA's threads: conflict-free reads).  W and the word base are
// multiples of 8, so every word lies wholly inside the row (cp.async) or wholly
// outside it, where edge replication (Z16) makes it 8 copies of the first or
// last pixel: no byte-wise clamped loads, and no read past the row end.
template <int S>
__device__ __forceinline__ void recon_row_stage(const uint8_t *row, int xs, int W, bool interior, uint2 *dst,
                                                int stride) {
    using Cfg = ReconCfg<S>;
    const int xb = xs & ~7;
    if (interior) {
#pragma unroll
        for (int i = 0; i < Cfg::NQ; i++)
            asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst + i * stride)),
                         "l"(row + xb + 8 * i)
                         : "memory");
    } else {
#pragma unroll
        for (int i = 0; i < Cfg::NQ; i++) {
            const int st = xb + 8 * i;
            if (st >= 0 && st < W) {
                asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst + i * stride)),
                             "l"(row + st)
                             : "memory");
            } else {
                const uint32_t v = 0x01010101u * row[st < 0 ? 0 : W - 1];
                dst[i * stride] = make_uint2(v, v);
            }
        }
    }
}

// Horizontal bilinear pass over one reference row: h[k] = packed pixels
// (2k, 2k+1) of (R[x](8-fx) + R[x+1]fx + 4) >> 3 for x = xs .. xs+BW-1.
template <int S>
__device__ __forceinline__ void recon_hpass(const uint2 (&q)[ReconCfg<S>::NQ], int xs, uint32_t fxc, uint32_t fx,
                                            uint32_t (&h)[ReconCfg<S>::NP]) {
    using Cfg = ReconCfg<S>;
    uint32_t w[2 * Cfg::NQ + 2];
#pragma unroll
    for (int i = 0; i < Cfg::NQ; i++) {
        w[2 * i] = q[i].x;
        w[2 * i + 1] = q[i].y;
    }
    w[2 * Cfg::NQ] = 0;
    w[2 * Cfg::NQ + 1] = 0;
    const int m = xs & 7;
    if (m >= 4) {
#pragma unroll
        for (int i = 0; i < 2 * Cfg::NQ + 1; i++) w[i] = w[i + 1];
    }
    const uint32_t sh = 8u * (uint32_t)(m & 3);
    uint32_t A[Cfg::NP + 2];
#pragma unroll
    for (int i = 0; i < Cfg::NA32; i++) {
        const uint32_t a = __funnelshift_r(w[i], w[i + 1], sh);
        A[2 * i] = prmt(a, 0u, 0x4140u);
        if (2 * i + 1 < Cfg::NP + 2) A[2 * i + 1] = prmt(a, 0u, 0x4342u);
    }
#pragma unroll
    for (int k = 0; k < Cfg::NP; k++) {
        const uint32_t B = __funnelshift_r(A[k], A[k + 1], 16);
        h[k] = ((A[k] * fxc + B * fx + 0x00040004u) >> 3) & 0x1FFF1FFFu;
    }
}

// Raw LR-row data for columns 8bx-1 .. 8bx+8: the aligned middle 8 values
// (16 B of int16 or 8 B of u8, zero-extended) plus the two clamped edges.
struct LrRaw {
    uint4 mid;
    int left, right;
};
__device__ __forceinline__ void recon_lr_load(const void *plane, bool is_u8, int row, int bx, int w, LrRaw &r) {
    if (is_u8) {
        const uint8_t *p = static_cast<const uint8_t *>(plane) + (size_t)row * w;
        const uint2 q = __ldg(reinterpret_cast<const uint2 *>(p + 8 * bx));
        r.mid = make_uint4(q.x, q.y, 0, 0);
        r.left = p[max(8 * bx - 1, 0)];
        r.right = p[min(8 * bx + 8, w - 1)];
    } else {
        const int16_t *p = static_cast<const int16_t *>(plane) + (size_t)row * w;
        r.mid = __ldg(reinterpret_cast<const uint4 *>(p + 8 * bx));
        r.left = p[max(8 * bx - 1, 0)];
        r.right = p[min(8 * bx + 8, w - 1)];
    }
}
__device__ __forceinline__ void recon_lr_unpack(const LrRaw &r, bool is_u8, int (&v)[10]) {
    v[0] = r.left;
    v[9] = r.right;
    if (is_u8) {
#pragma unroll
        for (int i = 0; i < 4; i++) {
            v[1 + i] = (r.mid.x >> (8 * i)) & 255;
            v[5 + i] = (r.mid.y >> (8 * i)) & 255;
        }
    } else {
        const uint32_t qq[4] = {r.mid.x, r.mid.y, r.mid.z, r.mid.w};
#pragma unroll
        for (int i = 0; i < 4; i++) {
            v[1 + 2 * i] = (int)(int16_t)(qq[i] & 0xFFFFu);
            v[2 + 2 * i] = (int)(int16_t)(qq[i] >> 16);
        }
    }
}

constexpr int kReconTX = 32, kReconTY = 4;

__device__ __forceinline__ uint32_t vmax_u16x2(uint32_t a, uint32_t b) {
    uint32_t r;
    asm("max.u16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
    return r;
}
__device__ __forceinline__ uint32_t vmin_u16x2(uint32_t a, uint32_t b) {
    uint32_t r;
    asm("min.u16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
    return r;
}

// Compile-time O6 taps.  For an axis coordinate X = S*m + ph + i:
//   u = 2X + 1 - S, x0 = m + floor((2(ph+i) + 1 - S) / 2S), w1 = round(128 rem / 2S).
__host__ __device__ constexpr int fdiv(int a, int b) { return a >= 0 ? a / b : -((-a + b - 1) / b); }
template <int S>
__host__ __device__ constexpr int tap_d(int k) { return fdiv(2 * k + 1 - S, 2 * S); }
template <int S>
__host__ __device__ constexpr int tap_w1(int k) { return (128 * ((2 * k + 1 - S) - 2 * S * tap_d<S>(k)) + S) / (2 * S); }

// All three planes of one thread's 8s x 8 tile; PH = Y0 mod S (compile time).
template <int S>
__device__ __forceinline__ void recon_planes(const StreamDesc &d, bool use_lr, const uint8_t *ref, const uint8_t *lr_f,
                                             const int16_t *res_f, uint8_t *out, size_t lrp, size_t hrp, int H, int W,
                                             int bx, int X0, int Y0, int Y0m, int xs, int iy0, bool interior,
                                             uint32_t fxc, uint32_t fxp, uint32_t fyc, uint32_t fyp) {
    using Cfg = ReconCfg<S>;
    constexpr int BW = Cfg::BW, NP = Cfg::NP;
    constexpr int RPT = Cfg::RPT;
    constexpr int DMIN = tap_d<S>(0), DMAX = tap_d<S>(S - 1) + 1;
    constexpr int NLR = DMAX - DMIN + 1 + (RPT / S - 1);  // LR rows: one period's window + slides
    static_assert(RPT % S == 0, "row groups are whole periods");
    constexpr int NT = kReconTX * kReconTY;
    extern __shared__ __align__(16) uint2 rsm[];  // [2 planes][9 rows][NQ words][NT threads]
    const int tid = threadIdx.y * kReconTX + threadIdx.x;
    auto stage = [&](int c) {
        if (use_lr) return;
        const uint8_t *P = ref + c * hrp;
        uint2 *buf = rsm + (size_t)(c & 1) * (RPT + 1) * Cfg::NQ * NT + tid;
#pragma unroll
        for (int j = 0; j <= RPT; j++) {
            const int r = min(max(iy0 + j, 0), H - 1);
            recon_row_stage<S>(P + (size_t)r * W, xs, W, interior, buf + j * Cfg::NQ * NT, NT);
        }
    };
    stage(0);
    asm volatile("cp.async.commit_group;" ::: "memory");
#pragma unroll 1
    for (int c = 0; c < 3; c++) {
        if (c + 1 < 3) stage(c + 1);
        asm volatile("cp.async.commit_group;" ::: "memory");
        const void *src = use_lr ? static_cast<const void *>(lr_f + c * lrp) : static_cast<const void *>(res_f + c * lrp);
        int lv[NLR][10];
#pragma unroll
        for (int t = 0; t < NLR; t++) {
            LrRaw raw;
            recon_lr_load(src, use_lr, min(max(Y0m + DMIN + t, 0), d.h - 1), bx, d.w, raw);
            recon_lr_unpack(raw, use_lr, lv[t]);
        }
        asm volatile("cp.async.wait_group 1;" ::: "memory");  // this plane's windows have landed
        const uint2 *buf = rsm + (size_t)(c & 1) * (RPT + 1) * Cfg::NQ * NT + tid;
        auto row = [&](int j, uint2 (&q)[Cfg::NQ]) {
#pragma unroll
            for (int i = 0; i < Cfg::NQ; i++) q[i] = buf[(j * Cfg::NQ + i) * NT];
        };
        uint32_t hprev[NP], hcur[NP];
        if (!use_lr) {
            uint2 q[Cfg::NQ];
            row(0, q);
            recon_hpass<S>(q, xs, fxc, fxp, hprev);
        }
#pragma unroll 1
        for (int it = 0; it < RPT / S; it++) {
#pragma unroll
            for (int jj = 0; jj < S; jj++) {  // one period of the vertical O6 taps
                const int j = it * S + jj;
                uint32_t pred[NP];
                if (!use_lr) {
                    uint2 q[Cfg::NQ];
                    row(j + 1, q);
                    recon_hpass<S>(q, xs, fxc, fxp, hcur);
#pragma unroll
                    for (int k = 0; k < NP; k++) {
                        pred[k] = ((hprev[k] * fyc + hcur[k] * fyp + 0x00040004u) >> 3) & 0x1FFF1FFFu;
                        hprev[k] = hcur[k];
                    }
                } else {
#pragma unroll
                    for (int k = 0; k < NP; k++) pred[k] = 0;
                }
                // up_s of the residual (or LR) plane at row Y0 + j (O6), compile-time taps;
                // lv[0] holds LR row Y0/S + DMIN + it (the window slides one LR row per period)
                const int ta = tap_d<S>(jj) - DMIN;
                const int wy = tap_w1<S>(jj);
                // per LR column t: V = (128-wy) a + wy b (vertical, exact); the
                // horizontal tap of pixel i is 128 V[d] + w1 (V[d+1] - V[d]).  Scaled
                // by 4 with the rounding constant and the +256 lane bias folded in, the
                // value r + 256 lands in the high half-word: one IMAD per pixel and one
                // PRMT per pixel pair.
                int base[10], dlt[9];
#pragma unroll
                for (int t = 0; t < 10; t++) {
                    const int V = (128 - wy) * lv[ta][t] + wy * lv[ta + 1][t];
                    base[t] = V * 512 + 4 * (8192 + (256 << 14));
                }
#pragma unroll
                for (int t = 0; t < 9; t++) dlt[t] = base[t + 1] - base[t];
                uint32_t o[BW / 4];
#pragma unroll
                for (int qd = 0; qd < BW / 4; qd++) {
                    uint32_t pr[2];
#pragma unroll
                    for (int hh = 0; hh < 2; hh++) {
                        const int i0 = 4 * qd + 2 * hh;
                        const int d0 = tap_d<S>(i0) + 1, d1 = tap_d<S>(i0 + 1) + 1;
                        const int w0 = tap_w1<S>(i0), w1 = tap_w1<S>(i0 + 1);
                        // (base + w1 * dlt / 128): dlt is a multiple of 512, so w1*dlt/128 = w1*(dlt/128) exactly
                        const uint32_t s0 = (uint32_t)(base[d0] + (w0 ? w0 * (dlt[d0] >> 7) : 0));
                        const uint32_t s1 = (uint32_t)(base[d1] + (w1 ? w1 * (dlt[d1] >> 7) : 0));
                        uint32_t x = prmt(s0, s1, 0x7632u);  // [r0 + 256, r1 + 256]
                        x += pred[i0 >> 1];                   // in [1, 766] per lane
                        pr[hh] = vmin_u16x2(vmax_u16x2(x, 0x01000100u), 0x01FF01FFu);  // clamp to [256, 511]
                    }
                    o[qd] = prmt(pr[0], pr[1], 0x6420u);  // low bytes = clamped value (x - 256)
                }
                uint2 *dst = reinterpret_cast<uint2 *>(out + c * hrp + (size_t)(Y0 + j) * W + X0);
#pragma unroll
                for (int qd = 0; qd < BW / 8; qd++) dst[qd] = make_uint2(o[2 * qd], o[2 * qd + 1]);
            }
#pragma unroll
            for (int t = 0; t + 1 < NLR; t++)
#pragma unroll
                for (int e = 0; e < 10; e++) lv[t][e] = lv[t + 1][e];
        }
    }
}

template <int S>
__global__ void __launch_bounds__(kReconTX *kReconTY, ReconCfg<S>::MINB)
    k_recon_step(const StreamDesc *sd, int n, int f, const uint8_t *is_anchor, uint8_t *const *hr_tab,
                 const int16_t *gold) {
    using Cfg = ReconCfg<S>;
    constexpr int BW = Cfg::BW, NP = Cfg::NP;
    const int sid = blockIdx.z;
    if (is_anchor[(size_t)sid * n + f]) return;
    const StreamDesc d = sd[sid];
    if (d.s != S) return;
    const int H = d.h * S, W = d.w * S;
    const int bx = blockIdx.x * kReconTX + threadIdx.x;  // LR block column
    const int rg = blockIdx.y * kReconTY + threadIdx.y;  // group of RPT HR rows
    const int X0 = bx * BW, Y0 = rg * Cfg::RPT;
    if (X0 >= W || Y0 >= H) return;
    const int bw = d.w / 8;
    const ns_block_mv mv = d.mv[(size_t)f * (d.h / 8) * bw + (size_t)(Y0 / BW) * bw + bx];
    const bool key = d.type[f] == NS_KEY;
    const bool use_lr = key || mv.ref == NS_REF_INTRA;
    uint8_t *out = hr_tab[d.hr_base + f];
    const size_t lrp = (size_t)d.h * d.w, hrp = (size_t)H * W;
    const uint8_t *ref = nullptr;
    if (!use_lr) {
        if (mv.ref == NS_REF_GOLDEN) {
            const int g = gold[(size_t)sid * (n + 1) + f];
            ref = g >= 0 ? hr_tab[d.hr_base + g] : d.hr_golden;
        } else {
            ref = f > 0 ? hr_tab[d.hr_base + f - 1] : d.hr_last;
        }
    }
    // warp geometry (O7): m = s * mv in 1/8 HR pel
    const int mx = S * mv.mvx, my = S * mv.mvy;
    const int xs = X0 + (mx >> 3);
    const uint32_t fx = (uint32_t)(mx & 7), fy = (uint32_t)(my & 7);
    // packed 2 x 16-bit arithmetic multiplies by a SCALAR (no cross-lane terms)
    const uint32_t fxp = fx, fyp = fy, fxc = 8u - fx, fyc = 8u - fy;
    const int iy0 = Y0 + (my >> 3);
    // every aligned word of the window inside the row -> unconditional cp.async
    const bool interior = xs >= 0 && (xs & ~7) + 8 * Cfg::NQ <= W;
    const uint8_t *lr_f = d.lr + (size_t)f * 3 * lrp;
    const int16_t *res_f = d.res + (size_t)f * 3 * lrp;

    recon_planes<S>(d, use_lr, ref, lr_f, res_f, out, lrp, hrp, H, W, bx, X0, Y0, Y0 / S, xs, iy0, interior, fxc,
                    fxp, fyc, fyp);
}

template <int S>
static size_t recon_smem() {
    return (size_t)2 * (ReconCfg<S>::RPT + 1) * ReconCfg<S>::NQ * kReconTX * kReconTY * sizeof(uint2);
}

template <int S>
static void recon_launch(dim3 g, cudaStream_t st, const StreamDesc *d_sd, int n, int f, const uint8_t *is_anchor,
                         uint8_t *const *hr, const int16_t *gold) {
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(k_recon_step<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)recon_smem<S>());
        // all of the unified L1/shared array as shared memory, so MINB CTAs fit
        cudaFuncSetAttribute(k_recon_step<S>, cudaFuncAttributePreferredSharedMemoryCarveout,
                             (int)cudaSharedmemCarveoutMaxShared);
        attr = true;
    }
    k_recon_step<S><<<g, dim3(kReconTX, kReconTY), recon_smem<S>(), st>>>(d_sd, n, f, is_anchor, hr, gold);
}

cudaError_t launch_recon_step(const StreamDesc *d_sd, int S, int n, int f, const int *max_lr_w,
                              const int *max_lr_h, const uint8_t *is_anchor, uint8_t *const *d_hr_table,
                              const int16_t *gold_idx, cudaStream_t st) {
    int nl = 0;
    for (int s = 2; s <= 4; s++) nl += max_lr_w[s] > 0;
    KScope ks(F_RECON, st, nl);
    for (int s = 2; s <= 4; s++) {
        if (max_lr_w[s] <= 0) continue;
        const int nbx = max_lr_w[s] / 8;          // LR block columns
        const int nrg = max_lr_h[s] * s / (s == 3 ? 6 : 8);  // groups of RPT HR rows
        dim3 g((nbx + kReconTX - 1) / kReconTX, (nrg + kReconTY - 1) / kReconTY, S);
        dim3 b(kReconTX, kReconTY);
        (void)b;
        if (s == 2) recon_launch<2>(g, st, d_sd, n, f, is_anchor, d_hr_table, gold_idx);
        if (s == 3) recon_launch<3>(g, st, d_sd, n, f, is_anchor, d_hr_table, gold_idx);
        if (s == 4) recon_launch<4>(g, st, d_sd, n, f, is_anchor, d_hr_table, gold_idx);
    }
    return cudaGetLastError();
}

// Chunk-end reference state: hr_last <- HR[n-1], hr_golden <- HR[gold[n]].
__global__ void k_state_copy(const StreamDesc *sd, int n, uint8_t *const *hr_tab, const int16_t *gold) {
    const int sid = blockIdx.y, which = blockIdx.z;
    const StreamDesc d = sd[sid];
    const size_t nvec = (size_t)3 * d.h * d.s * d.w * d.s / 16;
    uint8_t *dst;
    const uint8_t *src;
    if (which == 0) {
        dst = d.hr_last;
        src = hr_tab[d.hr_base + n - 1];
    } else {
        const int g = gold[(size_t)sid * (n + 1) + n];
        dst = d.hr_golden;
        src = g >= 0 ? hr_tab[d.hr_base + g] : nullptr;
    }
    if (!dst || !src || dst == src) return;
    const uint4 *s4 = reinterpret_cast<const uint4 *>(src);
    uint4 *d4 = reinterpret_cast<uint4 *>(dst);
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < nvec; i += (size_t)gridDim.x * blockDim.x)
        d4[i] = s4[i];
}

cudaError_t launch_state_copy(const StreamDesc *d_sd, int S, int n, uint8_t *const *d_hr_table,
                              const int16_t *gold_idx, size_t max_hr_bytes, cudaStream_t st) {
    const int blocks = (int)((max_hr_bytes / 16 + 255) / 256);
    KScope ks(F_STATE, st);
    dim3 g(blocks < 1 ? 1 : (blocks > 4096 ? 4096 : blocks), S, 2);
    k_state_copy<<<g, 256, 0, st>>>(d_sd, n, d_hr_table, gold_idx);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- K10 stats
// stats[s] = {frames, anchors, sum anchor score, total score, SSE vs gt, PSNR, 0, 0}
__global__ void k_stats_meta(const StreamDesc *sd, int S, int n, const uint8_t *is_anchor, const int64_t *score,
                             double *stats) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= S) return;
    double a = 0, sa = 0, st = 0;
    for (int f = 0; f < n; f++) {
        const double v = (double)score[(size_t)s * n + f];
        st += v;
        if (is_anchor[(size_t)s * n + f]) { a += 1; sa += v; }
    }
    double *o = stats + (size_t)s * 8;
    o[0] = n; o[1] = a; o[2] = sa; o[3] = st;
    o[4] = sd[s].gt ? 0.0 : -1.0;
    o[5] = -1.0; o[6] = 0; o[7] = 0;
}

__global__ void k_stats_sse(const StreamDesc *sd, int n, uint8_t *const *hr_tab, double *stats) {
    const int sf = blockIdx.y, sid = sf / n, f = sf % n;
    const StreamDesc d = sd[sid];
    if (!d.gt) return;
    const size_t nvec = (size_t)3 * d.h * d.s * d.w * d.s / 16;
    const uint4 *a = reinterpret_cast<const uint4 *>(hr_tab[d.hr_base + f]);
    const uint4 *b = reinterpret_cast<const uint4 *>(d.gt + (size_t)f * nvec * 16);
    unsigned long long acc = 0;
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < nvec; i += (size_t)gridDim.x * blockDim.x) {
        const uint4 x = a[i], y = b[i];
        const uint32_t xs[4] = {x.x, x.y, x.z, x.w}, ys[4] = {y.x, y.y, y.z, y.w};
#pragma unroll
        for (int j = 0; j < 4; j++)
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const int dd = (int)((xs[j] >> (8 * q)) & 255) - (int)((ys[j] >> (8 * q)) & 255);
                acc += (unsigned long long)(dd * dd);
            }
    }
    for (int off = 16; off; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
    if ((threadIdx.x & 31) == 0) atomicAdd(stats + (size_t)sid * 8 + 4, (double)acc);
}

__global__ void k_stats_final(const StreamDesc *sd, int S, int n, double *stats) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= S || !sd[s].gt) return;
    const double N = 3.0 * sd[s].h * sd[s].s * sd[s].w * sd[s].s * n;
    const double sse = stats[(size_t)s * 8 + 4];
    double p = sse == 0.0 ? 100.0 : 10.0 * log10(255.0 * 255.0 / (sse / N));
    stats[(size_t)s * 8 + 5] = p > 100.0 ? 100.0 : p;
}

cudaError_t launch_stats(const StreamDesc *d_sd, int S, int n, const uint8_t *is_anchor, const int64_t *score,
                         uint8_t *const *d_hr_table, size_t max_hr_bytes, double *stats, cudaStream_t st) {
    KScope ks(F_STATS, st, 3);
    k_stats_meta<<<(S + 127) / 128, 128, 0, st>>>(d_sd, S, n, is_anchor, score, stats);
    const int blocks = (int)((max_hr_bytes / 16 + 255) / 256);
    dim3 g(blocks < 1 ? 1 : (blocks > 1024 ? 1024 : blocks), S * n);
    k_stats_sse<<<g, 256, 0, st>>>(d_sd, n, d_hr_table, stats);
    k_stats_final<<<(S + 127) / 128, 128, 0, st>>>(d_sd, S, n, stats);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- weight repack
// bf16 blob (head, blocks x (conv1, conv2), end, up, tail; [Cout][Cin][3][3] +
// bias) -> per-layer UMMA B operand [split][tap][kc][kh][n][8] bf16 + fp32 bias.
__global__ void k_repack_b(const uint16_t *blob, size_t src_off, LayerShape ls, int C, int s, uint8_t *packed) {
    const size_t NT = ls.ntot / ls.nsplit;
    uint16_t *B = reinterpret_cast<uint16_t *>(packed + ls.b_off);
    if (ls.rot) {  // [dx 3][kc][kh 2][5 nb][8], strip of kernel rows dy = 2,1,0,2,1
        const int KC = ls.cin / 16, nb = ls.nb;
        const size_t total = (size_t)3 * KC * 2 * 5 * nb * 8;
        const int strip[5] = {2, 1, 0, 2, 1};
        for (size_t e = (size_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
             e += (size_t)gridDim.x * blockDim.x) {
            const int k8 = e % 8;
            const int nn = (e / 8) % (5 * nb);
            const int kh = (e / (8 * 5 * nb)) % 2;
            const int kc = (e / (16 * 5 * nb)) % KC;
            const int dx = (int)(e / ((size_t)16 * 5 * nb * KC));
            const int dy = strip[nn / nb], co = nn % nb;
            const int ci = kc * 16 + kh * 8 + k8;
            uint16_t v = 0;
            if (ci < ls.cin_real && co < ls.cout_real)
                v = blob[src_off + (((size_t)co * ls.cin_real + ci) * 3 + dy) * 3 + dx];
            B[e] = v;
        }
    } else {
    const size_t total = (size_t)9 * ls.cin * ls.ntot;
    for (size_t e = (size_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (size_t)gridDim.x * blockDim.x) {
        const int k8 = e % 8;
        const int nn = (e / 8) % NT;
        const int kh = (e / (8 * NT)) % 2;
        const int kc = (e / (16 * NT)) % (ls.cin / 16);
        const int tap = (e / ((size_t)ls.cin * NT)) % 9;
        const int sp = (int)(e / ((size_t)9 * ls.cin * NT));
        const int ci = kc * 16 + kh * 8 + k8;
        const int cop = sp * (int)NT + nn;
        uint16_t v = 0;
        if (ci < ls.cin_real && cop < ls.cout_real) {
            const int co = ls.perm ? (cop % C) * s * s + cop / C : cop;
            v = blob[src_off + (((size_t)co * ls.cin_real + ci) * 3 + tap / 3) * 3 + tap % 3];
        }
        B[e] = v;
    }
    }
    float *bias = reinterpret_cast<float *>(packed + ls.bias_off);
    for (int cop = blockIdx.x * blockDim.x + threadIdx.x; cop < ls.ntot; cop += gridDim.x * blockDim.x) {
        float v = 0.f;
        if (cop < ls.cout_real) {
            const int co = ls.perm ? (cop % C) * s * s + cop / C : cop;
            v = __uint_as_float((uint32_t)blob[src_off + (size_t)ls.cout_real * ls.cin_real * 9 + co] << 16);
        }
        bias[cop] = v;
    }
}

__device__ __forceinline__ float bf2f(uint16_t b) { return __uint_as_float((uint32_t)b << 16); }
__device__ __forceinline__ uint16_t f2bf(float f) {  // round to nearest even
    const uint32_t u = __float_as_uint(f);
    return (uint16_t)((u + 0x7FFFu + ((u >> 16) & 1u)) >> 16);
}

// Composed weights of tail o pixel-shuffle o upsampler (see CompShape): output
// n = (i s + j) 3 + co at LR offset (ty-2, tx-2) from input channel ci:
//   Wc = sum_{dY,dX in -1..1} sum_c Wt[co][c][dY][dX] Wup[c s^2 + i' s + j'][ci][ky][kx]
// with (i+dY) = s oy + i', (j+dX) = s ox + j', ky = ty - 1 - oy, kx = tx - 1 - ox.
__global__ void k_repack_comp(const uint16_t *blob, size_t up_off, size_t tail_off, int C, int s, CompShape cs,
                              uint8_t *packed) {
    const int nb = cs.nb, KC = C / 16, nout = s * s * 3, ns = cs.nstrip;
    const size_t total = (size_t)5 * KC * 2 * ns * nb * 8;
    const uint16_t *Wup = blob + up_off, *bup = blob + up_off + (size_t)s * s * C * C * 9;
    const uint16_t *Wt = blob + tail_off, *bt = blob + tail_off + (size_t)3 * C * 9;
    const int strip9[9] = {4, 3, 2, 1, 0, 4, 3, 2, 1};
    const int strip11[11] = {4, 3, 2, 1, 0, -1, 4, 3, 2, 1, 0};  // -1: zero block (6th ring slot)
    uint16_t *B = reinterpret_cast<uint16_t *>(packed + cs.b_off);
    for (size_t e = (size_t)blockIdx.x * blockDim.x + threadIdx.x; e < total; e += (size_t)gridDim.x * blockDim.x) {
        const int k8 = e % 8;
        const int nn = (e / 8) % (ns * nb);
        const int kh = (e / (8 * ns * nb)) % 2;
        const int kc = (e / (16 * ns * nb)) % KC;
        const int tx = (int)(e / ((size_t)16 * ns * nb * KC));
        const int ty = ns == 11 ? strip11[nn / nb] : strip9[nn / nb], n = nn % nb;
        if (ty < 0) { B[e] = 0; continue; }
        const int ci = kc * 16 + kh * 8 + k8;
        float acc = 0.f;
        if (n < nout) {
            const int co = n % 3, ij = n / 3, i = ij / s, j = ij % s;
            for (int dY = -1; dY <= 1; dY++)
                for (int dX = -1; dX <= 1; dX++) {
                    const int oy = (i + dY + s) / s - 1, ip = (i + dY + s) % s;
                    const int ox = (j + dX + s) / s - 1, jp = (j + dX + s) % s;
                    const int ky = ty - 1 - oy, kx = tx - 1 - ox;
                    if (ky < 0 || ky > 2 || kx < 0 || kx > 2) continue;
                    for (int c = 0; c < C; c++) {
                        const int uc = c * s * s + ip * s + jp;
                        acc += bf2f(Wt[((size_t)co * C + c) * 9 + (dY + 1) * 3 + (dX + 1)]) *
                               bf2f(Wup[((size_t)uc * C + ci) * 9 + ky * 3 + kx]);
                    }
                }
        }
        B[e] = f2bf(acc);
    }
    float *bias = reinterpret_cast<float *>(packed + cs.bias_off);
    for (int n = blockIdx.x * blockDim.x + threadIdx.x; n < nb; n += gridDim.x * blockDim.x) {
        float acc = 0.f;
        if (n < nout) {
            const int co = n % 3, ij = n / 3, i = ij / s, j = ij % s;
            acc = bf2f(bt[co]);
            for (int dY = -1; dY <= 1; dY++)
                for (int dX = -1; dX <= 1; dX++) {
                    const int ip = (i + dY + s) % s, jp = (j + dX + s) % s;
                    for (int c = 0; c < C; c++)
                        acc += bf2f(Wt[((size_t)co * C + c) * 9 + (dY + 1) * 3 + (dX + 1)]) *
                               bf2f(bup[c * s * s + ip * s + jp]);
                }
        }
        bias[n] = acc;
    }
}

// fp32 composed weights Wc[n][ci][ty*5+tx] and bias (same sums as k_repack_comp)
__global__ void k_repack_comp32(const uint16_t *blob, size_t up_off, size_t tail_off, int C, int s, float *Wc,
                                float *bc) {
    const int nout = s * s * 3;
    const uint16_t *Wup = blob + up_off, *bup = blob + up_off + (size_t)s * s * C * C * 9;
    const uint16_t *Wt = blob + tail_off, *bt = blob + tail_off + (size_t)3 * C * 9;
    const size_t total = (size_t)nout * C * 25;
    for (size_t e = (size_t)blockIdx.x * blockDim.x + threadIdx.x; e < total + nout;
         e += (size_t)gridDim.x * blockDim.x) {
        if (e < total) {
            const int tt = e % 25, ci = (e / 25) % C, n = (int)(e / (25 * C));
            const int ty = tt / 5, tx = tt % 5;
            const int co = n % 3, ij = n / 3, i = ij / s, j = ij % s;
            float acc = 0.f;
            for (int dY = -1; dY <= 1; dY++)
                for (int dX = -1; dX <= 1; dX++) {
                    const int oy = (i + dY + s) / s - 1, ip = (i + dY + s) % s;
                    const int ox = (j + dX + s) / s - 1, jp = (j + dX + s) % s;
                    const int ky = ty - 1 - oy, kx = tx - 1 - ox;
                    if (ky < 0 || ky > 2 || kx < 0 || kx > 2) continue;
                    for (int c = 0; c < C; c++)
                        acc += bf2f(Wt[((size_t)co * C + c) * 9 + (dY + 1) * 3 + (dX + 1)]) *
                               bf2f(Wup[((size_t)(c * s * s + ip * s + jp) * C + ci) * 9 + ky * 3 + kx]);
                }
            Wc[e] = acc;
        } else {
            const int n = (int)(e - total);
            const int co = n % 3, ij = n / 3, i = ij / s, j = ij % s;
            float acc = bf2f(bt[co]);
            for (int dY = -1; dY <= 1; dY++)
                for (int dX = -1; dX <= 1; dX++) {
                    const int ip = (i + dY + s) % s, jp = (j + dX + s) % s;
                    for (int c = 0; c < C; c++)
                        acc += bf2f(Wt[((size_t)co * C + c) * 9 + (dY + 1) * 3 + (dX + 1)]) *
                               bf2f(bup[c * s * s + ip * s + jp]);
                }
            bc[n] = acc;
        }
    }
}

// fp32 copies of the upsampler and tail (the border fix-up evaluates them exactly)
__global__ void k_repack_aux(const uint16_t *blob, size_t up_off, size_t n_up, size_t tail_off, size_t n_tail,
                             float *aux) {
    for (size_t e = (size_t)blockIdx.x * blockDim.x + threadIdx.x; e < n_up + n_tail; e += (size_t)gridDim.x * blockDim.x)
        aux[e] = bf2f(e < n_up ? blob[up_off + e] : blob[tail_off + (e - n_up)]);
}

cudaError_t launch_repack(const uint16_t *blob, int n_blocks, int C, int s, uint8_t *packed, cudaStream_t st) {
    KScope ks(F_REPACK, st, model_num_layers(n_blocks) + 3);
    size_t src = 0, up_off = 0, tail_off = 0;
    for (int l = 0; l < model_num_layers(n_blocks); l++) {
        LayerShape ls = model_layer(n_blocks, C, s, l);
        if (l == 2 * n_blocks + 2) up_off = src;
        if (l == 2 * n_blocks + 3) tail_off = src;
        k_repack_b<<<256, 256, 0, st>>>(blob, src, ls, C, s, packed);
        src += (size_t)ls.cout_real * ls.cin_real * 9 + ls.cout_real;
    }
    const CompShape cs = model_comp(n_blocks, C, s);
    k_repack_comp<<<256, 256, 0, st>>>(blob, up_off, tail_off, C, s, cs, packed);
    const size_t n_up = (size_t)s * s * C * C * 9 + (size_t)s * s * C, n_tail = (size_t)3 * C * 9 + 3;
    float *aux = reinterpret_cast<float *>(packed + cs.aux_off);
    k_repack_aux<<<256, 256, 0, st>>>(blob, up_off, n_up, tail_off, n_tail, aux);
    const size_t nout = (size_t)s * s * 3;
    k_repack_comp32<<<256, 256, 0, st>>>(blob, up_off, tail_off, C, s, aux + n_up + n_tail,
                                         aux + n_up + n_tail + nout * C * 25);
    return cudaGetLastError();
}

}  // namespace ns
