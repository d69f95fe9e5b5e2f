// k_recon.cu -- reuse-based reconstruction of non-anchor frames (K9; PAPER.md
// §2 P:89-91 and §6.1), chunk-end reference state, per-stream stats
// (K10) and the model weight repack (model pre-optimisation, §6.2).
#include <cstdint>
#include "ns_internal.h"

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

// One frame step f for all streams.  Each thread produces 8 consecutive HR
// pixels of one row (inside one 8x8 LR block, since 8s % 8 == 0) on all three
// planes:  anchor -> skip (SR output already in place); KEY or INTRA block ->
// up_s(LR[f]); otherwise clamp(warp_{s*mv}(HR[ref]) + up_s(res[f]), 0, 255).
constexpr int kReconThreads = 128;
__global__ void __launch_bounds__(kReconThreads)
    k_recon_step(const StreamDesc *sd, int n, int f, const uint8_t *is_anchor, uint8_t *const *hr_tab,
                 const int16_t *gold) {
    const int sid = blockIdx.z;
    if (is_anchor[(size_t)sid * n + f]) return;
    const StreamDesc d = sd[sid];
    const int s = d.s, H = d.h * s, W = d.w * s;
    const int Y = blockIdx.y;
    const int X0 = (blockIdx.x * kReconThreads + threadIdx.x) * 8;
    if (Y >= H || X0 >= W) return;
    const int bw = d.w / 8;
    const ns_block_mv mv = d.mv[(size_t)f * (d.h / 8) * bw + (size_t)(Y / (8 * s)) * bw + X0 / (8 * s)];
    const uint8_t type = d.type[f];
    uint8_t *out = hr_tab[d.hr_base + f];
    const size_t lrp = (size_t)d.h * d.w, hrp = (size_t)H * W;
    const bool use_lr = (type == NS_KEY) || (mv.ref == NS_REF_INTRA);
    const uint8_t *ref = nullptr;
    if (!use_lr) {
        if (mv.ref == NS_REF_GOLDEN) {
            const int g = gold[(size_t)sid * (n + 1) + f];
            ref = g >= 0 ? hr_tab[d.hr_base + g] : d.hr_golden;
        } else {
            ref = f > 0 ? hr_tab[d.hr_base + f - 1] : d.hr_last;
        }
    }
    int ya, yb, wy;
    up_tap_r(Y, s, d.h, ya, yb, wy);
    int xa[8], xb[8], wx[8];
#pragma unroll
    for (int i = 0; i < 8; i++) up_tap_r(X0 + i, s, d.w, xa[i], xb[i], wx[i]);
    // warp geometry (O7): m = s * mv in 1/8 HR pel
    const int mx = s * mv.mvx, my = s * mv.mvy;
    const int ix = X0 + (mx >> 3), fx = mx & 7;
    const int iy = Y + (my >> 3), fy = my & 7;
    const int r0 = min(max(iy, 0), H - 1), r1 = min(max(iy + 1, 0), H - 1);
#pragma unroll
    for (int c = 0; c < 3; c++) {
        uint32_t o[2] = {0, 0};
        if (use_lr) {
            const uint8_t *L = d.lr + ((size_t)f * 3 + c) * lrp;
            const uint8_t *La = L + (size_t)ya * d.w, *Lb = L + (size_t)yb * d.w;
#pragma unroll
            for (int i = 0; i < 8; i++) {
                const int v = (128 - wy) * ((128 - wx[i]) * La[xa[i]] + wx[i] * La[xb[i]]) +
                              wy * ((128 - wx[i]) * Lb[xa[i]] + wx[i] * Lb[xb[i]]);
                o[i >> 2] |= (uint32_t)((v + 8192) >> 14) << (8 * (i & 3));
            }
        } else {
            const int16_t *Rp = d.res + ((size_t)f * 3 + c) * lrp;
            const int16_t *Ra = Rp + (size_t)ya * d.w, *Rb = Rp + (size_t)yb * d.w;
            const uint8_t *P = ref + c * hrp;
            const uint8_t *P0 = P + (size_t)r0 * W, *P1 = P + (size_t)r1 * W;
#pragma unroll
            for (int i = 0; i < 8; i++) {
                const int xa_ = min(max(ix + i, 0), W - 1), xb_ = min(max(ix + i + 1, 0), W - 1);
                const int h0 = (P0[xa_] * (8 - fx) + P0[xb_] * fx + 4) >> 3;
                const int h1 = (P1[xa_] * (8 - fx) + P1[xb_] * fx + 4) >> 3;
                const int pred = (h0 * (8 - fy) + h1 * fy + 4) >> 3;
                const int v = (128 - wy) * ((128 - wx[i]) * Ra[xa[i]] + wx[i] * Ra[xb[i]]) +
                              wy * ((128 - wx[i]) * Rb[xa[i]] + wx[i] * Rb[xb[i]]);
                const int r = (v + 8192) >> 14;
                const int val = min(max(pred + r, 0), 255);
                o[i >> 2] |= (uint32_t)val << (8 * (i & 3));
            }
        }
        *reinterpret_cast<uint2 *>(out + c * hrp + (size_t)Y * W + X0) = make_uint2(o[0], o[1]);
    }
}

cudaError_t launch_recon_step(const StreamDesc *d_sd, int S, int n, int f, int maxW8, int maxH,
                              const uint8_t *is_anchor, uint8_t *const *d_hr_table, const int16_t *gold_idx,
                              cudaStream_t st) {
    KScope ks(F_RECON, st);
    dim3 g((maxW8 + kReconThreads - 1) / kReconThreads, maxH, S);
    k_recon_step<<<g, kReconThreads, 0, st>>>(d_sd, n, f, is_anchor, d_hr_table, gold_idx);
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
    const size_t total = (size_t)9 * ls.cin * ls.ntot;
    uint16_t *B = reinterpret_cast<uint16_t *>(packed + ls.b_off);
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

cudaError_t launch_repack(const uint16_t *blob, int n_blocks, int C, int s, uint8_t *packed, cudaStream_t st) {
    KScope ks(F_REPACK, st, model_num_layers(n_blocks));
    size_t src = 0;
    for (int l = 0; l < model_num_layers(n_blocks); l++) {
        LayerShape ls = model_layer(n_blocks, C, s, l);
        k_repack_b<<<256, 256, 0, st>>>(blob, src, ls, C, s, packed);
        src += (size_t)ls.cout_real * ls.cin_real * 9 + ls.cout_real;
    }
    return cudaGetLastError();
}

}  // namespace ns
