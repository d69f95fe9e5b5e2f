// k_recon.cu -- reuse-based reconstruction of non-anchor frames (K9; PAPER.md
// §2 P:89-91 and §6.1), chunk-end reference state, per-stream stats
// (K10) and the model weight repack (model pre-optimisation, §6.2).
#include <cstdint>
#include <type_traits>
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
// HR rings (nxt != NULL): a KEY/ALTREF frame g is GOLDEN for the frames up to
// the next KEY/ALTREF gn (inclusive: gn still references g), and after the last
// one for the rest of the chunk and the chunk-end state.  If its hr_out entry is
// written again before then (nxt[g] <= min(gn, n-1)) it must be saved into
// hr_golden: gsv[s][g] = 1.
__global__ void k_golden_index(const StreamDesc *sd, int S, int n, const int16_t *nxt, int16_t *gold, uint8_t *gsv) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= S) return;
    const uint8_t *T = sd[s].type;
    int g = -1;
    for (int f = 0; f < n; f++) {
        gold[(size_t)s * (n + 1) + f] = (int16_t)g;
        if ((T[f] & NS_TYPE_MASK) == NS_KEY || (T[f] & NS_TYPE_MASK) == NS_ALTREF) g = f;
    }
    gold[(size_t)s * (n + 1) + n] = (int16_t)g;
    if (!nxt) return;
    int gn = n;
    for (int f = n - 1; f >= 0; f--) {
        const bool golden = (T[f] & NS_TYPE_MASK) == NS_KEY || (T[f] & NS_TYPE_MASK) == NS_ALTREF;
        gsv[(size_t)s * n + f] = golden && nxt[(size_t)s * n + f] <= min(gn, n - 1);
        if (golden) gn = f;
    }
}

cudaError_t launch_golden_index(const StreamDesc *d_sd, int S, int n, const int16_t *nxt, int16_t *gold_idx,
                                uint8_t *gsv, cudaStream_t st) {
    KScope ks(F_RECON, st);
    k_golden_index<<<(S + 127) / 128, 128, 0, st>>>(d_sd, S, n, nxt, gold_idx, gsv);
    return cudaGetLastError();
}

// One frame step f for all streams (K9).  A thread owns one LR block column
// (8s HR pixels wide, the motion vector is uniform there) x RPT HR rows x 3
// planes:  anchor -> skip (SR output already in place); KEY frame or INTRA
// block -> up_s(LR[f]); otherwise clamp(warp_{s*mv}(HR[ref]) + up_s(res[f])).
//
// Memory: every global read is asynchronous.  The CTA's residual tile (all
// three planes: 4*RPT/s + 2 LR rows x 256 + 16 columns of i16) is staged
// cooperatively with 16-B cp.async at entry; each thread's warp windows (the
// MV-displaced reference rows, as aligned 8-B words) are staged per plane with
// cp.async, double-buffered so plane c+1 is in flight while plane c computes.
//
// Arithmetic (two pixels per 32-bit register, 16-bit lanes, every lane value
// < 2^16 so lanes never carry into each other):
//  * warp, horizontal pass (O7): v = R[x](8-fx) + R[x+1]fx + 4 in [4, 2044];
//    the pass result floor(v/8) is kept scaled by 8, h8 = v & ~7 (no shift);
//  * vertical pass: 8 (h0(8-fy) + h1 fy + 4) = h8_0(8-fy) + h8_1 fy + 32, so
//    pred = floor(that / 64);
//  * up_s (O6) per pixel r = floor((v + 8192) / 2^14) lands in the high half of
//    a 32-bit value with a +256 bias; one PRMT packs a pixel pair;
//  * X = 64 (r + 256) + h8_0(8-fy) + h8_1 fy + 32 <= 49056 per lane, and
//    floor(X / 64) = pred + r + 256 (64 (r + 256) is a multiple of 64), so the
//    clamp of pred + r to [0, 255] is a clamp of X to [2^14, 2^15 - 1]; X >> 6
//    then holds 256 + out in each lane and one PRMT packs 4 output bytes.
template <int N, int I = 0, class F>
__device__ __forceinline__ void static_for(F &&f) {
    if constexpr (I < N) {
        f(std::integral_constant<int, I>{});
        static_for<N, I + 1>(f);
    }
}

// CTA shape: kReconTX LR block columns x kReconTY thread rows (RPT HR rows each)
#ifndef NS_RECON_TX
#define NS_RECON_TX 32
#endif
#ifndef NS_RECON_TY
#define NS_RECON_TY 4
#endif
constexpr int kReconTX = NS_RECON_TX, kReconTY = NS_RECON_TY;
#ifndef NS_RECON_RPT3
#define NS_RECON_RPT3 6  // HR rows per thread at s = 3 (a multiple of 3)
#endif
constexpr int kReconNT = kReconTX * kReconTY;
#ifndef NS_RECON_MINB3
#define NS_RECON_MINB3 (512 / (NS_RECON_TX * NS_RECON_TY))
#endif
// Plane geometry of a reconstruction thread.  Luma (and every 4:4:4 plane):
// a thread owns one LR block column = 8 LR / 8s HR pixels, motion at 1/8 pel.
// 4:2:0 chroma (CH, reading R9): the block is 4 x 4 LR / 4s x 4s HR chroma
// pixels, motion = the luma vector read in 1/16 chroma pel.
template <int S, bool CH = false>
struct ReconCfg {
    static constexpr int LRB = CH ? 4 : 8;          // LR pixels per block side in this plane
    static constexpr int BW = LRB * S;              // HR pixels per thread row
    static constexpr int NP = BW / 2;               // 16-bit pairs per row
    static constexpr int WIN = BW + 1;              // reference bytes per row
    static constexpr int NQ = (7 + WIN + 7) / 8;    // aligned 64-bit words per row
    static constexpr int PB = CH ? 4 : 3;           // sub-pel bits of the motion (1/8 or 1/16)
    static constexpr int NLR = LRB + 2;             // LR columns an output row's O6 taps touch
    static constexpr int RPT = (S == 3) ? NS_RECON_RPT3 : 8;  // HR rows per thread: a multiple of S
    static_assert(RPT % S == 0 && BW % RPT == 0, "a thread's rows lie in one block row (uniform MV)");
    static_assert(BW % 4 == 0, "pixel quads of the even/odd pair interleave");
    static constexpr int PER = RPT / S;             // periods of the vertical O6 taps
    // resident CTAs per SM (registers): 512 threads at 128 registers for s = 3
    static constexpr int MINB = (S == 3) ? NS_RECON_MINB3 : (384 / kReconNT > 0 ? 384 / kReconNT : 1);
    static constexpr int RES_COLS = LRB * kReconTX + 16;   // residual tile columns (16-B halo chunk per side)
    static constexpr int NPL = CH ? 2 : 3;          // planes a CTA can step (U, V | up to 3)
    // per-thread 8-B slots of the shared window buffer: RPT+1 window rows of NQ
    // words; KEY-frame / INTRA threads keep their LR rows there instead (2 slots
    // per LR row, PER+2 rows per plane): all planes at once when they fit,
    // else two alternating plane sets -- which can need more slots than the
    // window rows (4:2:0 chroma at s = 2: 24 > 18)
    static constexpr int LRS = (PER + 2) * 2;
    static constexpr bool LR_ALL = NPL * LRS <= (RPT + 1) * NQ;
    static constexpr int SLOTS = (RPT + 1) * NQ > (LR_ALL ? NPL : 2) * LRS ? (RPT + 1) * NQ : (LR_ALL ? NPL : 2) * LRS;
};

template <int S, bool CH = false>
struct ReconSmem {
    using Cfg = ReconCfg<S, CH>;
    static constexpr int RROWS = kReconTY * Cfg::PER + 2;      // residual tile LR rows
    static constexpr size_t REF = (size_t)Cfg::SLOTS * kReconNT * 8;
    static constexpr size_t RES = (size_t)Cfg::NPL * RROWS * Cfg::RES_COLS * 2;
    static constexpr size_t BAR = REF + RES;                           // mbarrier of the residual tile
    static constexpr size_t BYTES = BAR + 16;
};

__device__ __forceinline__ uint32_t prmt(uint32_t a, uint32_t b, uint32_t sel) {
    uint32_t r;
    asm("prmt.b32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(sel));
    return r;
}
__device__ __forceinline__ uint32_t mad_u32(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t r;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(r) : "r"(a), "r"(b), "r"(c));
    return r;
}
// (an L2 prefetch-size hint, .L2::128B / 256B, on these copies measured neutral)
__device__ __forceinline__ void cp_async8(void *dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async4(void *dst, const void *src) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}

// Stage the raw aligned 64-bit words covering reference bytes xs .. xs+BW of
// one row into shared memory: dst[i * stride] is word i (struct-of-arrays
// across the CTA's threads: conflict-free reads).  The plane width and the
// word base are multiples of 8 (4:2:0 requires w % 16 == 0, so chroma planes
// are too), so every word lies wholly inside the row or wholly outside it; an
// outside word stages the row's first / last word instead, and recon_load_row
// replicates its edge pixel (Z16) after the copy lands: every global read
// stays an asynchronous copy, and none reads past the row.
template <int S, bool CH>
__device__ __forceinline__ void recon_row_stage(const uint8_t *row, int xs, int W, bool interior, uint2 *dst,
                                                int stride) {
    using Cfg = ReconCfg<S, CH>;
    const int xb = xs & ~7;
#pragma unroll
    for (int i = 0; i < Cfg::NQ; i++) {
        const int st = interior ? xb + 8 * i : min(max(xb + 8 * i, 0), W - 8);
        cp_async8(dst + i * stride, row + st);
    }
}
// Load one staged window row (NQ words) into registers; for a non-interior
// window replicate the edge pixel into the words that lie outside the row
// (first word at xb).  (on = false: a KEY-frame / INTRA thread, whose warp
// weights are all 0 and whose slots hold LR rows in flight: nothing is read,
// so no shared-memory race.)  wfix is warp-uniform (some lane's window leaves
// the row): the replication is one byte permute per half-word with the
// selector chosen per word -- identity inside the row, byte 0 (the row's first
// pixel) left of it, byte 7 (its last) right of it -- so the row body carries
// 2 NQ permutes behind one uniform branch instead of per-word branches (the
// recon loop is instruction-cache sensitive: DESIGN.md §7).
template <int S, bool CH>
__device__ __forceinline__ void recon_load_row(const uint2 *row, bool on, bool wfix, int xb, int W,
                                               uint2 (&q)[ReconCfg<S, CH>::NQ]) {
    using Cfg = ReconCfg<S, CH>;
#pragma unroll
    for (int i = 0; i < Cfg::NQ; i++) q[i] = on ? row[i * kReconNT] : make_uint2(0u, 0u);
    if (wfix) {
#pragma unroll
        for (int i = 0; i < Cfg::NQ; i++) {
            const int st = xb + 8 * i;
            const uint32_t sx = st < 0 ? 0x0000u : (st >= W ? 0x7777u : 0x3210u);
            const uint32_t sy = st < 0 ? 0x0000u : (st >= W ? 0x7777u : 0x7654u);
            q[i] = make_uint2(prmt(q[i].x, q[i].y, sx), prmt(q[i].x, q[i].y, sy));
        }
    }
}

// Horizontal bilinear pass over one staged reference row.  Pixel pairs are
// even/odd interleaved: pair 2g holds pixels (4g, 4g+2) and pair 2g+1 pixels
// (4g+1, 4g+3), so both operands of each pass come from one byte permute of
// the aligned window word (no per-pair realignment):
//   v[2g] = E_g (F-fx) + O_g fx + F/2,  v[2g+1] = O_g (F-fx) + E'_g fx + F/2  (F = 2^PB)
// with E_g = [p4g, p4g+2], O_g = [p4g+1, p4g+3], E'_g = [p4g+2, p4g+4].
// Luma keeps 8 floor(v/8) (v & ~7, the scale folded into the vertical pass);
// chroma keeps floor(v/16) (every lane < 2^12).
template <int S, bool CH>
__device__ __forceinline__ void recon_hpass(const uint2 (&q)[ReconCfg<S, CH>::NQ], int m, uint32_t fxc, uint32_t fx,
                                            uint32_t (&h)[ReconCfg<S, CH>::NP]) {
    using Cfg = ReconCfg<S, CH>;
    constexpr int NG = Cfg::BW / 4;
    uint32_t w[2 * Cfg::NQ + 2];
#pragma unroll
    for (int i = 0; i < Cfg::NQ; i++) {
        w[2 * i] = q[i].x;
        w[2 * i + 1] = q[i].y;
    }
    w[2 * Cfg::NQ] = 0;
    w[2 * Cfg::NQ + 1] = 0;
    if (m >= 4) {
#pragma unroll
        for (int i = 0; i < 2 * Cfg::NQ + 1; i++) w[i] = w[i + 1];
    }
    const uint32_t sh = 8u * (uint32_t)(m & 3);
    uint32_t E[NG + 1], O[NG];
#pragma unroll
    for (int g = 0; g <= NG; g++) {
        const uint32_t a = __funnelshift_r(w[g], w[g + 1], sh);
        E[g] = prmt(a, 0u, 0x4240u);
        if (g < NG) O[g] = prmt(a, 0u, 0x4341u);
    }
#pragma unroll
    for (int g = 0; g < NG; g++) {
        const uint32_t E1 = __funnelshift_r(E[g], E[g + 1], 16);
        if constexpr (CH) {
            h[2 * g] = ((E[g] * fxc + O[g] * fx + 0x00080008u) >> 4) & 0x0FFF0FFFu;
            h[2 * g + 1] = ((O[g] * fxc + E1 * fx + 0x00080008u) >> 4) & 0x0FFF0FFFu;
        } else {
            h[2 * g] = (E[g] * fxc + O[g] * fx + 0x00040004u) & 0xFFF8FFF8u;
            h[2 * g + 1] = (O[g] * fxc + E1 * fx + 0x00040004u) & 0xFFF8FFF8u;
        }
    }
}
// pixel (within the thread's row) of lane e of pair k (even/odd interleave)
__host__ __device__ constexpr int pair_px(int k, int e) { return 4 * (k >> 1) + (k & 1) + 2 * e; }

// LR rows of KEY frames / INTRA blocks (Z17) are staged per thread in the
// thread's (otherwise unused) warp-window slots, two per LR row: the aligned
// word of the block's LRB columns, and [the 4 columns left | the 4 columns
// right] (clamped to the row; the edge columns are replaced on use when
// outside, Z16).
template <bool CH>
__device__ __forceinline__ void recon_lr_row_stage(const uint8_t *plane, int row, int bx, int w, uint2 *dst) {
    constexpr int LRB = CH ? 4 : 8;
    const uint8_t *p = plane + (size_t)row * w;
    if constexpr (CH) cp_async4(dst, p + LRB * bx);
    else cp_async8(dst, p + LRB * bx);
    uint32_t *e = reinterpret_cast<uint32_t *>(dst + kReconNT);
    cp_async4(e, p + max(LRB * bx - 4, 0));
    cp_async4(e + 1, p + min(LRB * bx + LRB, w - 4));
}
template <bool CH>
__device__ __forceinline__ void recon_lr_row_smem(const uint2 *src, bool left_in, bool right_in,
                                                  int (&v)[(CH ? 4 : 8) + 2]) {
    constexpr int LRB = CH ? 4 : 8;
    const uint2 q = src[0], e = src[kReconNT];
#pragma unroll
    for (int i = 0; i < 4; i++) {
        v[1 + i] = (q.x >> (8 * i)) & 255;
        if (!CH) v[5 + i] = (q.y >> (8 * i)) & 255;
    }
    v[0] = left_in ? (int)(e.x >> 24) : v[1];
    v[LRB + 1] = right_in ? (int)(e.y & 255) : v[LRB];
}

// Residual-row values for LR columns LRB bx - 1 .. LRB bx + LRB from the staged
// tile row `p` (p points at tile column LRB tx, i.e. LR column LRB bx - 8).
template <bool CH>
__device__ __forceinline__ void recon_res_row_smem(const int16_t *p, bool left_in, bool right_in,
                                                   int (&v)[(CH ? 4 : 8) + 2]) {
    constexpr int LRB = CH ? 4 : 8;
    uint32_t qq[LRB / 2];
    if constexpr (CH) {
        const uint2 m = *reinterpret_cast<const uint2 *>(p + 8);
        qq[0] = m.x; qq[1] = m.y;
    } else {
        const uint4 m = *reinterpret_cast<const uint4 *>(p + 8);
        qq[0] = m.x; qq[1] = m.y; qq[2] = m.z; qq[3] = m.w;
    }
#pragma unroll
    for (int i = 0; i < LRB / 2; i++) {
        v[1 + 2 * i] = (int)(int16_t)(qq[i] & 0xFFFFu);
        v[2 + 2 * i] = __mulhi((int)qq[i], 65536);  // arithmetic >> 16 on the FMA pipe
    }
    const int l = p[7], r = p[8 + LRB];
    v[0] = left_in ? l : v[1];
    v[LRB + 1] = right_in ? r : v[LRB];
}

// Compile-time O6 taps.  For an axis coordinate X = S*m + ph + i:
//   u = 2X + 1 - S, x0 = m + floor((2(ph+i) + 1 - S) / 2S), w1 = round(128 rem / 2S).
__host__ __device__ constexpr int fdiv(int a, int b) { return a >= 0 ? a / b : -((-a + b - 1) / b); }
template <int S>
__host__ __device__ constexpr int tap_d(int k) { return fdiv(2 * k + 1 - S, 2 * S); }
template <int S>
__host__ __device__ constexpr int tap_w1(int k) { return (128 * ((2 * k + 1 - S) - 2 * S * tap_d<S>(k)) + S) / (2 * S); }

// up_s (O6) of one output row from the two LR rows a (top) and b (bottom) with
// vertical weight WY: u[k] = pixel pair k as [r + 256 | r' + 256] (16-bit lanes).
//   V[t] = (128 - WY) a[t] + WY b[t]            (exact, per LR column t)
//   v    = 128 V[d] + w1 (V[d+1] - V[d])          (exact 2-D O6 sum, d = tap)
//   s    = 4 (v + 8192 + 2^22) = 512 V[d] + 4 w1 (V[d+1] - V[d]) + KB
// and r + 256 = s >> 16 (high half-word).
template <int S, bool CH, int WY>
__device__ __forceinline__ void recon_up_row(const int (&a)[ReconCfg<S, CH>::NLR], const int (&b)[ReconCfg<S, CH>::NLR],
                                             uint32_t (&u)[ReconCfg<S, CH>::NP]) {
    constexpr int BW = ReconCfg<S, CH>::BW, NLR = ReconCfg<S, CH>::NLR;
    constexpr int KB = 4 * 8192 + 4 * (256 << 14);
    int V[NLR], base[NLR];
#pragma unroll
    for (int t = 0; t < NLR; t++) {
        V[t] = WY ? (128 - WY) * a[t] + WY * b[t] : 128 * a[t];
        base[t] = (int)mad_u32((uint32_t)V[t], 512u, (uint32_t)KB);
    }
#pragma unroll
    for (int k = 0; k < BW / 2; k++) {
        uint32_t sv[2];
#pragma unroll
        for (int e = 0; e < 2; e++) {
            const int i = pair_px(k, e);
            const int d = tap_d<S>(i) + 1, w1 = tap_w1<S>(i);
            sv[e] = (uint32_t)(w1 ? base[d] + (4 * w1) * (V[d + 1] - V[d]) : base[d]);
        }
        u[k] = prmt(sv[0], sv[1], 0x7632u);
    }
}

// Output rows: each thread stores its BW bytes per row as 8-B stores (4-B
// stores when BW is not a multiple of 8: 4:2:0 chroma at s = 3).  (Staging the
// warp's row in shared memory and storing whole 16-B chunks -- the pattern a
// store-only probe ran 2.2x faster, tools/mem_probe.cu -- measured slower in
// this kernel: +11% instructions for stores that were not its bottleneck.)
template <int S, bool CH>
__device__ __forceinline__ void recon_store_row(uint8_t *dst, const uint32_t (&o)[ReconCfg<S, CH>::BW / 4], bool on) {
    constexpr int BW = ReconCfg<S, CH>::BW;
    if constexpr (BW % 8 == 0) {
#pragma unroll
        for (int q = 0; q < BW / 8; q++)
            asm volatile("{ .reg .pred p; setp.ne.u32 p, %3, 0; @p st.global.v2.b32 [%0], {%1, %2}; }" ::"l"(dst + 8 * q),
                         "r"(o[2 * q]), "r"(o[2 * q + 1]), "r"((uint32_t)on)
                         : "memory");
    } else {
#pragma unroll
        for (int q = 0; q < BW / 4; q++)
            asm volatile("{ .reg .pred p; setp.ne.u32 p, %2, 0; @p st.global.b32 [%0], %1; }" ::"l"(dst + 4 * q),
                         "r"(o[q]), "r"((uint32_t)on)
                         : "memory");
    }
}

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

// fd[s][f]: the frame step's pointers resolved once per chunk.
// HR rings (gsv / asrc non-NULL, ns.h): GOLDEN g is read from hr_out[g] while its
// entry holds it; if g must be saved (gsv), step g + 1 copies HR[g] into
// hr_golden -- nothing reads hr_golden during that step, the frames of step g + 1
// still read hr_out[g] (intact: hr_out[f] != hr_out[f-1]) -- and later steps
// read the copy.  An anchor SR'd into the anchor cache (asrc) is copied into
// its entry at its own step.
__global__ void k_frame_desc(const StreamDesc *sd, int S, int n, const uint8_t *is_anchor, uint8_t *const *hr_tab,
                             const int16_t *gold, const uint8_t *gsv, const uint8_t *const *asrc, FrameDesc *fd) {
    const int e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= S * n) return;
    const int sid = e / n, f = e % n;
    const StreamDesc d = sd[sid];
    const size_t lrp = (size_t)d.h * d.w;
    FrameDesc o{};
    o.lr_f = d.lr + (size_t)f * d.lr_frame;
    o.res_f = d.res + (size_t)f * d.lr_frame;
    (void)lrp;
    o.mv_f = d.mv + (size_t)f * (d.h / 8) * (d.w / 8);
    o.out = hr_tab[d.hr_base + f];
    o.ref_last = f > 0 ? hr_tab[d.hr_base + f - 1] : d.hr_last;
    const int g = gold[(size_t)sid * (n + 1) + f];
    const bool saved = g >= 0 && gsv && gsv[(size_t)sid * n + g] && f >= g + 2;
    o.ref_gold = g >= 0 && !saved ? hr_tab[d.hr_base + g] : d.hr_golden;
    o.asrc = asrc ? asrc[e] : nullptr;
    o.gsave_src = nullptr;
    o.gsave_dst = nullptr;
    if (gsv && f > 0 && gsv[e - 1]) {
        o.gsave_src = hr_tab[d.hr_base + f - 1];
        o.gsave_dst = d.hr_golden;
    }
    o.w = d.w;
    o.h = d.h;
    o.s = (int16_t)d.s;
    o.anchor = is_anchor[e] ? 1 : 0;
    o.key = (d.type[f] & NS_TYPE_MASK) == NS_KEY;
    o.fmt = d.fmt;
    o.interp = d.interp;
    fd[e] = o;
}

cudaError_t launch_frame_desc(const StreamDesc *d_sd, int S, int n, const uint8_t *is_anchor,
                              uint8_t *const *d_hr_table, const int16_t *gold_idx, const uint8_t *gsv,
                              const uint8_t *const *asrc, FrameDesc *fd, cudaStream_t st) {
    KScope ks(F_RECON, st);
    k_frame_desc<<<(S * n + 127) / 128, 128, 0, st>>>(d_sd, S, n, is_anchor, d_hr_table, gold_idx, gsv, asrc, fd);
    return cudaGetLastError();
}

// Copies the CTA's HR tile (rows y0 .. y1, bytes x0 .. x1 of each of the 3
// planes) from src to dst in 8-B words (W is a multiple of 8): the HR-ring
// anchor copy and GOLDEN save, done by the frame step's own CTAs.
__device__ __forceinline__ void recon_tile_copy(const uint8_t *src, uint8_t *dst, size_t hrp, int W, int x0, int x1,
                                                int y0, int y1, int tid, int nt, int planes) {
    const int wpr = (x1 - x0) >> 3, rows = y1 - y0, per_plane = wpr * rows;
    for (int i = tid; i < planes * per_plane; i += nt) {
        const int c = i / per_plane, r = (i % per_plane) / wpr, q = i % wpr;
        const size_t off = (size_t)c * hrp + (size_t)(y0 + r) * W + x0 + 8 * q;
        *reinterpret_cast<uint2 *>(dst + off) = *reinterpret_cast<const uint2 *>(src + off);
    }
}

template <int S, bool CH>
__global__ void __launch_bounds__(kReconNT, ReconCfg<S, CH>::MINB)
    k_recon_step(const FrameDesc *fdesc, int n, int f, int s0) {
    using Cfg = ReconCfg<S, CH>;
    using Sm = ReconSmem<S, CH>;
    constexpr int NP = Cfg::NP, RPT = Cfg::RPT, NQ = Cfg::NQ, LRB = Cfg::LRB, PB = Cfg::PB, NLR = Cfg::NLR;
    constexpr int RC = Cfg::RES_COLS;
    const int sid = s0 + blockIdx.z;
    const FrameDesc fd = fdesc[(size_t)sid * n + f];
    if (fd.s != S) return;                              // CTA-uniform
    if (CH && fd.fmt != NS_FMT_I420) return;
    const int w = fd.w, h = fd.h;
    // this launch's plane geometry: full planes, or the 4:2:0 chroma planes
    const int pw = CH ? w / 2 : w, ph = CH ? h / 2 : h, W = S * pw, H = S * ph;
    const int bx0 = blockIdx.x * kReconTX;              // first LR block column of the CTA
    const int Y0c = blockIdx.y * kReconTY * RPT;        // first HR row of the CTA
    if (LRB * bx0 >= pw || Y0c >= H) return;            // CTA-uniform
    const int tid = threadIdx.y * kReconTX + threadIdx.x;
    // planes: 3 (4:4:4), the luma plane of a 4:2:0 frame, or its two chroma planes
    const size_t lrp = (size_t)h * w, hrp = (size_t)S * h * S * w;                   // full-size planes
    const size_t plr = (size_t)ph * pw, phr = (size_t)H * W;                         // this launch's planes
    const size_t lr0 = CH ? lrp : 0, hr0 = CH ? hrp : 0;                             // first plane's offset
    const int np_ = CH ? 2 : (fd.fmt == NS_FMT_I420 ? 1 : 3);
    if (fd.gsave_src || (fd.anchor && fd.asrc)) {       // HR rings only (k_frame_desc)
        const int x0 = Cfg::BW * bx0, x1 = min(Cfg::BW * (bx0 + kReconTX), W), y1 = min(Y0c + kReconTY * RPT, H);
        if (fd.gsave_src) recon_tile_copy(fd.gsave_src + hr0, fd.gsave_dst + hr0, phr, W, x0, x1, Y0c, y1, tid, kReconNT, np_);
        if (fd.anchor && fd.asrc) recon_tile_copy(fd.asrc + hr0, fd.out + hr0, phr, W, x0, x1, Y0c, y1, tid, kReconNT, np_);
    }
    if (fd.anchor) return;                              // CTA-uniform: the anchor's SR bytes are in place
    if (fd.interp != NS_INTERP_BILINEAR) return;        // CTA-uniform: an 8-tap stream steps in k_recon8

    extern __shared__ __align__(16) uint8_t recon_sm[];
    uint2 *rsm = reinterpret_cast<uint2 *>(recon_sm);                  // [RPT+1][NQ][NT] warp windows
    int16_t *tres = reinterpret_cast<int16_t *>(recon_sm + Sm::REF);   // [planes][RROWS][RC] residual tile

    // residual tile: tile row r <-> LR row Y0c/S - 1 + r (clamped, Z16), tile
    // column t <-> LR column LRB bx0 - 8 + t; the part inside the row arrives as one
    // bulk copy per (plane, row) issued by warp 0 (columns outside the row are
    // never read: the edge columns are clamped on use).  One bulk copy per row
    // instead of per-thread 16-B chunks: the chunk loop's index arithmetic was
    // ~6% of the kernel's instructions (ncu source counters).
    uint64_t *tbar = reinterpret_cast<uint64_t *>(recon_sm + Sm::BAR);
    if (!fd.key && tid < 32) {
        const int col_lo = max(LRB * bx0 - 8, 0), col_hi = min(LRB * bx0 - 8 + RC, pw);
        const uint32_t bytes = (uint32_t)(col_hi - col_lo) * 2u;
        if (tid == 0) {
            mbar_init(tbar, 1);
            fence_mbar_init();
            mbar_arrive_expect_tx(tbar, np_ * Sm::RROWS * bytes);
        }
        __syncwarp();
        for (int e = tid; e < np_ * Sm::RROWS; e += 32) {
            const int c = e / Sm::RROWS, rr = e % Sm::RROWS;
            const int row = min(max(Y0c / S - 1 + rr, 0), ph - 1);
            bulk_load(tres + (size_t)e * RC + (col_lo - (LRB * bx0 - 8)),
                      fd.res_f + lr0 + c * plr + (size_t)row * pw + col_lo, bytes, tbar);
        }
    }

    const int bx = bx0 + threadIdx.x;
    const int Y0 = Y0c + threadIdx.y * RPT;
    const bool valid = LRB * bx < pw && Y0 < H;
    const int X0 = bx * Cfg::BW;
    ns_block_mv mv{};
    if (valid) mv = fd.mv_f[(size_t)(Y0 / Cfg::BW) * (w / 8) + bx];
    // KEY frames and INTRA blocks: up_s(LR[f]) (Z17) through the same arithmetic,
    // with a zero prediction (all warp weights 0) and LR rows instead of residual rows
    const bool use_lr = fd.key || mv.ref == NS_REF_INTRA;
    const uint8_t *ref = (mv.ref == NS_REF_GOLDEN ? fd.ref_gold : fd.ref_last) + hr0;
    // warp geometry (O7 / R9): m = s * mv in 1/2^PB HR pel of this plane
    const int mx = S * mv.mvx, my = S * mv.mvy;
    const int xs = X0 + (mx >> PB);
    constexpr uint32_t F = 1u << PB;
    const uint32_t fx = use_lr ? 0u : (uint32_t)(mx & (F - 1)), fy = use_lr ? 0u : (uint32_t)(my & (F - 1));
    const uint32_t fxc = use_lr ? 0u : F - fx, fyc = use_lr ? 0u : F - fy;  // lanes x SCALAR: no cross-lane terms
    const int iy0 = Y0 + (my >> PB);
    const bool interior = xs >= 0 && (xs & ~7) + 8 * NQ <= W;
    // Reference windows live in ONE buffer of RPT+1 rows: row r of plane c+1 is
    // staged right after plane c's warp pass has read row r, one commit group per
    // row, so before the pass over row r there are always exactly RPT groups newer
    // than row r's (wait_group RPT).  LR rows (use_lr threads) ride in the group
    // of row 0: when all planes fit the thread's slots they are staged at once
    // with plane 0 -- LR may be host memory read across PCIe
    // (ns_enhance_streams_host), so its latency is paid once, not per plane --
    // otherwise per plane, alternating between two slot sets.
    constexpr int LRS = Cfg::LRS;                           // slots per plane's LR rows
    constexpr bool LR_ALL = Cfg::LR_ALL;
    auto lr_slots = [&](int c) { return (LR_ALL ? c : (c & 1)) * LRS * kReconNT; };
    uint2 *wbuf = rsm + tid;
    auto stage_row = [&](int c, int r) {
        if (!valid || c >= np_) return;
        if (use_lr) {
            if (r == 0 && (!LR_ALL || c == 0)) {
#pragma unroll 1
                for (int cc = c; cc < (LR_ALL ? np_ : c + 1); cc++)
#pragma unroll
                    for (int t = 0; t < Cfg::PER + 2; t++)
                        recon_lr_row_stage<CH>(fd.lr_f + lr0 + cc * plr, min(max(Y0 / S - 1 + t, 0), ph - 1), bx, pw,
                                               wbuf + lr_slots(cc) + t * 2 * kReconNT);
            }
            return;
        }
        const int rr = min(max(iy0 + r, 0), H - 1);
        recon_row_stage<S, CH>(ref + c * phr + (size_t)rr * W, xs, W, interior, wbuf + r * NQ * kReconNT, kReconNT);
    };
    for (int r = 0; r <= RPT; r++) {
        stage_row(0, r);
        asm volatile("cp.async.commit_group;" ::: "memory");
    }
    const bool left_in = bx > 0, right_in = LRB * bx + LRB < pw;
    const int m = xs & 7;
    const bool wfix = __any_sync(0xffffffffu, valid && !interior && !use_lr);  // warp-uniform
    uint8_t *outp = fd.out + hr0 + (size_t)Y0 * W + X0;
    // combine (see the top of this file): luma X = 64 (r + 256) + 8h0 (8-fy) + 8h1 fy + 32,
    // chroma X = 16 (r + 256) + h0 (16-fy) + h1 fy + 8; floor(X / 2^SH) = pred + r + 256
    constexpr uint32_t SH = CH ? 4 : 6;
    constexpr uint32_t UMUL = 1u << SH, UADD = CH ? 0x00080008u : 0x00200020u;
    constexpr uint32_t XLO = (256u << SH) * 0x00010001u, XHI = ((512u << SH) - 1) * 0x00010001u;

#pragma unroll 1
    for (int c = 0; c < np_; c++) {
        asm volatile("cp.async.wait_group %0;" ::"n"(RPT) : "memory");
        if (c == 0) {
            __syncthreads();                                    // (orders the tile barrier's init)
            if (!fd.key) mbar_wait(tbar, 0);                    // the residual tile
        }
        // (use_lr threads run the warp pass on zero words: every weight is 0, so pred = 0)
        const int16_t *tp = tres + ((size_t)c * Sm::RROWS + threadIdx.y * Cfg::PER) * RC + LRB * threadIdx.x;
        const uint2 *lrb = wbuf + lr_slots(c);
        uint8_t *outc = outp + c * phr;
        uint32_t hA[NP], hB[NP];   // warp rows j (prev) and j + 1 (cur), ping-pong by row parity
        {
            uint2 q[NQ];
            recon_load_row<S, CH>(wbuf, !use_lr, wfix, xs & ~7, W, q);
            recon_hpass<S, CH>(q, m, fxc, fx, hA);
        }
        stage_row(c + 1, 0);
        asm volatile("cp.async.commit_group;" ::: "memory");
#pragma unroll 1
        for (int it = 0; it < Cfg::PER; it++) {
            int rv[3][NLR];  // LR rows it .. it + 2 of this thread
            if (!use_lr) {
#pragma unroll
                for (int t = 0; t < 3; t++) recon_res_row_smem<CH>(tp + (it + t) * RC, left_in, right_in, rv[t]);
            } else {
#pragma unroll
                for (int t = 0; t < 3; t++) recon_lr_row_smem<CH>(lrb + (it + t) * 2 * kReconNT, left_in, right_in, rv[t]);
            }
            auto one = [&](auto jc) {
                constexpr int jj = decltype(jc)::value;
                constexpr int ta = tap_d<S>(jj) + 1;
                const int j = it * S + jj;
                uint32_t(&hp)[NP] = (jj & 1) ? hB : hA;
                uint32_t(&hc)[NP] = (jj & 1) ? hA : hB;
                asm volatile("cp.async.wait_group %0;" ::"n"(RPT) : "memory");
                uint2 q[NQ];
                recon_load_row<S, CH>(wbuf + (j + 1) * NQ * kReconNT, !use_lr, wfix, xs & ~7, W, q);
                uint32_t u[NP], x[NP], o[Cfg::BW / 4];
                recon_up_row<S, CH, tap_w1<S>(jj)>(rv[ta], rv[ta + 1], u);   // independent of q: covers the load
                recon_hpass<S, CH>(q, m, fxc, fx, hc);
                stage_row(c + 1, j + 1);
                asm volatile("cp.async.commit_group;" ::: "memory");
#pragma unroll
                for (int k = 0; k < NP; k++) {
                    const uint32_t X = mad_u32(hp[k], fyc, mad_u32(hc[k], fy, mad_u32(u[k], UMUL, UADD)));
                    x[k] = __umulhi(vmin_u16x2(vmax_u16x2(X, XLO), XHI), 1u << (32 - SH));  // >> SH
                }
#pragma unroll
                for (int q = 0; q < Cfg::BW / 4; q++) o[q] = prmt(x[2 * q], x[2 * q + 1], 0x6240u);
                recon_store_row<S, CH>(outc + (size_t)j * W, o, valid);
            };
            static_for<S>(one);
            if constexpr (S & 1) {  // the period ended on an even row: its warp row is in hB
#pragma unroll
                for (int k = 0; k < NP; k++) hA[k] = hB[k];
            }
        }
    }
}

// ---------------------------------------------------------------- 8-tap MC (NEXT-2, R13)
// Streams whose codec predicts with VP9's 8-tap sub-pel filters (ns_chunk.interp,
// include/ns.h): the reused frame is predicted the way the decoder predicted
// its LR frame -- libvpx convolve8 on the HR reference at 1/16 pel (2 s mv for
// luma, s mv for 4:2:0 chroma), 8 taps at -3..+4, each pass rounded by 7 bits
// and clipped to a byte, edges replicated -- then the O8 combine with up_s of
// the residual, exactly as in k_recon_step.
//
// A thread owns 4 LR columns (4s HR pixels; half a luma block, a whole chroma
// block) over one block row (8s luma / 4s chroma HR rows), so its motion
// vector and kernel are uniform.  Its reference window rows (4s + 7 bytes,
// R + 7 rows) stream through a shared-memory ring by cp.async; each row's
// horizontal pass (16-bit lanes holding two pixels, even/odd interleaved as in
// k_recon_step) goes into a per-thread shared-memory ring of 8 rows, and the
// vertical pass of output row j runs as soon as window row j + 7 is filtered.
// (Keeping those 8 rows in registers needs the row loop fully unrolled: 5.9K
// instructions that miss the instruction cache, 167 registers, 3 CTAs per SM
// -- 204 vs 147 ms per c4 step.)
// 16-bit lanes: a pass sums 8 taps of bytes with a bias of 128 * 128 + 64 per
// lane, sum + bias in [2678, 62858] for every kernel (the sharpest phase has
// positive taps 182, negative 54), so the packed multiply-adds never carry
// across lanes; the clamp to [128 * 128, 384 * 128 - 1] is the byte clip.
//
// VP9's kernels (libvpx vp9_filter.c: sub_pel_filters_8, _8lp, _8s), a
// transcription of its own (the oracle keeps another).
__constant__ int16_t c_vp9_f8[3][16][8] = {
    {{0, 0, 0, 128, 0, 0, 0, 0},        {0, 1, -5, 126, 8, -3, 1, 0},
     {-1, 3, -10, 122, 18, -6, 2, 0},   {-1, 4, -13, 118, 27, -9, 3, -1},
     {-1, 4, -16, 112, 37, -11, 4, -1}, {-1, 5, -18, 105, 48, -14, 4, -1},
     {-1, 5, -19, 97, 58, -16, 5, -1},  {-1, 6, -19, 88, 68, -18, 5, -1},
     {-1, 6, -19, 78, 78, -19, 6, -1},  {-1, 5, -18, 68, 88, -19, 6, -1},
     {-1, 5, -16, 58, 97, -19, 5, -1},  {-1, 4, -14, 48, 105, -18, 5, -1},
     {-1, 4, -11, 37, 112, -16, 4, -1}, {-1, 3, -9, 27, 118, -13, 4, -1},
     {0, 2, -6, 18, 122, -10, 3, -1},   {0, 1, -3, 8, 126, -5, 1, 0}},
    {{0, 0, 0, 128, 0, 0, 0, 0},        {-3, -1, 32, 64, 38, 1, -3, 0},
     {-2, -2, 29, 63, 41, 2, -3, 0},    {-2, -2, 26, 63, 43, 4, -4, 0},
     {-2, -3, 24, 62, 46, 5, -4, 0},    {-2, -3, 21, 60, 49, 7, -4, 0},
     {-1, -4, 18, 59, 51, 9, -4, 0},    {-1, -4, 16, 57, 53, 12, -4, -1},
     {-1, -4, 14, 55, 55, 14, -4, -1},  {-1, -4, 12, 53, 57, 16, -4, -1},
     {0, -4, 9, 51, 59, 18, -4, -1},    {0, -4, 7, 49, 60, 21, -3, -2},
     {0, -4, 5, 46, 62, 24, -3, -2},    {0, -4, 4, 43, 63, 26, -2, -2},
     {0, -3, 2, 41, 63, 29, -2, -2},    {0, -3, 1, 38, 64, 32, -1, -3}},
    {{0, 0, 0, 128, 0, 0, 0, 0},        {-1, 3, -7, 127, 8, -3, 1, 0},
     {-2, 5, -13, 125, 17, -6, 3, -1},  {-3, 7, -17, 121, 27, -10, 5, -2},
     {-4, 9, -20, 115, 37, -13, 6, -2}, {-4, 10, -23, 108, 48, -16, 8, -3},
     {-4, 10, -24, 100, 59, -19, 9, -3}, {-4, 11, -24, 90, 70, -21, 10, -4},
     {-4, 11, -23, 80, 80, -23, 11, -4}, {-4, 10, -21, 70, 90, -24, 11, -4},
     {-3, 9, -19, 59, 100, -24, 10, -4}, {-3, 8, -16, 48, 108, -23, 10, -4},
     {-2, 6, -13, 37, 115, -20, 9, -4}, {-2, 5, -10, 27, 121, -17, 7, -3},
     {-1, 3, -6, 17, 125, -13, 5, -2},  {0, 1, -3, 8, 127, -7, 3, -1}}};

constexpr int kR8TX = 32, kR8TY = 4, kR8NT = kR8TX * kR8TY;
#ifndef NS_R8_LA
#define NS_R8_LA 4     // window rows in flight per thread
#endif
#ifndef NS_R8_UNROLL
#define NS_R8_UNROLL 1 // row-loop unroll of k_recon8
#endif
#define NS_PRAGMA_(x) _Pragma(#x)
#define NS_UNROLL_(n) NS_PRAGMA_(unroll n)
constexpr uint32_t kR8Bias = (128u * 128u + 64u) * 0x00010001u;
constexpr uint32_t kR8Lo = (128u * 128u) * 0x00010001u, kR8Hi = (384u * 128u - 1u) * 0x00010001u;

// One LR row of a k_recon8 thread's 6 O6 source columns (4 own + one each
// side, clamped, Z16): LR bytes (KEY / INTRA) or the residual.
template <bool LR>
__device__ __forceinline__ void r8_lr_row(const void *plane, int row, int pw, int c0, int cl, int cr, int (&v)[6]) {
    if constexpr (LR) {
        const uint8_t *p = static_cast<const uint8_t *>(plane) + (size_t)row * pw;
        const uint32_t q4 = *reinterpret_cast<const uint32_t *>(p + c0);
#pragma unroll
        for (int e = 0; e < 4; e++) v[1 + e] = (q4 >> (8 * e)) & 255;
        v[0] = p[cl];
        v[5] = p[cr];
    } else {
        const int16_t *p = static_cast<const int16_t *>(plane) + (size_t)row * pw;
        const uint2 q4 = *reinterpret_cast<const uint2 *>(p + c0);
        v[1] = (int)(int16_t)(q4.x & 0xFFFFu); v[2] = (int)(int16_t)(q4.x >> 16);
        v[3] = (int)(int16_t)(q4.y & 0xFFFFu); v[4] = (int)(int16_t)(q4.y >> 16);
        v[0] = p[cl];
        v[5] = p[cr];
    }
}

template <int S, bool CH>
struct R8Cfg {
    static constexpr int TW = 4 * S;                  // HR pixels per thread row (4 LR columns)
    static constexpr int NPT = TW / 2;                // 16-bit pairs per row
    static constexpr int R = CH ? 4 * S : 8 * S;      // HR rows per thread: one block row (uniform vector)
    static constexpr int NW = R + 7;                  // window rows
    static constexpr int NQ = (7 + TW + 7 + 7) / 8;   // aligned 8-B words per window row
    static constexpr int JMAX = pair_px(NPT - 1, 0) + 7;  // last pair source P_j of a row
    static constexpr int GMAX = JMAX / 4 + 1;         // aligned 4-byte groups a row's pass touches
    static_assert(4 * (GMAX + 1) + 7 <= 8 * NQ + 8, "window words cover every pass source");
    static constexpr int LA = NS_R8_LA, NR = LA + 1;  // window rows in flight; ring slots
    static constexpr size_t WIN = (size_t)NR * NQ * kR8NT * 8;             // [NR][NQ][NT] 8-B words
    static constexpr size_t TRING = (size_t)8 * (NPT / 2) * kR8NT * 8;     // [8][NPT/2][NT] pass rows
    static constexpr size_t SMEM = WIN + TRING;
};

template <int S, bool CH>
__global__ void __launch_bounds__(kR8NT) k_recon8(const FrameDesc *fdesc, int n, int f, int s0) {
    using Cfg = R8Cfg<S, CH>;
    constexpr int TW = Cfg::TW, NPT = Cfg::NPT, R = Cfg::R, NW = Cfg::NW, NQ = Cfg::NQ, LA = Cfg::LA, NR = Cfg::NR;
    constexpr int GMAX = Cfg::GMAX;
    const int sid = s0 + blockIdx.z;
    const FrameDesc fd = fdesc[(size_t)sid * n + f];
    if (fd.s != S || fd.interp == NS_INTERP_BILINEAR || fd.anchor) return;   // CTA-uniform
    if (CH && fd.fmt != NS_FMT_I420) return;
    const int w = fd.w, h = fd.h;
    const int pw = CH ? w / 2 : w, ph = CH ? h / 2 : h, W = S * pw, H = S * ph;
    const int gx0 = blockIdx.x * kR8TX;
    const int Y0c = blockIdx.y * kR8TY * R;
    if (4 * gx0 >= pw || Y0c >= H) return;              // CTA-uniform
    __shared__ int16_t s_f8[3 * 16 * 8];
    extern __shared__ __align__(16) uint8_t r8_sm[];
    const int tid = threadIdx.y * kR8TX + threadIdx.x;
    for (int i = tid; i < 3 * 16 * 8; i += kR8NT) s_f8[i] = (&c_vp9_f8[0][0][0])[i];
    __syncthreads();
    const int gx = gx0 + threadIdx.x;
    const int Y0 = Y0c + threadIdx.y * R;
    if (4 * gx >= pw || Y0 >= H) return;                // (no barrier below)

    const size_t lrp = (size_t)h * w, hrp = (size_t)S * h * S * w;
    const size_t plr = (size_t)ph * pw, phr = (size_t)H * W;
    const size_t lr0 = CH ? lrp : 0, hr0 = CH ? hrp : 0;
    const int np_ = CH ? 2 : (fd.fmt == NS_FMT_I420 ? 1 : 3);
    const int bxm = CH ? gx : gx >> 1, bym = Y0 / R;
    const ns_block_mv mv = fd.mv_f[(size_t)bym * (w / 8) + bxm];
    const bool use_lr = fd.key || mv.ref == NS_REF_INTRA;
    const int kern = fd.interp == NS_INTERP_SWITCHABLE ? (mv.filter > 2 ? 0 : mv.filter) : fd.interp - 1;
    const int qx = (CH ? 1 : 2) * S * mv.mvx, qy = (CH ? 1 : 2) * S * mv.mvy;
    const int X0 = gx * TW;
    const int xs = X0 + (qx >> 4) - 3, ys = Y0 + (qy >> 4) - 3;
    uint32_t fx[8], fy[8];
#pragma unroll
    for (int t = 0; t < 8; t++) {
        fx[t] = (uint32_t)(int)s_f8[(kern * 16 + (qx & 15)) * 8 + t];
        fy[t] = (uint32_t)(int)s_f8[(kern * 16 + (qy & 15)) * 8 + t];
    }
    const int xb = xs & ~7, m = xs & 7;
    const bool interior = xb >= 0 && xb + 8 * NQ <= W;
    const uint8_t *ref = (mv.ref == NS_REF_GOLDEN ? fd.ref_gold : fd.ref_last) + hr0;
    uint2 *ring = reinterpret_cast<uint2 *>(r8_sm) + tid;                         // [NR][NQ][NT]
    uint2 *tring = reinterpret_cast<uint2 *>(r8_sm + Cfg::WIN) + tid;            // [8][NPT/2][NT]
    const int c0 = 4 * gx, cl = max(c0 - 1, 0), cr = min(c0 + 4, pw - 1);
    const int lr_row0 = Y0 / S - 1;

#pragma unroll 1
    for (int c = 0; c < np_; c++) {
        const uint8_t *refc = ref + c * phr;
        int st_slot = 0, rd_slot = 0;
        auto stage = [&](int i) {
            if (!use_lr && i < NW) {
                const uint8_t *row = refc + (size_t)min(max(ys + i, 0), H - 1) * W;
                uint2 *dst = ring + st_slot * NQ * kR8NT;
#pragma unroll
                for (int q = 0; q < NQ; q++)
                    cp_async8(dst + q * kR8NT, row + (interior ? xb + 8 * q : min(max(xb + 8 * q, 0), W - 8)));
            }
            st_slot = st_slot == NR - 1 ? 0 : st_slot + 1;
            asm volatile("cp.async.commit_group;" ::: "memory");
        };
#pragma unroll
        for (int i = 0; i < LA; i++) stage(i);
        const void *src_c = use_lr ? static_cast<const void *>(fd.lr_f + lr0 + c * plr)
                                   : static_cast<const void *>(fd.res_f + lr0 + c * plr);
        auto lr_row = [&](int k, int (&v)[6]) {
            const int row = min(max(lr_row0 + k, 0), ph - 1);
            if (use_lr) r8_lr_row<true>(src_c, row, pw, c0, cl, cr, v);
            else r8_lr_row<false>(src_c, row, pw, c0, cl, cr, v);
        };
        int rv[3][6];
        lr_row(0, rv[0]);
        lr_row(1, rv[1]);
        lr_row(2, rv[2]);
        uint8_t *outc = fd.out + hr0 + c * phr + (size_t)Y0 * W + X0;
        NS_UNROLL_(NS_R8_UNROLL)
        for (int i = 0; i < NW; i++) {
            asm volatile("cp.async.wait_group %0;" ::"n"(LA - 1) : "memory");
            uint2 q[NQ];
            const uint2 *src = ring + rd_slot * NQ * kR8NT;
            rd_slot = rd_slot == NR - 1 ? 0 : rd_slot + 1;
#pragma unroll
            for (int k = 0; k < NQ; k++) q[k] = use_lr ? make_uint2(0u, 0u) : src[k * kR8NT];
            if (!interior) {
#pragma unroll
                for (int k = 0; k < NQ; k++) {
                    const int st = xb + 8 * k;
                    if (st < 0) { const uint32_t v = prmt(q[k].x, 0u, 0x0000u); q[k] = make_uint2(v, v); }
                    else if (st >= W) { const uint32_t v = prmt(q[k].y, 0u, 0x3333u); q[k] = make_uint2(v, v); }
                }
            }
            stage(i + LA);
            uint32_t wv[2 * NQ + 2];
#pragma unroll
            for (int k = 0; k < NQ; k++) { wv[2 * k] = q[k].x; wv[2 * k + 1] = q[k].y; }
            wv[2 * NQ] = 0;
            wv[2 * NQ + 1] = 0;
            if (m >= 4) {
#pragma unroll
                for (int k = 0; k < 2 * NQ + 1; k++) wv[k] = wv[k + 1];
            }
            const uint32_t sh = 8u * (uint32_t)(m & 3);
            uint32_t E[GMAX + 1], O[GMAX + 1];
#pragma unroll
            for (int g = 0; g <= GMAX; g++) {
                const uint32_t a = __funnelshift_r(wv[g], wv[g + 1], sh);
                E[g] = prmt(a, 0u, 0x4240u);
                O[g] = prmt(a, 0u, 0x4341u);
            }
            auto P = [&](int j) -> uint32_t {
                const int g = j >> 2;
                switch (j & 3) {
                    case 0: return E[g];
                    case 1: return O[g];
                    case 2: return __funnelshift_r(E[g], E[g + 1], 16);
                    default: return __funnelshift_r(O[g], O[g + 1], 16);
                }
            };
            uint2 *trow = tring + (i & 7) * (NPT / 2) * kR8NT;
#pragma unroll
            for (int k2 = 0; k2 < NPT / 2; k2++) {
                uint32_t tv[2];
#pragma unroll
                for (int e = 0; e < 2; e++) {
                    const int x0 = pair_px(2 * k2 + e, 0);
                    uint32_t acc = kR8Bias;
#pragma unroll
                    for (int t = 0; t < 8; t++) acc = mad_u32(P(x0 + t), fx[t], acc);
                    acc = vmin_u16x2(vmax_u16x2(acc, kR8Lo), kR8Hi);
                    tv[e] = ((acc - kR8Lo) >> 7) & 0x00FF00FFu;
                }
                trow[k2 * kR8NT] = make_uint2(tv[0], tv[1]);
            }
            if (i < 7) continue;
            const int j = i - 7, jj = j % S;
            if (jj == 0 && j > 0) {   // a new O6 period: shift the source rows in
#pragma unroll
                for (int t = 0; t < 6; t++) { rv[0][t] = rv[1][t]; rv[1][t] = rv[2][t]; }
                lr_row(j / S + 2, rv[2]);
            }
            const int ta = tap_d<S>(jj) + 1, wy = tap_w1<S>(jj);
            int V[6], base[6];
#pragma unroll
            for (int t = 0; t < 6; t++) {
                const int a = ta ? rv[1][t] : rv[0][t], b = ta ? rv[2][t] : rv[1][t];
                V[t] = (128 - wy) * a + wy * b;
                base[t] = (int)mad_u32((uint32_t)V[t], 512u, (uint32_t)(4 * 8192 + 4 * (384 << 14)));
            }
            uint32_t acc[NPT];
#pragma unroll
            for (int k = 0; k < NPT; k++) acc[k] = kR8Bias;
#pragma unroll
            for (int r = 0; r < 8; r++) {
                const uint2 *tr = tring + ((j + r) & 7) * (NPT / 2) * kR8NT;
#pragma unroll
                for (int k2 = 0; k2 < NPT / 2; k2++) {
                    const uint2 tv = tr[k2 * kR8NT];
                    acc[2 * k2] = mad_u32(tv.x, fy[r], acc[2 * k2]);
                    acc[2 * k2 + 1] = mad_u32(tv.y, fy[r], acc[2 * k2 + 1]);
                }
            }
            uint32_t x[NPT], o[TW / 4];
#pragma unroll
            for (int k = 0; k < NPT; k++) {
                uint32_t sv[2];
#pragma unroll
                for (int e = 0; e < 2; e++) {
                    const int px = pair_px(k, e);
                    const int d = tap_d<S>(px) + 1, w1 = tap_w1<S>(px);
                    sv[e] = (uint32_t)(w1 ? base[d] + (4 * w1) * (V[d + 1] - V[d]) : base[d]);
                }
                const uint32_t u = prmt(sv[0], sv[1], 0x7632u);
                const uint32_t a = vmin_u16x2(vmax_u16x2(acc[k], kR8Lo), kR8Hi);
                const uint32_t pv = use_lr ? 0x00800080u : (a >> 7) & 0x01FF01FFu;
                x[k] = vmin_u16x2(vmax_u16x2(pv + u, 0x02000200u), 0x02FF02FFu);
            }
#pragma unroll
            for (int qq = 0; qq < TW / 4; qq++) o[qq] = prmt(x[2 * qq], x[2 * qq + 1], 0x6240u);
            uint8_t *dst = outc + (size_t)j * W;
            if constexpr (TW % 16 == 0) {
#pragma unroll
                for (int qq = 0; qq < TW / 16; qq++)
                    *reinterpret_cast<uint4 *>(dst + 16 * qq) = make_uint4(o[4 * qq], o[4 * qq + 1], o[4 * qq + 2], o[4 * qq + 3]);
            } else if constexpr (TW % 8 == 0) {
#pragma unroll
                for (int qq = 0; qq < TW / 8; qq++) *reinterpret_cast<uint2 *>(dst + 8 * qq) = make_uint2(o[2 * qq], o[2 * qq + 1]);
            } else {
#pragma unroll
                for (int qq = 0; qq < TW / 4; qq++) *reinterpret_cast<uint32_t *>(dst + 4 * qq) = o[qq];
            }
        }
    }
}

// Carveout: just enough shared memory for MINB resident CTAs, the rest of the
// 256-KB array stays L1 (the window words of neighbouring threads overlap and
// hit there): the maximum-shared carveout (28 KB of L1) vs this (60 KB) measured
// 70.2 vs 62.8 ms of reconstruction per c4 step (tools/ab_libs.sh, one box).
template <int S, bool CH>
constexpr int recon_carveout_pct() {
    return (int)((ReconCfg<S, CH>::MINB * (ReconSmem<S, CH>::BYTES + 1024) * 100 + 228 * 1024 - 1) / (228 * 1024));
}

template <int S, bool CH>
static cudaError_t recon_launch(dim3 g, cudaStream_t st, const FrameDesc *fd, int n, int f, int s0) {
    if (cudaError_t e = ensure_kernel_smem<k_recon_step<S, CH>>((int)ReconSmem<S, CH>::BYTES,
                                                                 recon_carveout_pct<S, CH>());
        e != cudaSuccess)
        return e;
    k_recon_step<S, CH><<<g, dim3(kReconTX, kReconTY), ReconSmem<S, CH>::BYTES, st>>>(fd, n, f, s0);
    return cudaGetLastError();
}

template <int S, bool CH>
static cudaError_t recon8_launch(int max_pw, int max_ph, cudaStream_t st, const FrameDesc *fd, int n, int f, int s0,
                                 int nstreams) {
    using Cfg = R8Cfg<S, CH>;
    if (cudaError_t e = ensure_kernel_smem<k_recon8<S, CH>>((int)Cfg::SMEM); e != cudaSuccess) return e;
    dim3 g((max_pw / 4 + kR8TX - 1) / kR8TX, (max_ph * S / Cfg::R + kR8TY - 1) / kR8TY, nstreams);
    k_recon8<S, CH><<<g, dim3(kR8TX, kR8TY), Cfg::SMEM, st>>>(fd, n, f, s0);
    return cudaGetLastError();
}

cudaError_t launch_recon_step(const FrameDesc *fd, int S, int n, int f, const int *max_lr_w, const int *max_lr_h,
                              const int *has_i420, const int *e8, cudaStream_t st, int s0) {
    int nl = 0;
    for (int s = 2; s <= 4; s++) nl += (max_lr_w[s] > 0) + (has_i420[s] != 0) + (e8[s] & 1) + ((e8[s] >> 1) & 1);
    KScope ks(F_RECON, st, nl);
    for (int s = 2; s <= 4; s++) {
        if (max_lr_w[s] <= 0) continue;
        const int nbx = max_lr_w[s] / 8;          // LR block columns
        const int rpt = s == 2 ? ReconCfg<2>::RPT : s == 3 ? ReconCfg<3>::RPT : ReconCfg<4>::RPT;
        const int nrg = (max_lr_h[s] * s + rpt - 1) / rpt;  // groups of RPT HR rows
        dim3 g((nbx + kReconTX - 1) / kReconTX, (nrg + kReconTY - 1) / kReconTY, S);
        cudaError_t e = s == 2 ? recon_launch<2, false>(g, st, fd, n, f, s0)
                        : s == 3 ? recon_launch<3, false>(g, st, fd, n, f, s0) : recon_launch<4, false>(g, st, fd, n, f, s0);
        if (e != cudaSuccess) return e;
        if (has_i420[s]) {  // the chroma planes of the 4:2:0 streams of this scale, same frame step
            const int nrc = (max_lr_h[s] / 2 * s + rpt - 1) / rpt;
            dim3 gc(g.x, (nrc + kReconTY - 1) / kReconTY, S);
            e = s == 2 ? recon_launch<2, true>(gc, st, fd, n, f, s0)
                : s == 3 ? recon_launch<3, true>(gc, st, fd, n, f, s0) : recon_launch<4, true>(gc, st, fd, n, f, s0);
            if (e != cudaSuccess) return e;
        }
        // 8-tap streams (after k_recon_step, which did their HR-ring copies)
        const int W8 = max_lr_w[s], H8 = max_lr_h[s];
        if (e8[s] & 1) {
            e = s == 2 ? recon8_launch<2, false>(W8, H8, st, fd, n, f, s0, S)
                : s == 3 ? recon8_launch<3, false>(W8, H8, st, fd, n, f, s0, S) : recon8_launch<4, false>(W8, H8, st, fd, n, f, s0, S);
            if (e != cudaSuccess) return e;
        }
        if (e8[s] & 2) {
            e = s == 2 ? recon8_launch<2, true>(W8 / 2, H8 / 2, st, fd, n, f, s0, S)
                : s == 3 ? recon8_launch<3, true>(W8 / 2, H8 / 2, st, fd, n, f, s0, S)
                         : recon8_launch<4, true>(W8 / 2, H8 / 2, st, fd, n, f, s0, S);
            if (e != cudaSuccess) return e;
        }
    }
    return cudaGetLastError();
}

// Chunk-end reference state: hr_last <- HR[n-1], hr_golden <- HR[gold[n]].
__global__ void k_state_copy(const StreamDesc *sd, int n, uint8_t *const *hr_tab, const int16_t *gold,
                             const uint8_t *gsv) {
    const int sid = blockIdx.y, which = blockIdx.z;
    const StreamDesc d = sd[sid];
    const size_t nvec = (size_t)d.hr_frame / 16;
    uint8_t *dst;
    const uint8_t *src;
    if (which == 0) {
        dst = d.hr_last;
        src = hr_tab[d.hr_base + n - 1];
    } else {
        // HR rings: a saved GOLDEN is in hr_golden already (its entry may be gone)
        const int g = gold[(size_t)sid * (n + 1) + n];
        dst = d.hr_golden;
        src = g >= 0 && !(gsv && gsv[(size_t)sid * n + g]) ? hr_tab[d.hr_base + g] : nullptr;
    }
    if (!dst || !src || dst == src) return;
    const uint4 *s4 = reinterpret_cast<const uint4 *>(src);
    uint4 *d4 = reinterpret_cast<uint4 *>(dst);
    for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < nvec; i += (size_t)gridDim.x * blockDim.x)
        d4[i] = s4[i];
}

cudaError_t launch_state_copy(const StreamDesc *d_sd, int S, int n, uint8_t *const *d_hr_table,
                              const int16_t *gold_idx, const uint8_t *gsv, size_t max_hr_bytes, cudaStream_t st) {
    const int blocks = (int)((max_hr_bytes / 16 + 255) / 256);
    KScope ks(F_STATE, st);
    dim3 g(blocks < 1 ? 1 : (blocks > 4096 ? 4096 : blocks), S, 2);
    k_state_copy<<<g, 256, 0, st>>>(d_sd, n, d_hr_table, gold_idx, gsv);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- K10 stats
// stats[s] = {frames, anchors, sum anchor score, total score, SSE vs gt, PSNR, 0, 0}
__global__ void k_stats_meta(const StreamDesc *sd, int S, int n, const uint8_t *is_anchor, const int64_t *score,
                             double *stats) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= S) return;
    double a = 0, sa = 0, st = 0, shown = 0;
    for (int f = 0; f < n; f++) {
        const double v = (double)score[(size_t)s * n + f];
        st += v;
        if (is_anchor[(size_t)s * n + f]) { a += 1; sa += v; }
        shown += (sd[s].type[f] & NS_INVISIBLE) ? 0 : 1;   // invisible frames are not displayed (R12)
    }
    double *o = stats + (size_t)s * 8;
    o[0] = shown; o[1] = a; o[2] = sa; o[3] = st;
    o[4] = sd[s].gt ? 0.0 : -1.0;
    o[5] = -1.0; o[6] = 0; o[7] = 0;
}

__global__ void k_stats_sse(const StreamDesc *sd, int n, uint8_t *const *hr_tab, double *stats) {
    const int sf = blockIdx.x, sid = sf / n, f = sf % n;   // (stream, frame) on x: S*n may exceed 65535
    const StreamDesc d = sd[sid];
    if (!d.gt || (d.type[f] & NS_INVISIBLE)) return;   // quality over the displayed frames
    const size_t nvec = (size_t)d.hr_frame / 16;
    const uint4 *a = reinterpret_cast<const uint4 *>(hr_tab[d.hr_base + f]);
    const uint4 *b = reinterpret_cast<const uint4 *>(d.gt + (size_t)f * nvec * 16);
    unsigned long long acc = 0;
    for (size_t i = (size_t)blockIdx.y * blockDim.x + threadIdx.x; i < nvec; i += (size_t)gridDim.y * blockDim.x) {
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
    const double N = (double)sd[s].hr_frame * stats[(size_t)s * 8 + 0];   // displayed frames
    const double sse = stats[(size_t)s * 8 + 4];
    double p = sse == 0.0 ? 100.0 : 10.0 * log10(255.0 * 255.0 / (sse / N));
    stats[(size_t)s * 8 + 5] = p > 100.0 ? 100.0 : p;
}

cudaError_t launch_stats(const StreamDesc *d_sd, int S, int n, const uint8_t *is_anchor, const int64_t *score,
                         uint8_t *const *d_hr_table, size_t max_hr_bytes, double *stats, cudaStream_t st) {
    // max_hr_bytes == 0: no stream carries ground truth, so there is no SSE pass
    KScope ks(F_STATS, st, max_hr_bytes ? 3 : 1);
    k_stats_meta<<<(S + 127) / 128, 128, 0, st>>>(d_sd, S, n, is_anchor, score, stats);
    if (max_hr_bytes) {
        // one CTA row per (stream, frame), ~4 CTAs per SM-resident wave over the frame
        const int blocks = (int)((max_hr_bytes / 16 + 255) / 256);
        dim3 g(S * n, blocks < 1 ? 1 : (blocks > 64 ? 64 : blocks));
        k_stats_sse<<<g, 256, 0, st>>>(d_sd, n, d_hr_table, stats);
        k_stats_final<<<(S + 127) / 128, 128, 0, st>>>(d_sd, S, n, stats);
    }
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
