/*
 * ns_oracle.c -- plain, slow, obviously-correct CPU oracle for the NeuroScaler
 * data-parallel enhancement hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or constant with the CUDA path
 * (paper_conf_sigcomm_yeolkjyh22_b200/csrc) and includes nothing from it.
 *
 * Citations: "P:n" = /root/reference/PAPER.md line n; "O<k>"/"Z<k>" = the
 * readings of SURVEY.md §8(c), restated in DESIGN.md "Readings".
 *
 * Precision: the paper does not state the inference precision (P:259 only
 * names TensorRT 8.0.3), so the SR network here is computed in fp64 from the
 * bf16 weight bit patterns (converted exactly).  Everything else is exact
 * integer arithmetic.
 *
 * Functions (each a direct transcription of its definition, no blocking):
 *   or_score            O2: score[f] = sum |res[f]|
 *   or_upsample         O6: fixed-point bilinear x s upsample (Z15, Z16)
 *   or_warp_plane       O7: 1/8-pel two-pass bilinear warp of an HR plane (Z14)
 *   or_reconstruct      O8: reuse-based reconstruction of a chunk
 *   or_reconstruct_i420 O8 on YUV 4:2:0 frames, chroma MC at 1/16 pel (NEXT-2; R9)
 *   (both take `interp`: 0 = the bilinear of O7 / R9, 1-4 = VP9's 8-tap
 *    sub-pel filters, NEXT-2, reading R13)
 *   or_conv3x3          3x3 cross-correlation, zero padding 1 (EDSR conv, P:306 / [89])
 *   or_pixel_shuffle    PyTorch-order pixel shuffle (EDSR upsampler)
 *   or_sr_forward       O5: the whole SR DNN on one LR frame ("8 residual
 *                       blocks, 32 channels, scale 3"; Z12, Z13)
 *
 * Anchor gain / selection (Alg. 1) lives in oracle/select.py.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

/* 8 bytes per 8x8 LR block: int16 mvx, int16 mvy (1/8 LR pel), uint8 ref,
   uint8 filter (the block's 8-tap kernel when interp = 4), 2 pad.
   Layout restated from DESIGN.md "Data layout" (not included from include/). */
typedef struct { int16_t mvx, mvy; uint8_t ref; uint8_t filter; uint8_t pad[2]; } or_mv;
enum { OR_KEY = 0, OR_ALTREF = 1, OR_NORMAL = 2 };
enum { OR_LAST = 0, OR_GOLDEN = 1, OR_INTRA = 2 };

static int64_t floor_div(int64_t a, int64_t b) { /* b > 0 */
    int64_t q = a / b;
    if ((a % b) != 0 && (a < 0)) q -= 1;
    return q;
}
static int clampi(int v, int lo, int hi) { return v < lo ? lo : (v > hi ? hi : v); }

/* ---------------------------------------------------------------- O2 score */
/* "the total residual pixel value is approximated as the size of an encoded
   residual frame".  Default: the exact total |residual| (Z8); when the
   proxy res_size is given it is used instead. */
void or_score(const int16_t *res, int n, int h, int w, const uint32_t *res_size, int64_t *score)
{
    for (int f = 0; f < n; f++) {
        if (res_size) { score[f] = (int64_t)res_size[f]; continue; }
        int64_t s = 0;
        const int16_t *r = res + (size_t)f * 3 * h * w;
        for (size_t i = 0; i < (size_t)3 * h * w; i++) s += r[i] < 0 ? -(int64_t)r[i] : (int64_t)r[i];
        score[f] = s;
    }
}

/* ---------------------------------------------------------------- O6 upsample */
/* Per axis, output coordinate X in [0, s*len): the source position is
   (X + 0.5)/s - 0.5 (half-pixel centres, Z15) = u / (2s) with u = 2X + 1 - s.
   x0 = floor(u / 2s), remainder rem = u - 2s*x0, Q7 weight of the right tap
   w1 = round_half_up(128 * rem / 2s).  Taps clamp to [0, len-1] (Z16). */
static void up_tap(int X, int s, int len, int *i0, int *i1, int *w1)
{
    int u = 2 * X + 1 - s;
    int x0 = (int)floor_div(u, 2 * s);
    int rem = u - 2 * s * x0;
    *w1 = (128 * rem + s) / (2 * s);          /* floor(128 rem/(2s) + 1/2) */
    *i0 = clampi(x0, 0, len - 1);
    *i1 = clampi(x0 + 1, 0, len - 1);
}

/* One plane, int32 in/out (caller converts u8 / i16).
   v = (128-wy)[(128-wx)P00 + wx P01] + wy[(128-wx)P10 + wx P11];
   out = floor((v + 8192) / 2^14). */
void or_upsample(const int32_t *in, int h, int w, int s, int32_t *out)
{
    int H = s * h, W = s * w;
    for (int Y = 0; Y < H; Y++) {
        int y0, y1, wy;
        up_tap(Y, s, h, &y0, &y1, &wy);
        for (int X = 0; X < W; X++) {
            int x0, x1, wx;
            up_tap(X, s, w, &x0, &x1, &wx);
            int64_t p00 = in[(size_t)y0 * w + x0], p01 = in[(size_t)y0 * w + x1];
            int64_t p10 = in[(size_t)y1 * w + x0], p11 = in[(size_t)y1 * w + x1];
            int64_t v = (128 - wy) * ((128 - wx) * p00 + wx * p01) + wy * ((128 - wx) * p10 + wx * p11);
            out[(size_t)Y * W + X] = (int32_t)floor_div(v + 8192, 16384);
        }
    }
}

/* ---------------------------------------------------------------- O7 warp */
/* HR pixel (X, Y) lies in LR block (X / 8s, Y / 8s).  Its motion vector, in
   1/8 LR pel, is scaled by the SR factor: m = s * mv (1/8 HR pel).
   pred(X, Y) = ref(X + m_x/8, Y + m_y/8) with VP9-style two-pass bilinear
   sub-pel interpolation (Z14) and edge-replicated borders (Z16):
     ix = X + floor(m_x / 8), fx = m_x mod 8 (same for y);
     h(r) = (R[r][ix] (8 - fx) + R[r][ix+1] fx + 4) >> 3   for r = iy, iy+1;
     pred = (h(iy) (8 - fy) + h(iy+1) fy + 4) >> 3.                     */
static uint8_t warp_px(const uint8_t *ref, int H, int W, int X, int Y, int mx, int my)
{
    int ix = X + (int)floor_div(mx, 8), fx = mx - 8 * (int)floor_div(mx, 8);
    int iy = Y + (int)floor_div(my, 8), fy = my - 8 * (int)floor_div(my, 8);
    int xa = clampi(ix, 0, W - 1), xb = clampi(ix + 1, 0, W - 1);
    int ya = clampi(iy, 0, H - 1), yb = clampi(iy + 1, 0, H - 1);
    int h0 = (ref[(size_t)ya * W + xa] * (8 - fx) + ref[(size_t)ya * W + xb] * fx + 4) >> 3;
    int h1 = (ref[(size_t)yb * W + xa] * (8 - fx) + ref[(size_t)yb * W + xb] * fx + 4) >> 3;
    return (uint8_t)((h0 * (8 - fy) + h1 * fy + 4) >> 3);
}

/* Warp a whole HR plane with a per-LR-block motion field (bw = w/8 blocks/row). */
void or_warp_plane(const uint8_t *ref, int H, int W, int s, const or_mv *mv, int bw, uint8_t *pred)
{
    for (int Y = 0; Y < H; Y++)
        for (int X = 0; X < W; X++) {
            const or_mv *b = &mv[(size_t)(Y / (8 * s)) * bw + X / (8 * s)];
            pred[(size_t)Y * W + X] = warp_px(ref, H, W, X, Y, s * b->mvx, s * b->mvy);
        }
}

/* ---------------------------------------------------------------- 8-tap MC (NEXT-2, R13) */
/* VP9's sub-pel interpolation kernels (libvpx vp9/common/vp9_filter.c:
   sub_pel_filters_8, _8lp, _8s), 16 phases of 8 taps, each row summing to 128
   (FILTER_BITS 7).  Index: [kernel][phase][tap], kernel 0 = EIGHTTAP
   (regular), 1 = EIGHTTAP_SMOOTH, 2 = EIGHTTAP_SHARP (libvpx's order). */
static const int OR_F8[3][16][8] = {
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

/* Read-only access for the pins (tests/test_oracle_eighttap.py). */
int or_filter8(int kernel, int phase, int tap)
{
    if (kernel < 0 || kernel > 2 || phase < 0 || phase > 15 || tap < 0 || tap > 7) return -1000;
    return OR_F8[kernel][phase][tap];
}

static int clip_pixel(int v) { return v < 0 ? 0 : (v > 255 ? 255 : v); }

/* libvpx vpx_convolve8 semantics on the HR reference, positions in 1/16 pel
   (q4): pixel (X, Y) with offset (qx, qy) samples x16 = 16 X + qx.  Horizontal
   pass over the 8 rows iy-3 .. iy+4, each clip_pixel(ROUND_POWER_OF_TWO(
   sum_k F[px][k] R[row][ix-3+k], 7)), then the vertical pass over those 8
   values with F[py]; coordinates clamped to the plane (edge replicate, Z16). */
static uint8_t warp_px8(const uint8_t *ref, int H, int W, int X, int Y, int qx, int qy, int kernel)
{
    const int64_t x16 = 16 * (int64_t)X + qx, y16 = 16 * (int64_t)Y + qy;
    const int ix = (int)floor_div(x16, 16), px = (int)(x16 - 16 * (int64_t)ix);
    const int iy = (int)floor_div(y16, 16), py = (int)(y16 - 16 * (int64_t)iy);
    int t[8];
    for (int r = 0; r < 8; r++) {
        const int yy = clampi(iy - 3 + r, 0, H - 1);
        int sum = 0;
        for (int k = 0; k < 8; k++) sum += OR_F8[kernel][px][k] * ref[(size_t)yy * W + clampi(ix - 3 + k, 0, W - 1)];
        t[r] = clip_pixel((int)floor_div(sum + 64, 128));
    }
    int sum = 0;
    for (int r = 0; r < 8; r++) sum += OR_F8[kernel][py][r] * t[r];
    return (uint8_t)clip_pixel((int)floor_div(sum + 64, 128));
}

/* The kernel a block uses: interp 1..3 -> kernel interp-1 for every block;
   interp 4 (VP9's SWITCHABLE) -> the block's own filter byte (0..2; larger
   values read as 0, include/ns.h). */
static int block_kernel(int interp, const or_mv *b) { return interp == 4 ? (b->filter > 2 ? 0 : b->filter) : interp - 1; }

/* ---------------------------------------------------------------- O8 reconstruct */
/* Frame by frame in decode order (reuse previous SR frames guided by
   reference index, MV and residual; loss resets at an anchor; the
   decoder caches SR anchors and reuses them for the others):
     anchor           : HR[f] = SR(LR[f])  (caller pre-filled hr[f])
     non-anchor KEY   : HR[f] = up_s(LR[f])                          (Z17)
     otherwise, per 8x8 LR block:
        INTRA         : up_s(LR[f])                                  (Z17)
        LAST / GOLDEN : clamp(warp(HR[ref]) + up_s(res[f]), 0, 255)
   LAST = HR[f-1] (hr_last when f = 0); GOLDEN = HR of the latest KEY/ALTREF
   before f (hr_golden when none).  up_s(res) is taken over the whole plane.
   At chunk end hr_last <- HR[n-1], hr_golden <- current GOLDEN (if non-NULL).
   hr: [n][3][s*h][s*w]; lr, res: [n][3][h][w]; mv: [n][h/8][w/8]. */
int or_reconstruct(int w, int h, int s, int n, const uint8_t *lr, const int16_t *res,
                   const or_mv *mv, const uint8_t *type, const uint8_t *is_anchor,
                   uint8_t *hr, uint8_t *hr_last, uint8_t *hr_golden, int interp)
{
    if (interp < 0 || interp > 4) return -2;
    const int H = s * h, W = s * w, bw = w / 8;
    const size_t lr_plane = (size_t)h * w, hr_plane = (size_t)H * W;
    int32_t *in = (int32_t *)malloc(lr_plane * sizeof(int32_t));
    int32_t *up_lr = (int32_t *)malloc(hr_plane * sizeof(int32_t));
    int32_t *up_res = (int32_t *)malloc(hr_plane * sizeof(int32_t));
    uint8_t *pred = (uint8_t *)malloc(hr_plane);
    if (!in || !up_lr || !up_res || !pred) { free(in); free(up_lr); free(up_res); free(pred); return -3; }
    const uint8_t *golden = hr_golden;   /* 3 planes */
    for (int f = 0; f < n; f++) {
        uint8_t *out = hr + (size_t)f * 3 * hr_plane;
        const uint8_t *last = f > 0 ? hr + (size_t)(f - 1) * 3 * hr_plane : hr_last;
        if (!is_anchor[f]) {
            const or_mv *mvf = mv + (size_t)f * (h / 8) * bw;
            for (int c = 0; c < 3; c++) {
                const uint8_t *lrp = lr + ((size_t)f * 3 + c) * lr_plane;
                const int16_t *rp = res + ((size_t)f * 3 + c) * lr_plane;
                uint8_t *op = out + (size_t)c * hr_plane;
                for (size_t i = 0; i < lr_plane; i++) in[i] = lrp[i];
                or_upsample(in, h, w, s, up_lr);
                if ((type[f] & 0x7F) == OR_KEY) {
                    for (size_t i = 0; i < hr_plane; i++) op[i] = (uint8_t)up_lr[i];
                    continue;
                }
                for (size_t i = 0; i < lr_plane; i++) in[i] = rp[i];
                or_upsample(in, h, w, s, up_res);
                for (int Y = 0; Y < H; Y++)
                    for (int X = 0; X < W; X++) {
                        const or_mv *b = &mvf[(size_t)(Y / (8 * s)) * bw + X / (8 * s)];
                        size_t i = (size_t)Y * W + X;
                        if (b->ref == OR_INTRA) { op[i] = (uint8_t)up_lr[i]; continue; }
                        const uint8_t *r = (b->ref == OR_GOLDEN ? golden : last);
                        if (!r) { free(in); free(up_lr); free(up_res); free(pred); return -1; }
                        /* R13: luma q4 offset = 2 s mv (1/8 -> 1/16 pel) */
                        int p = interp ? warp_px8(r + (size_t)c * hr_plane, H, W, X, Y, 2 * s * b->mvx, 2 * s * b->mvy,
                                                  block_kernel(interp, b))
                                       : warp_px(r + (size_t)c * hr_plane, H, W, X, Y, s * b->mvx, s * b->mvy);
                        op[i] = (uint8_t)clampi(p + up_res[i], 0, 255);
                    }
            }
        }
        if ((type[f] & 0x7F) == OR_KEY || (type[f] & 0x7F) == OR_ALTREF) golden = out;  /* R12: 0x80 = invisible */
    }
    if (hr_last && n > 0) memmove(hr_last, hr + (size_t)(n - 1) * 3 * hr_plane, 3 * hr_plane);
    if (hr_golden && golden && golden != hr_golden) memmove(hr_golden, golden, 3 * hr_plane);
    free(in); free(up_lr); free(up_res); free(pred);
    return 0;
}

/* ---------------------------------------------------------------- O8 in YUV 4:2:0 (NEXT-2) */
/* The codec's own colour format (VP9 profile 0 streams are YUV 4:2:0; SURVEY
   Z18 / §8(f) NEXT-2).  A frame is Y [h][w], then U and V [h/2][w/2]; HR the
   same at s x.  Reading R9, VP9's rule for 4:2:0: a block's
   chroma motion vector is its luma vector taken at twice the precision, i.e.
   the same number in 1/16 chroma pel (libvpx's chroma MC is the 1/16-pel
   bilinear/8-tap family; here bilinear, as O7).  So for an HR chroma pixel
   (X, Y) of the LR block (X / 4s, Y / 4s) with m = s * mv:
     ix = X + floor(m_x / 16), fx = m_x mod 16 (same for y);
     h(r) = (R[r][ix] (16 - fx) + R[r][ix+1] fx + 8) >> 4 for r = iy, iy+1;
     pred = (h(iy) (16 - fy) + h(iy+1) fy + 8) >> 4
   (= libvpx taps {128 - 8f, 8f} with FILTER_BITS 7), edge-replicated (Z16).
   Luma is O7 unchanged; up_s (O6) runs per plane at its own size. */
static uint8_t warp_px16(const uint8_t *ref, int H, int W, int X, int Y, int mx, int my)
{
    int ix = X + (int)floor_div(mx, 16), fx = mx - 16 * (int)floor_div(mx, 16);
    int iy = Y + (int)floor_div(my, 16), fy = my - 16 * (int)floor_div(my, 16);
    int xa = clampi(ix, 0, W - 1), xb = clampi(ix + 1, 0, W - 1);
    int ya = clampi(iy, 0, H - 1), yb = clampi(iy + 1, 0, H - 1);
    int h0 = (ref[(size_t)ya * W + xa] * (16 - fx) + ref[(size_t)ya * W + xb] * fx + 8) >> 4;
    int h1 = (ref[(size_t)yb * W + xa] * (16 - fx) + ref[(size_t)yb * W + xb] * fx + 8) >> 4;
    return (uint8_t)((h0 * (16 - fy) + h1 * fy + 8) >> 4);
}

/* Same decode-order rules as or_reconstruct (O8), per plane of the 4:2:0 frame.
   lr, res: [n][h*w*3/2]; hr: [n][s*h*s*w*3/2]; hr_last, hr_golden one HR frame. */
int or_reconstruct_i420(int w, int h, int s, int n, const uint8_t *lr, const int16_t *res,
                        const or_mv *mv, const uint8_t *type, const uint8_t *is_anchor,
                        uint8_t *hr, uint8_t *hr_last, uint8_t *hr_golden, int interp)
{
    if (interp < 0 || interp > 4) return -2;
    const int H = s * h, W = s * w, bw = w / 8;
    const size_t lrf = (size_t)h * w * 3 / 2, hrf = (size_t)H * W * 3 / 2;
    int32_t *in = (int32_t *)malloc((size_t)h * w * sizeof(int32_t));
    int32_t *up_lr = (int32_t *)malloc((size_t)H * W * sizeof(int32_t));
    int32_t *up_res = (int32_t *)malloc((size_t)H * W * sizeof(int32_t));
    if (!in || !up_lr || !up_res) { free(in); free(up_lr); free(up_res); return -3; }
    const uint8_t *golden = hr_golden;
    for (int f = 0; f < n; f++) {
        uint8_t *out = hr + (size_t)f * hrf;
        const uint8_t *last = f > 0 ? hr + (size_t)(f - 1) * hrf : hr_last;
        if (!is_anchor[f]) {
            const or_mv *mvf = mv + (size_t)f * (h / 8) * bw;
            for (int c = 0; c < 3; c++) {
                /* plane geometry: luma full size, chroma half size; offset in the frame */
                const int ph = c ? h / 2 : h, pw = c ? w / 2 : w, PH = s * ph, PW = s * pw;
                const size_t lo = c == 0 ? 0 : (size_t)h * w + (size_t)(c - 1) * ph * pw;
                const size_t ho = c == 0 ? 0 : (size_t)H * W + (size_t)(c - 1) * PH * PW;
                const int blk = c ? 4 * s : 8 * s;            /* HR pixels per LR block side */
                const uint8_t *lrp = lr + (size_t)f * lrf + lo;
                const int16_t *rp = res + (size_t)f * lrf + lo;
                uint8_t *op = out + ho;
                for (size_t i = 0; i < (size_t)ph * pw; i++) in[i] = lrp[i];
                or_upsample(in, ph, pw, s, up_lr);
                if ((type[f] & 0x7F) == OR_KEY) {
                    for (size_t i = 0; i < (size_t)PH * PW; i++) op[i] = (uint8_t)up_lr[i];
                    continue;
                }
                for (size_t i = 0; i < (size_t)ph * pw; i++) in[i] = rp[i];
                or_upsample(in, ph, pw, s, up_res);
                for (int Y = 0; Y < PH; Y++)
                    for (int X = 0; X < PW; X++) {
                        const or_mv *b = &mvf[(size_t)(Y / blk) * bw + X / blk];
                        size_t i = (size_t)Y * PW + X;
                        if (b->ref == OR_INTRA) { op[i] = (uint8_t)up_lr[i]; continue; }
                        const uint8_t *r = (b->ref == OR_GOLDEN ? golden : last);
                        if (!r) { free(in); free(up_lr); free(up_res); return -1; }
                        /* R13: q4 offset = 2 s mv for luma, s mv for chroma (already 1/16 chroma pel, R9) */
                        int p = interp ? warp_px8(r + ho, PH, PW, X, Y, (c ? 1 : 2) * s * b->mvx, (c ? 1 : 2) * s * b->mvy,
                                                  block_kernel(interp, b))
                              : c ? warp_px16(r + ho, PH, PW, X, Y, s * b->mvx, s * b->mvy)
                                  : warp_px(r + ho, PH, PW, X, Y, s * b->mvx, s * b->mvy);
                        op[i] = (uint8_t)clampi(p + up_res[i], 0, 255);
                    }
            }
        }
        if ((type[f] & 0x7F) == OR_KEY || (type[f] & 0x7F) == OR_ALTREF) golden = out;  /* R12: 0x80 = invisible */
    }
    if (hr_last && n > 0) memmove(hr_last, hr + (size_t)(n - 1) * hrf, hrf);
    if (hr_golden && golden && golden != hr_golden) memmove(hr_golden, golden, hrf);
    free(in); free(up_lr); free(up_res);
    return 0;
}

/* ---------------------------------------------------------------- SR (O5) */
/* 3x3 cross-correlation with zero padding 1 (PyTorch Conv2d semantics):
   out[co][y][x] = b[co] + sum_{ci,ky,kx} W[co][ci][ky][kx] in[ci][y+ky-1][x+kx-1]. */
void or_conv3x3(const double *in, int cin, int h, int w, const double *wt, const double *bias,
                int cout, double *out)
{
    #pragma omp parallel for schedule(dynamic, 1)
    for (int co = 0; co < cout; co++) {
        double *o = out + (size_t)co * h * w;
        for (size_t i = 0; i < (size_t)h * w; i++) o[i] = bias ? bias[co] : 0.0;
        for (int ci = 0; ci < cin; ci++)
            for (int ky = 0; ky < 3; ky++)
                for (int kx = 0; kx < 3; kx++) {
                    const double wv = wt[(((size_t)co * cin + ci) * 3 + ky) * 3 + kx];
                    const double *ip = in + (size_t)ci * h * w;
                    for (int y = 0; y < h; y++) {
                        int yy = y + ky - 1;
                        if (yy < 0 || yy >= h) continue;
                        for (int x = 0; x < w; x++) {
                            int xx = x + kx - 1;
                            if (xx < 0 || xx >= w) continue;
                            o[(size_t)y * w + x] += wv * ip[(size_t)yy * w + xx];
                        }
                    }
                }
    }
}

/* PyTorch PixelShuffle: out[c][s*y+i][s*x+j] = in[c*s*s + i*s + j][y][x]. */
void or_pixel_shuffle(const double *in, int cout, int h, int w, int s, double *out)
{
    const int H = s * h, W = s * w;
    for (int c = 0; c < cout; c++)
        for (int i = 0; i < s; i++)
            for (int j = 0; j < s; j++)
                for (int y = 0; y < h; y++)
                    for (int x = 0; x < w; x++)
                        out[((size_t)c * H + s * y + i) * W + s * x + j] =
                            in[(((size_t)c * s * s + i * s + j) * h + y) * w + x];
}

static double bf16_to_double(uint16_t b)
{
    uint32_t u = (uint32_t)b << 16;
    float f;
    memcpy(&f, &u, 4);
    return (double)f;
}

/* Number of uint16 entries in the weight blob: head, B x (conv1, conv2), end,
   up, tail; each [Cout][Cin][3][3] followed by bias[Cout]. */
size_t or_blob_len(int B, int C, int s)
{
    size_t n = (size_t)C * 3 * 9 + C;
    n += (size_t)2 * B * ((size_t)C * C * 9 + C);
    n += (size_t)C * C * 9 + C;
    n += (size_t)s * s * C * C * 9 + (size_t)s * s * C;
    n += (size_t)3 * C * 9 + 3;
    return n;
}

/* Reads one conv's weights+bias (as fp64) from the blob cursor. */
static const uint16_t *take_conv(const uint16_t *p, int cout, int cin, double **wt, double **bias)
{
    size_t nw = (size_t)cout * cin * 9;
    *wt = (double *)malloc(nw * sizeof(double));
    *bias = (double *)malloc((size_t)cout * sizeof(double));
    for (size_t i = 0; i < nw; i++) (*wt)[i] = bf16_to_double(p[i]);
    for (int i = 0; i < cout; i++) (*bias)[i] = bf16_to_double(p[nw + i]);
    return p + nw + cout;
}

/* O5: the SR network on one LR frame [3][h][w] (u8), weights = bf16 blob.
     x  = LR - 128                                             (Z13)
     h0 = conv(x; head)
     h  = h0; for b in 1..B: h = h + conv(ReLU(conv(h; b.1)); b.2)   (EDSR block,
                                                no BN, res_scale 1; [89] P:541)
     h  = h0 + conv(h; end)                                   (global skip)
     u  = pixel_shuffle(conv(h; up), s)                       (upsampler)
     t  = conv(u; tail)                                       (HR tail, C -> 3)
     out = clamp(floor(up_s(LR) + t + 0.5), 0, 255)           (Z12: integer
                                                bilinear skip, O6)
   out: [3][s*h][s*w] u8.  t_out (optional, [3][s*h][s*w] fp64) receives t.
   Returns 0, or -3 on allocation failure. */
int or_sr_forward(const uint8_t *lr, int h, int w, int B, int C, int s, const uint16_t *blob,
                  uint8_t *out, double *t_out)
{
    const size_t P = (size_t)h * w, HP = (size_t)s * s * P;
    const int H = s * h, W = s * w;
    double *x = (double *)malloc(3 * P * sizeof(double));
    double *h0 = (double *)malloc((size_t)C * P * sizeof(double));
    double *hh = (double *)malloc((size_t)C * P * sizeof(double));
    double *t1 = (double *)malloc((size_t)C * P * sizeof(double));
    double *t2 = (double *)malloc((size_t)C * P * sizeof(double));
    double *upc = (double *)malloc((size_t)s * s * C * P * sizeof(double));
    double *u = (double *)malloc((size_t)C * HP * sizeof(double));
    double *t = (double *)malloc(3 * HP * sizeof(double));
    int32_t *lin = (int32_t *)malloc(P * sizeof(int32_t));
    int32_t *lup = (int32_t *)malloc(HP * sizeof(int32_t));
    int rc = 0;
    if (!x || !h0 || !hh || !t1 || !t2 || !upc || !u || !t || !lin || !lup) { rc = -3; goto done; }

    for (size_t i = 0; i < 3 * P; i++) x[i] = (double)lr[i] - 128.0;
    const uint16_t *p = blob;
    double *wt, *bias;

    p = take_conv(p, C, 3, &wt, &bias);
    or_conv3x3(x, 3, h, w, wt, bias, C, h0);
    free(wt); free(bias);
    memcpy(hh, h0, (size_t)C * P * sizeof(double));

    for (int b = 0; b < B; b++) {
        p = take_conv(p, C, C, &wt, &bias);
        or_conv3x3(hh, C, h, w, wt, bias, C, t1);
        free(wt); free(bias);
        for (size_t i = 0; i < (size_t)C * P; i++) t1[i] = t1[i] > 0.0 ? t1[i] : 0.0;
        p = take_conv(p, C, C, &wt, &bias);
        or_conv3x3(t1, C, h, w, wt, bias, C, t2);
        free(wt); free(bias);
        for (size_t i = 0; i < (size_t)C * P; i++) hh[i] += t2[i];
    }
    p = take_conv(p, C, C, &wt, &bias);
    or_conv3x3(hh, C, h, w, wt, bias, C, t2);
    free(wt); free(bias);
    for (size_t i = 0; i < (size_t)C * P; i++) hh[i] = h0[i] + t2[i];

    p = take_conv(p, s * s * C, C, &wt, &bias);
    or_conv3x3(hh, C, h, w, wt, bias, s * s * C, upc);
    free(wt); free(bias);
    or_pixel_shuffle(upc, C, h, w, s, u);

    p = take_conv(p, 3, C, &wt, &bias);
    or_conv3x3(u, C, H, W, wt, bias, 3, t);
    free(wt); free(bias);

    for (int c = 0; c < 3; c++) {
        for (size_t i = 0; i < P; i++) lin[i] = lr[(size_t)c * P + i];
        or_upsample(lin, h, w, s, lup);
        for (size_t i = 0; i < HP; i++) {
            double v = floor((double)lup[i] + t[(size_t)c * HP + i] + 0.5);
            out[(size_t)c * HP + i] = (uint8_t)(v < 0.0 ? 0.0 : (v > 255.0 ? 255.0 : v));
        }
    }
    if (t_out) memcpy(t_out, t, 3 * HP * sizeof(double));
done:
    free(x); free(h0); free(hh); free(t1); free(t2); free(upc); free(u); free(t); free(lin); free(lup);
    return rc;
}

/* PSNR over all 3 planes, capped at 100 dB. */
double or_psnr(const uint8_t *a, const uint8_t *b, size_t n)
{
    double sse = 0.0;
    for (size_t i = 0; i < n; i++) { double d = (double)a[i] - (double)b[i]; sse += d * d; }
    if (sse == 0.0) return 100.0;
    double p = 10.0 * log10(255.0 * 255.0 / (sse / (double)n));
    return p > 100.0 ? 100.0 : p;
}
