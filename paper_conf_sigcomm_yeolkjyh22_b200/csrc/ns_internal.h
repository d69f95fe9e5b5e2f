// ns_internal.h -- shared host/device definitions of libneuroscaler (not ABI).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstddef>
#include <atomic>
#include <vector>
#include "../../include/ns.h"

namespace ns {

constexpr int kMaxFrames = 256;
constexpr int kTile = 128;        // output pixels per UMMA M tile (one row segment)
constexpr int kHalo = kTile + 2;  // input pixels per tile row (3x3 halo)

// Device-side per-stream descriptor (built by the host from ns_chunk).
struct StreamDesc {
    const uint8_t *lr;
    const int16_t *res;
    const ns_block_mv *mv;
    const uint8_t *type;
    const uint32_t *res_size;
    uint8_t *hr_last;
    uint8_t *hr_golden;
    const uint8_t *gt;
    const uint8_t *wts;    // packed model operands (see model layout below)
    int32_t w, h, s, n;
    int32_t hr_base;       // index of hr_out[s][0] in the device hr table
    int32_t group;         // SR shape group index (ns_enhance_streams)
    int32_t job_base;      // first SR job slot of this stream in its group
    int32_t job_cap;       // slots of its group; a given anchor map's anchors beyond it are demoted (ns.h)
    int32_t use_res_size;
    int32_t job_goff;      // first job slot of the stream's SR shape group
    int32_t fmt;           // NS_FMT_444 | NS_FMT_I420
    int32_t interp;        // NS_INTERP_* (k_recon_step: bilinear streams; k_recon8: the 8-tap ones)
    int64_t lr_frame;      // elements per LR / residual frame: 3 h w, or h w 3/2 (I420)
    int64_t hr_frame;      // bytes per HR frame: 3 H W, or H W 3/2 (I420)
    uint8_t *acache;       // HR rings: the group's anchor cache (job slot j at acache + (j - job_goff) * stride)
    uint64_t acache_stride;
};

// Per (stream, frame) reconstruction step descriptor, resolved once per chunk
// after selection (k_frame_desc): a recon CTA reads its 64 B and can start
// staging at once, instead of walking sd -> type / is_anchor / gold -> hr table.
struct __align__(16) FrameDesc {
    const uint8_t *lr_f;       // LR[f] [3][h][w]
    const int16_t *res_f;      // res[f] [3][h][w]
    const ns_block_mv *mv_f;   // mv[f] [h/8][w/8]
    uint8_t *out;              // HR[f]
    const uint8_t *ref_last;   // HR[f-1] or hr_last
    const uint8_t *ref_gold;   // HR of the latest KEY/ALTREF g < f (its copy in hr_golden from step
                               // g+2 on when g was saved), or hr_golden
    const uint8_t *asrc;       // an anchor whose slot an earlier frame uses (HR ring): its SR output
                               // in the anchor cache, copied to out at this step
    const uint8_t *gsave_src;  // f-1 is a KEY/ALTREF frame whose ring slot is reused while it is still
    uint8_t *gsave_dst;        // GOLDEN: HR[f-1] is saved into hr_golden (= gsave_dst) at this step
    int32_t w, h;              // LR size
    int16_t s;                 // scale
    uint8_t anchor, key;       // is_anchor[f], type[f] == KEY
    int32_t fmt;               // NS_FMT_444 | NS_FMT_I420
    int32_t interp;            // NS_INTERP_*: 0 -> k_recon_step, else k_recon8
    int32_t pad2;
};
static_assert(sizeof(FrameDesc) == 96, "FrameDesc is one 96-B record");

// One anchor-SR job (device).
struct SrJob {
    const uint8_t *lr;     // [3][h][w]
    uint8_t *hr;           // [3][s*h][s*w]
    const uint8_t *wts;    // packed model operands
};

// Packed model: per layer L a UMMA B operand (bf16, K-major core matrices)
// [split][tap 9][kc CIN/16][kh 2][n NT][8] followed by fp32 bias[NTOT],
// each region 128-B aligned.  Layers: 0 head (CIN 16, 3 real), 1..2B body,
// 2B+1 end, 2B+2 up (NTOT = s*s*C, rows permuted to (i, j, c) order for the
// fused pixel shuffle), 2B+3 tail (NTOT = 16, 3 real).
// Rotated layers (rot = 1: head, body, end, tail) instead hold, per tap column
// dx and 16-channel K chunk, a 5-block strip [W_dy2; W_dy1; W_dy0; W_dy2;
// W_dy1] of nb output rows each: [dx 3][kc][kh 2][5 nb][8] bf16, then fp32
// bias[nb] (see k_conv_rot).
struct LayerShape {
    int cin, cin_real, ntot, nsplit, cout_real;
    int perm;              // 0 none, 1 pixel-shuffle permutation
    int rot, nb;           // rotated-accumulator layout and its block width
    size_t b_off, bias_off, bytes;  // offsets from the model base
};

int model_num_layers(int n_blocks);
LayerShape model_layer(int n_blocks, int C, int s, int L);
size_t model_packed_bytes(int n_blocks, int C, int s);

// Derived regions after the blob layers:
//  * COMP: tail o pixel-shuffle o upsampler composed into one 5x5 conv at LR
//    resolution, h (C ch) -> s*s*3 outputs (n = (i*s + j)*3 + co), padded to nb;
//    UMMA B operand of the rotated 5x5 conv: [tx 5][kc][kh 2][nstrip nb][8] bf16,
//    then fp32 bias[nb].
//  * AUX (fp32, for the exact frame-border fix-up): W_up [s*s*C][C][9], b_up,
//    W_tail [3][C][9], b_tail, then the composed Wc [s*s*3][C][25], bc [s*s*3].
struct CompShape {
    int nb;                  // padded outputs per block (16 | 32 | 48)
    int nstrip;              // strip blocks: 9 = [4,3,2,1,0,4,3,2,1] (5-block window)
    size_t b_off, bias_off;  // composed operand / bias
    size_t aux_off;          // fp32 W_up, b_up, W_tail, b_tail (contiguous)
};
CompShape model_comp(int n_blocks, int C, int s);

// ------------------------------------------------------------ launch wrappers
// Every launch goes through these (kernels live in k_*.cu); each returns the
// cudaError_t of the launch.  `st` is the stream.
cudaError_t launch_score(const StreamDesc *d_sd, int S, int n, int max_frame_vec8, int64_t *score,
                         cudaStream_t st);
cudaError_t launch_select(const StreamDesc *d_sd, const int64_t *score, int S, int n, int k, int fresh,
                          int selector, int64_t *gain, int32_t *rank, uint8_t *is_anchor, int32_t *order,
                          cudaStream_t st);
// ns_select_merge: global selection over gathered [S][n] gain / rank / type arrays.
cudaError_t launch_merge(int S, int n, const int64_t *gain, const int32_t *rank_in, const uint8_t *type,
                         const int32_t *sid, const int64_t *cost, int64_t budget, int32_t *order, int32_t *grank,
                         int32_t *pos_stream, int32_t *cut, int32_t *rank, uint8_t *is_anchor, cudaStream_t st);
cudaError_t launch_global(const StreamDesc *d_sd, int S, int n, const int64_t *gain, const int32_t *order,
                          const int64_t *cost, int64_t budget, int32_t *grank, int32_t *pos_stream,
                          int32_t *cut, int32_t *rank, uint8_t *is_anchor, cudaStream_t st);
// Anchors -> SR job slots.  topk: stream s owns slots [job_base, job_base + k).
// Otherwise slots are assigned deterministically, stream by stream in each
// group's list order (glist / goff: the streams of group g are
// glist[goff[g] .. goff[g+1])), and anchors beyond the group's job_cap are
// demoted (is_anchor cleared: the frame is reconstructed instead).  acount:
// [S] scratch.  HR rings (else both NULL): prv [S][n] = the previous frame of
// the stream writing the same hr_out entry (-1: none); an anchor with prv >= 0
// is SR'd into the anchor cache and asrc[s][f] records where.
cudaError_t launch_compact(const StreamDesc *d_sd, int S, int n, uint8_t *is_anchor, uint8_t *const *d_hr_table,
                           SrJob *jobs, int32_t *job_count, int n_groups, const int32_t *glist,
                           const int32_t *goff, int32_t *acount, int topk, const int16_t *prv,
                           const uint8_t **asrc, cudaStream_t st,
                           uint8_t *lr_stage = nullptr, size_t lr_stride = 0, const uint8_t **lr_src = nullptr,
                           uint32_t *lr_len = nullptr);
// Copies every filled job's LR frame (lr_len[j] > 0) from lr_src[j] (host-mapped
// memory) to jobs[j].lr (device staging set by launch_compact).
cudaError_t launch_lr_gather(const SrJob *jobs, const uint8_t *const *lr_src, const uint32_t *lr_len, int max_jobs,
                             size_t max_len, cudaStream_t st);
// gold [S][n+1]; HR rings (nxt [S][n] = the next frame writing the same hr_out
// entry, n: none): gsv [S][n] = 1 for a KEY/ALTREF frame that must be saved into
// hr_golden because its slot is reused while it is GOLDEN; nxt = NULL: no saves.
cudaError_t launch_golden_index(const StreamDesc *d_sd, int S, int n, const int16_t *nxt, int16_t *gold_idx,
                                uint8_t *gsv, cudaStream_t st);
// max_lr_w / max_lr_h: [5] indexed by scale (0 = no stream of that scale)
// fd[s][f] for all streams and frames (after launch_golden_index)
// gsv / asrc: from launch_golden_index / launch_compact for HR rings, else NULL
cudaError_t launch_frame_desc(const StreamDesc *d_sd, int S, int n, const uint8_t *is_anchor,
                              uint8_t *const *d_hr_table, const int16_t *gold_idx, const uint8_t *gsv,
                              const uint8_t *const *asrc, FrameDesc *fd, cudaStream_t st);
// max_lr_w / max_lr_h: [5] per scale; has_i420[5]: a 4:2:0 stream of that scale
// (its chroma planes then step in k_recon_step<s, true> in the same frame
// step); e8[5]: bit 0 an 8-tap stream of that scale (k_recon8), bit 1 an
// 8-tap 4:2:0 one (k_recon8<s, true> for its chroma).  Streams [s0, s0 + S)
// of the frame-descriptor table.
cudaError_t launch_recon_step(const FrameDesc *fd, int S, int n, int f, const int *max_lr_w, const int *max_lr_h,
                              const int *has_i420, const int *e8, cudaStream_t st, int s0 = 0);
cudaError_t launch_state_copy(const StreamDesc *d_sd, int S, int n, uint8_t *const *d_hr_table,
                              const int16_t *gold_idx, const uint8_t *gsv, size_t max_hr_bytes, cudaStream_t st);
cudaError_t launch_stats(const StreamDesc *d_sd, int S, int n, const uint8_t *is_anchor, const int64_t *score,
                         uint8_t *const *d_hr_table, size_t max_hr_bytes, double *stats, cudaStream_t st);
cudaError_t launch_repack(const uint16_t *blob, int n_blocks, int C, int s, uint8_t *packed, cudaStream_t st);

// SR (k_sr.cu)
struct SrArena {
    int h, w, C, s, nb;        // shape and batch capacity (jobs per batch)
    int fmt;                   // NS_FMT_444 | NS_FMT_I420 (input conversion, output packing)
    uint8_t *hr_tmp;           // I420: the net's full-resolution HR output [job][3][sH][sW], packed to 4:2:0 after
    uint16_t *x0, *h0, *hb, *tb;       // bf16 activations, layout [job][H][C/8][W][8]
    float *band;                       // border fix-up: u on the HR frame-edge bands
    uint8_t *lr8;                      // u8 LR copy [job][H][3][wp] (upsampler skip taps), wp = W rounded to 16
    int wp;
    CUtensorMap tm_x0, tm_h0, tm_hb, tm_tb, tm_tb5, tm_hb5;   // *5: 132-px boxes (5x5 conv)
    CUtensorMap tm_lr8;                // box: kLrBoxW px x 3 planes x 3 rows
};
int sr_batch_jobs(int h, int w, int sms);  // jobs per SR batch of one shape (k_sr.cu)
size_t sr_arena_bytes(int h, int w, int C, int s, int nb, int fmt);
int sr_arena_init(SrArena *a, int h, int w, int C, int s, int nb, int fmt, uint8_t *mem);  // 0 ok
// Runs the whole net on jobs [j0, j0+nj) of a device job table (all of one
// shape).  job_count (device) may be NULL; otherwise CTAs of jobs >= *job_count exit.
cudaError_t sr_run_batch(const SrArena *a, int n_blocks, const SrJob *jobs, int j0, int nj,
                         const int32_t *job_count, cudaStream_t st);

// Sets a kernel's dynamic shared memory limit (and, optionally, the preferred
// shared-memory carveout in percent of the unified L1/shared array) once per
// DEVICE: function attributes belong to the context of the device current at
// the call, and a process may drive several devices (ns.h: one context per
// device).  One flag word per kernel instantiation (template on the kernel
// pointer), bit d = device d done; thread-safe.
template <auto K>
cudaError_t ensure_kernel_smem(int bytes, int carveout_pct = -1) {
    static std::atomic<unsigned long long> done{0};
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e != cudaSuccess) return e;
    const unsigned long long bit = 1ull << (dev & 63);
    if (done.load(std::memory_order_acquire) & bit) return cudaSuccess;
    e = cudaFuncSetAttribute(K, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    if (e == cudaSuccess && carveout_pct >= 0)
        e = cudaFuncSetAttribute(K, cudaFuncAttributePreferredSharedMemoryCarveout, carveout_pct);
    if (e == cudaSuccess) done.fetch_or(bit, std::memory_order_release);
    return e;
}

// Hybrid encoding (ns_hybrid.cu, nvJPEG)
int hybrid_quality_table2(int n_anchors, int n_frames);
struct HybridEncoder;
int hybrid_create(int device, cudaStream_t stream, HybridEncoder **out, char *err, size_t errlen);
void hybrid_destroy(HybridEncoder *e);
struct HybridFrame {
    const uint8_t *hr;   // HR frame planes (device)
    int H, W, fmt, quality;
};
int hybrid_encode_frames(HybridEncoder *e, int n, const HybridFrame *fr, std::vector<std::vector<uint8_t>> &out,
                         cudaStream_t stream, char *err, size_t errlen);

// Kernel families for ns_launch_count / ns_profile_read.
enum Fam { F_SCORE = 0, F_SELECT, F_GLOBAL, F_COMPACT, F_SR_PREP, F_SR_HEAD, F_SR_BODY, F_SR_END, F_SR_UP,
           F_SR_TAIL, F_RECON, F_STATE, F_STATS, F_REPACK, F_COUNT };
const char *fam_name(int fam);

// Wraps the launch(es) of one kernel family on stream `st`: counts launches
// and, when profiling is enabled, brackets them with CUDA events.
struct KScope {
    int fam, n;
    cudaStream_t st;
    void *rec;
    KScope(int fam, cudaStream_t st, int n = 1);
    ~KScope();
};

}  // namespace ns
