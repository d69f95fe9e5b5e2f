/*
 * ns.h -- C ABI of libneuroscaler.so: the data-parallel enhancement hot path of
 * NeuroScaler (SIGCOMM '22), B200-native (sm_100a).
 *
 * "NeuroScaler takes an ingest stream and a DNN pair and outputs a
 *  high-resolution stream" (§4).  Per stream and per chunk the
 * library (1) scores frames from codec metadata and selects anchor frames
 * without inference (§5.1, Alg. 1), (2) runs the
 * stream's content-aware SR DNN on the anchors only (§6.2), and (3)
 * rebuilds every other frame by reusing cached SR frames guided by reference
 * index, motion vector and residual (§2, §6.1).  Many streams
 * are batched per call, so one kernel serves many streams without GPU
 * context switches (§6.2).
 *
 * Conventions (all calls):
 *  - Every pointer inside ns_chunk / ns_sr_job and every output array is a
 *    DEVICE pointer owned by the caller, unless a comment says "host".
 *  - Every call is asynchronous on `stream` (a cudaStream_t; NULL = legacy
 *    default stream).  The library performs no host synchronisation on the
 *    hot path and no device allocation after ns_ctx_create (memory
 *    pre-allocation, App. A): working memory is carved
 *    from the context pool.
 *  - Arguments are validated on the host before anything is enqueued; on any
 *    error nothing is launched, the call returns a negative ns_status and
 *    ns_last_error() describes the problem.
 *  - A context is bound to one device and is not thread-safe; use one context
 *    per device per host thread.
 *
 * Data layout:
 *  - LR frames u8, 3 full-resolution planes [n][3][h][w]; residual int16
 *    [n][3][h][w] with values in [-255, 255]; HR frames u8 [3][s*h][s*w].
 *  - Motion: one ns_block_mv per 8x8 LR block, [n][h/8][w/8], MVs in 1/8 LR
 *    pel, pred(x) = ref(x + mv) (reading Z14).
 */
#ifndef NEUROSCALER_NS_H
#define NEUROSCALER_NS_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define NS_API __attribute__((visibility("default")))
#else
#define NS_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    NS_OK = 0,
    NS_EINVAL = -1,        /* invalid argument (see ns_last_error)              */
    NS_ECUDA = -2,         /* a CUDA runtime error; message includes its string */
    NS_ENOMEM = -3,        /* the context pool is too small for the request     */
    NS_EUNSUPPORTED = -4   /* device is not sm_100 / shape not supported        */
} ns_status;

/* Frame types exported by the decoder (G_key, G_altref, G_normal).
   Codec neutrality (§9): "to support the H.26x codecs, we only need to
   replace the VPx-/AV1-specific frame groups (G_key, G_altref, G_normal) with
   the H.26x-specific groups (G_I, G_P, G_B)" -- the same three tiers, so an
   H.26x decoder exports I as the key tier (reset points, selected first), P
   as the high-reference tier and B as the normal tier (reading R8, DESIGN.md
   §3; GOLDEN is then the latest I/P frame in decode order). */
typedef enum {
    NS_KEY = 0, NS_ALTREF = 1, NS_NORMAL = 2,
    NS_I = NS_KEY, NS_P = NS_ALTREF, NS_B = NS_NORMAL
} ns_frame_type;
/* Invisible frames (NEXT-2): VP9's alternative reference frames are "invisible
   frames only used for interframe compression", shown later by an
   overlay frame.  NS_INVISIBLE OR'ed into a type byte marks a frame that is
   selected in its group, enhanced and kept as a reference exactly like a
   visible one, but not displayed: the stats count and score only displayed
   frames (reading R12).  Every call masks the type with NS_TYPE_MASK. */
#define NS_INVISIBLE 0x80
#define NS_TYPE_MASK 0x7F

/* Reference index of a block ("reference index"). */
typedef enum { NS_REF_LAST = 0, NS_REF_GOLDEN = 1, NS_REF_INTRA = 2 } ns_ref;

/* One 8x8 LR block's motion vector (1/8 LR pel) and reference. 8 bytes.
   A codec's larger partitions (VP9 16x16 .. 64x64) are their vector repeated
   on every 8x8 block they cover (reading R14). */
typedef struct {
    int16_t mvx, mvy;
    uint8_t ref;        /* ns_ref */
    uint8_t filter;     /* NS_INTERP_SWITCHABLE chunks: this block's 8-tap kernel,
                           0 EIGHTTAP, 1 EIGHTTAP_SMOOTH, 2 EIGHTTAP_SHARP (values
                           above 2 read as 0); ignored otherwise               */
    uint8_t pad[2];
} ns_block_mv;

/* Sub-pel motion compensation of a stream (ns_chunk.interp; SURVEY §8(f)
   NEXT-2, reading R13).  P:89 names "lightweight bilinear interpolation":
   NS_INTERP_BILINEAR (0, the default) is the two-pass bilinear of reading
   Z14 (R9 for 4:2:0 chroma).  The others are VP9's own sub-pel filters
   (libvpx vpx_convolve8 semantics), so a reused frame is predicted the way
   the decoder predicted its LR frame: positions in 1/16 pel (2 s mv for luma,
   s mv for 4:2:0 chroma), 8 taps at -3..+4, each pass rounded by 7 bits and
   clipped to a byte, edges replicated.  SWITCHABLE takes the kernel per block
   (ns_block_mv.filter), as VP9's per-block interp_filter. */
enum {
    NS_INTERP_BILINEAR = 0,
    NS_INTERP_EIGHTTAP = 1,         /* libvpx sub_pel_filters_8   */
    NS_INTERP_EIGHTTAP_SMOOTH = 2,  /* libvpx sub_pel_filters_8lp */
    NS_INTERP_EIGHTTAP_SHARP = 3,   /* libvpx sub_pel_filters_8s  */
    NS_INTERP_SWITCHABLE = 4
};

typedef struct ns_ctx ns_ctx;
typedef struct ns_model ns_model;

/* Frame formats (codec-faithful formats).
   NS_FMT_444:  three full-resolution planes per frame (reading Z18), the
                layouts given below.
   NS_FMT_I420: the codec's YUV 4:2:0 -- Y [h][w], then U, V [h/2][w/2] per LR
                frame (lr u8, res int16), the same at s x per HR frame; w and
                h multiples of 16 (whole 8x8 chroma blocks).  Motion
                vectors stay one per 8x8 luma block; the chroma planes use the
                block's vector read in 1/16 chroma pel (VP9's 4:2:0 rule,
                reading R9) with the 16-phase bilinear.  An anchor is SR'd by
                the 4:4:4 net on (Y, up_2(U), up_2(V)) and its HR chroma taken
                back to 4:2:0 by the rounded 2x2 average (reading R10). */
enum { NS_FMT_444 = 0, NS_FMT_I420 = 1 };

/* One stream's chunk (= GOP of n_frames frames) as the decoder exports it
   (frame type and residual; reference index, MV). */
typedef struct {
    int32_t w, h;              /* LR size; w % 8 == 0, h % 8 == 0, w,h >= 8         */
    int32_t scale;             /* SR factor s in {2, 3, 4}; must equal model scale   */
    int32_t n_frames;          /* 1 <= n <= 256; per call S <= 65535, S * n <= 2^20  */
    const uint8_t *lr;         /* [n][3][h][w] decoded LR frames                     */
    const int16_t *res;        /* [n][3][h][w] decoded residual                      */
    const ns_block_mv *mv;     /* [n][h/8][w/8]                                      */
    const uint8_t *type;       /* [n] ns_frame_type                                  */
    const uint32_t *res_size;  /* [n] optional encoded-size proxy or NULL    */
    const ns_model *model;     /* this stream's content-aware DNN             */
    uint8_t *hr_last;          /* [3][s*h][s*w] LAST reference entering the chunk;
                                  overwritten with HR[n-1] at chunk end. May be NULL
                                  if no frame references LAST before a KEY frame.  */
    uint8_t *hr_golden;        /* [3][s*h][s*w] GOLDEN reference entering the chunk;
                                  overwritten with the chunk's last KEY/ALTREF HR.
                                  May be NULL under the same condition.            */
    const uint8_t *gt;         /* optional [n][3][s*h][s*w] ground truth for stats   */
    int32_t format;            /* NS_FMT_444 (0, the layouts above) | NS_FMT_I420   */
    int32_t interp;            /* NS_INTERP_* (0 = bilinear); the codec's MC filter */
} ns_chunk;

/* Anchor selection mode (§5.1 top-k per chunk; §5.2 global budget).
   NS_GIVEN_ANCHORS: the anchor map was decided elsewhere -- by ns_select_merge
   over the streams of every GPU (§5.2 global selection across GPUs)
   -- and is passed in `anchor_in`; `cost` and `budget` are those of that global
   selection (this call's streams' entries of cost[]), which bound the anchors
   this call can receive (sum of their cost <= budget).  A map that breaks that
   bound is not an error (it is device data): per SR shape group the anchors
   take job slots stream by stream, frame by frame, and those beyond the
   group's min(streams * n, budget / min cost) slots are DEMOTED -- their
   is_anchor_out entry is cleared and the frame is reconstructed like any
   other non-anchor frame (deterministic; nothing is left stale).  Only
   ns_enhance_streams and ns_enhance_streams_host accept it. */
enum { NS_TOPK_PER_STREAM = 0, NS_GLOBAL_BUDGET = 1, NS_GIVEN_ANCHORS = 2 };
/* Residual carried from the G_altref pass into the G_normal pass (reading Z2,
   default) or recomputed per group (literal Alg. 1 line 2). */
enum { NS_CARRY = 0, NS_FRESH = 1 };
/* Anchor selector (top-k mode only).  NS_SEL_NEUROSCALER: Alg. 1 + Fig. 10.
   The two real-time baselines of §3:
     NS_SEL_KEY          "Key SR": key frames only -- the first min(k, #key)
                         key frames (k = n: every key frame; reading R6);
     NS_SEL_KEY_UNIFORM  "Key+Uniform SR": key frames, then the equally spaced
                         frames U = { floor(j*n/k) : 0 <= j < k } (reading R5),
                         priority (key asc, U asc, rest asc), first k anchors.
   Per-frame SR is top-k with k = n under any selector.  gain is
   INT64_MAX for key frames and 0 otherwise under the baselines. */
enum { NS_SEL_NEUROSCALER = 0, NS_SEL_KEY = 1, NS_SEL_KEY_UNIFORM = 2 };

typedef struct {
    int32_t mode;              /* NS_TOPK_PER_STREAM | NS_GLOBAL_BUDGET | NS_GIVEN_ANCHORS */
    int32_t k;                 /* top-k mode: anchors per stream, 0 <= k <= n         */
    int64_t budget;            /* global / given mode: T_intv * M in cost units */
    const int64_t *cost;       /* HOST [S]: T_DNN of one anchor of stream s, >= 1     */
    int32_t group_residual;    /* NS_CARRY | NS_FRESH                                 */
    int32_t use_res_size;      /* 1: score = res_size (P:191 proxy) when non-NULL     */
    int32_t selector;          /* NS_SEL_* (top-k mode; 0 otherwise)                  */
    int32_t reserved;          /* 0                                                   */
    const uint8_t *anchor_in;  /* NS_GIVEN_ANCHORS: DEVICE [S][n] 0/1, else NULL      */
} ns_select_params;

/* One anchor-SR job: HR = SR_model(LR) (O5). */
typedef struct {
    const ns_model *model;
    const uint8_t *lr;         /* [3][h][w] (NS_FMT_I420: Y, U, V planes of 4:2:0)     */
    int32_t w, h;
    uint8_t *hr_out;           /* [3][s*h][s*w] (NS_FMT_I420: 4:2:0 at s x)          */
    int32_t format;            /* NS_FMT_444 | NS_FMT_I420                           */
} ns_sr_job;

/* Creates a context on `device` with a device memory pool of pool_bytes
   ("pre-allocates ... and construct a memory pool when a program
   launches").  NS_EUNSUPPORTED if the device is not compute capability 10.0.
   *out receives the context (host object). */
NS_API ns_status ns_ctx_create(int device, size_t pool_bytes, ns_ctx **out);
NS_API ns_status ns_ctx_destroy(ns_ctx *ctx);

/* Reserves a model slot (weights + packed kernel operands) from the pool.
   n_blocks >= 1, n_ch in {16, 32}, scale in {2, 3, 4} (8 blocks, 32
   channels, scale 3).  The kernels are shape-specialised on (n_ch, scale) at
   build time; weights are runtime data ("model pre-optimization"). */
NS_API ns_status ns_model_create(ns_ctx *ctx, int n_blocks, int n_ch, int scale, ns_model **out);

/* Refits the model with a bf16 weight blob (uint16 bit patterns, DEVICE or
   HOST pointer -- detected) of exactly ns_model_blob_len() entries, in the
   order head, blocks x (conv1, conv2), end, up, tail; each [Cout][Cin][3][3]
   followed by bias[Cout] (head Cin = 3, up Cout = s*s*C, tail Cout = 3).
   Repacks into the kernels' operand layout on `stream`; no re-planning. */
NS_API ns_status ns_model_set_weights(ns_model *m, const uint16_t *bf16_blob, size_t n, void *stream);
NS_API size_t ns_model_blob_len(int n_blocks, int n_ch, int scale);
NS_API ns_status ns_model_destroy(ns_model *m);

/* Anchor scoring + zero-inference selection for S streams (§5.1).
   chunks: HOST array [S]; all chunks must have the same n_frames.
   Outputs (DEVICE, [S][n]): gain (KEY frames: INT64_MAX, "equal anchor gain"
   P:170-176), rank (position in the per-stream priority order, or in the
   global order in NS_GLOBAL_BUDGET mode), is_anchor (0/1). */
NS_API ns_status ns_select_anchors(ns_ctx *ctx, const ns_chunk *chunks, int S, const ns_select_params *p,
                            int64_t *gain, int32_t *rank, uint8_t *is_anchor, void *stream);

/* Global anchor selection over streams gathered from every GPU (§5.2: "select
   anchor frames globally across all streams").
   Each GPU first runs ns_select_anchors on its own streams in
   NS_TOPK_PER_STREAM mode with NS_SEL_NEUROSCALER (any k: only the per-stream
   Alg. 1 gain is used), then the callers all-gather, per stream, gain[n],
   type[n], cost and a global stream id, and every GPU calls this with the
   identical gathered arrays, so every GPU computes the identical selection
   with no further exchange.  Inputs, all DEVICE, S = streams over all GPUs in
   any order: gain int64 [S][n]; rank_in int32 [S][n] or NULL -- NOT trusted:
   each stream's priority order is rebuilt here from (type asc, gain desc,
   frame asc), which is the rank ns_select_anchors returns in that mode
   (reading Z5), so a rank array from another mode or selector cannot corrupt
   the merge; type u8 [S][n]; sid int32 [S] distinct global stream
   ids (the stream key of the merged order, readings Z5, R7); cost int64 [S] >= 1.
   The merged order is G_key by (sid, frame), then G_altref, then G_normal, each
   by (gain desc, sid asc, frame asc); the anchors are its longest prefix with
   summed cost <= budget (Z7).  Outputs DEVICE [S][n]: rank (global
   position), is_anchor.  Equals ns_select_anchors in NS_GLOBAL_BUDGET mode over
   the same streams ordered by sid.  The values of cost/sid are not validated
   (device data); S * n <= 2^20. */
NS_API ns_status ns_select_merge(ns_ctx *ctx, int S, int n, const int64_t *gain, const int32_t *rank_in,
                                 const uint8_t *type, const int32_t *sid, const int64_t *cost, int64_t budget,
                                 int32_t *rank, uint8_t *is_anchor, void *stream);

/* SR on a host-supplied job list (jobs: HOST array [n_jobs]).  Jobs may mix
   models and resolutions; they are grouped by shape internally.  lr and
   hr_out must be 16-B aligned (as the chunk buffers). */
NS_API ns_status ns_sr_anchors(ns_ctx *ctx, const ns_sr_job *jobs, int n_jobs, void *stream);

/* Reuse-based reconstruction of every non-anchor frame of S chunks (§2, §6.1).
   is_anchor: DEVICE [S][n].  hr_out: HOST table [S*n] of DEVICE pointers, each
   [3][s*h][s*w]; anchors' entries must already hold the SR output (e.g. from
   ns_sr_anchors), so every entry of the table must be distinct (checked:
   NS_EINVAL; HR rings need ns_enhance_streams), and none may be a stream's
   hr_last / hr_golden (checked).  Writes hr_last / hr_golden at chunk end. */
NS_API ns_status ns_reconstruct_chunk(ns_ctx *ctx, const ns_chunk *chunks, int S, const uint8_t *is_anchor,
                               uint8_t *const *hr_out, void *stream);

/* The whole hot path for S streams: select -> SR on anchors (grouped across
   streams) -> reconstruct.  hr_out: HOST table [S*n] of DEVICE pointers, each
   [3][s*h][s*w], where frame f of stream s is written.
   HR rings: a stream's row may repeat entries (e.g. hr_out[s][f] = ring[f % R],
   R >= 2), so a long chunk of many streams needs O(S * R) HR frames instead of
   O(S * n).  Rules, all checked (NS_EINVAL):
     - hr_out[s][f] != hr_out[s][f-1] (frame f reads HR[f-1] as LAST);
     - no entry is shared with another stream or is any stream's state slot;
     - a ring stream needs hr_golden (GOLDEN is kept there: HR of the latest
       KEY/ALTREF is saved into it at the step after it) and no gt.
   After the call, each entry holds the LAST frame written to it.  Anchors of
   a ring stream are SR'd into a context-owned anchor cache (carved from the
   pool on first use: NS_ENOMEM if it does not fit) and copied into their
   slot at their own frame step (the client "caches [SR anchors] in
   memory" and reuses them).
   is_anchor_out (DEVICE [S][n]) may be NULL.  stats: DEVICE [S][8] fp64 or
   NULL: {displayed frames, anchors, sum anchor score, total score, SSE vs gt
   over the displayed frames (or -1), PSNR vs gt (or -1), 0, 0}. */
NS_API ns_status ns_enhance_streams(ns_ctx *ctx, const ns_chunk *chunks, int S, const ns_select_params *p,
                             uint8_t *const *hr_out, uint8_t *is_anchor_out, double *stats, void *stream);

/* The whole hot path with the decoder's outputs in HOST memory -- the ingest
   case, where decoded chunks arrive on the host -- and the outputs
   in HBM.  Same arguments and results as ns_enhance_streams, except:
     - chunks[s].lr, .res, .mv, .type, .res_size are HOST pointers to
       page-locked, device-mapped memory (cudaHostAlloc / cudaHostRegister;
       checked: NS_EINVAL otherwise); hr_last, hr_golden, gt stay DEVICE.
     - The library uploads the streams in groups on an internal copy stream:
       res/mv/type/res_size of group g+1 are copied while group g runs on
       `stream` (two staging buffers carved from the context pool on first use;
       NS_ENOMEM if the pool is too small).  LR is never copied wholesale: only
       the anchors' LR frames (the SR input) are gathered from host memory after
       selection, and KEY-frame / intra blocks read their LR in place.
     - NS_GLOBAL_BUDGET needs every stream's scores before selecting, so it
       runs as one group (no overlap).
   *h2d_bytes (HOST, may be NULL) receives the bytes this call moves from host
   to device: the uploads plus the gathered anchor LR frames (intra-block LR
   reads, a few percent of blocks, are not counted).  The call returns once
   everything is enqueued; results are ready when `stream` reaches them. */
NS_API ns_status ns_enhance_streams_host(ns_ctx *ctx, const ns_chunk *chunks, int S, const ns_select_params *p,
                                         uint8_t *const *hr_out, uint8_t *is_anchor_out, double *stats,
                                         uint64_t *h2d_bytes, void *stream);

/* ------------------------------------------------------------------ hybrid encoding
   Hybrid encoding of the super-resolved anchors (§6.1 "Hybrid video encoding",
   P:233-239).  The ingest video is reused as it is (its
   bitstream is outside this library: decoding and re-encoding video are out
   of scope); only the SR anchor frames are compressed, with an image codec --
   baseline JPEG through nvJPEG, 4:4:4 (the HR frames carry three
   full-resolution planes, reading Z18) -- and every frame of every chunk gets
   a header: "A new header attached to each frame contains the frame type
   (i.e., anchor or non-anchor frame) and the super-resolved frame for an
   anchor frame".  Package of one stream = n_frames x
   (ns_hybrid_header, then `bytes` of JPEG for an anchor, nothing otherwise). */
#define NS_HYBRID_MAGIC 0x4648534Eu   /* "NSHF" little-endian */
typedef struct {
    uint32_t magic;    /* NS_HYBRID_MAGIC                                       */
    uint32_t stream;   /* stream index within the call                          */
    uint16_t frame;    /* frame index within the chunk                          */
    uint8_t anchor;    /* 1: the JPEG of the super-resolved frame follows        */
    uint8_t quality;   /* JPEG quality it was coded at (0 for a non-anchor)     */
    uint32_t bytes;    /* payload bytes after this header                       */
} ns_hybrid_header;   /* 16 bytes */

/* Table 2, JPEG column: the quality for a chunk with n_anchors of
   n_frames frames as anchors -- fraction <= 5%: 95; <= 7.5%: 90; <= 10%: 80;
   above 10% JPEG "cannot meet the bitrate constraint": -1.  Also -1
   for invalid counts.  Host only. */
NS_API int ns_hybrid_quality(int n_anchors, int n_frames);

/* Encodes the anchors of S chunks after ns_enhance_streams and packages them.
   is_anchor: HOST [S][n] (e.g. a copy of is_anchor_out); hr_out: HOST table
   [S*n] of DEVICE pointers as passed to ns_enhance_streams (only the anchors'
   entries are read, so they must still hold their frames: with HR rings, call
   this before a later frame reuses an anchor's entry).  quality: 1..100, or
   0 = Table 2 per stream (NS_EUNSUPPORTED if a stream's anchor fraction is
   above 10%).  out: HOST buffer of out_cap bytes; the S packages are written
   back to back and out_len (HOST [S]) receives each one's size; NS_ENOMEM if
   out_cap is too small (out_len then holds what was needed so far).  Not on
   the GPU hot path: the encoder is created on first use and the call returns
   once every bitstream is in `out` (it synchronises `stream`). */
NS_API ns_status ns_encode_anchors(ns_ctx *ctx, const ns_chunk *chunks, int S, const uint8_t *is_anchor,
                                   uint8_t *const *hr_out, int quality, uint8_t *out, size_t out_cap,
                                   size_t *out_len, void *stream);

/* Number of this library's kernel launches enqueued by the calling thread
   since the last reset (for the bench's gpu_launches claim). */
NS_API uint64_t ns_launch_count(int reset);

/* Per-kernel-family device time (profiling; off by default).  When enabled,
   every launch wrapper brackets its kernel(s) with CUDA events on the call's
   stream.  ns_profile_enable(1) clears and starts, (0) stops (records are kept).
   ns_profile_read synchronises the recorded events and fills one entry per
   family (out must hold >= 16 entries) -- total_ms is the union of the
   family's event intervals -- plus, when out holds more, an entry "any": the
   union over all families (device time in which some library work ran);
   returns the number written or < 0. */
typedef struct {
    char name[24];
    uint64_t launches;     /* kernels launched                         */
    uint64_t scopes;       /* event-bracketed launch groups             */
    double total_ms;       /* device time with >= 1 group running (the union of the groups' intervals) */
} ns_prof_entry;
NS_API int ns_profile_enable(int on);
NS_API int ns_profile_read(ns_prof_entry *out, int max);

/* Thread-local description of the last error (includes cudaGetErrorString for
   NS_ECUDA).  Never NULL. */
NS_API const char *ns_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* NEUROSCALER_NS_H */
