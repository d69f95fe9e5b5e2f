// ns_api.cu -- host side of the C ABI declared in include/ns.h: argument
// validation, the pre-allocated context pool (App. A),
// model slots + weight refit, descriptor staging and the
// multi-stream batcher that drives the kernels.
#include <cstdarg>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <atomic>
#include <mutex>
#include <algorithm>
#include <deque>
#include <map>
#include <tuple>
#include <unordered_map>
#include <vector>
#include "ns_internal.h"

using namespace ns;

// ------------------------------------------------------------------ errors / counters
static thread_local char g_err[512] = "";
static std::atomic<uint64_t> g_launches{0};

static ns_status fail(ns_status st, const char *fmt, ...) {
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_err, sizeof(g_err), fmt, ap);
    va_end(ap);
    return st;
}
static ns_status cuda_fail(cudaError_t e, const char *where) {
    return fail(NS_ECUDA, "%s: %s (%s)", where, cudaGetErrorString(e), cudaGetErrorName(e));
}
#define NS_CUDA(call)                                           \
    do {                                                        \
        cudaError_t _e = (call);                                \
        if (_e != cudaSuccess) return cuda_fail(_e, #call);     \
    } while (0)

namespace {
struct ProfRec {
    int fam;
    int n;
    cudaEvent_t e0, e1;
};
std::mutex g_pmu;
std::atomic<bool> g_prof{false};
std::vector<ProfRec> g_recs;
std::vector<cudaEvent_t> g_evpool;
cudaEvent_t ev_get() {
    if (!g_evpool.empty()) {
        cudaEvent_t e = g_evpool.back();
        g_evpool.pop_back();
        return e;
    }
    cudaEvent_t e = nullptr;
    cudaEventCreate(&e);
    return e;
}
const char *kFamNames[] = {"score", "select", "global", "compact", "sr_prep", "sr_head", "sr_body", "sr_end",
                           "sr_up", "sr_tail", "recon", "state", "stats", "repack"};
}  // namespace

namespace ns {
const char *fam_name(int fam) { return (fam >= 0 && fam < F_COUNT) ? kFamNames[fam] : "?"; }

KScope::KScope(int fam_, cudaStream_t st_, int n_) : fam(fam_), n(n_), st(st_), rec(nullptr) {
    g_launches.fetch_add((uint64_t)n, std::memory_order_relaxed);
    if (g_prof.load(std::memory_order_relaxed)) {
        std::lock_guard<std::mutex> lk(g_pmu);
        ProfRec *r = new ProfRec{fam, n, ev_get(), ev_get()};
        cudaEventRecord(r->e0, st);
        rec = r;
    }
}
KScope::~KScope() {
    if (!rec) return;
    ProfRec *r = static_cast<ProfRec *>(rec);
    cudaEventRecord(r->e1, st);
    std::lock_guard<std::mutex> lk(g_pmu);
    g_recs.push_back(*r);
    delete r;
}

// ------------------------------------------------------------------ model layout
int model_num_layers(int n_blocks) { return 2 * n_blocks + 4; }

static size_t align128(size_t v) { return (v + 127) / 128 * 128; }

LayerShape model_layer(int n_blocks, int C, int s, int L) {
    LayerShape ls{};
    if (L == 0) {
        ls.cin = 16; ls.cin_real = 3; ls.ntot = C; ls.cout_real = C;
    } else if (L <= 2 * n_blocks + 1) {
        ls.cin = C; ls.cin_real = C; ls.ntot = C; ls.cout_real = C;
    } else if (L == 2 * n_blocks + 2) {
        ls.cin = C; ls.cin_real = C; ls.ntot = s * s * C; ls.cout_real = s * s * C; ls.perm = 1;
    } else {
        ls.cin = C; ls.cin_real = C; ls.ntot = 16; ls.cout_real = 3;
    }
    ls.nsplit = ls.ntot > 256 ? 2 : 1;
    ls.rot = ls.perm ? 0 : 1;
    ls.nb = ls.ntot;
    size_t off = 0;
    for (int l = 0; l < L; l++) off += model_layer(n_blocks, C, s, l).bytes;
    const size_t bbytes = ls.rot ? (size_t)30 * ls.cin * ls.nb : (size_t)9 * ls.cin * ls.ntot * 2;
    ls.b_off = off;
    ls.bias_off = off + align128(bbytes);
    ls.bytes = align128(bbytes) + align128((size_t)ls.ntot * 4);
    return ls;
}

static size_t blob_layers_bytes(int n_blocks, int C, int s) {
    size_t t = 0;
    for (int l = 0; l < model_num_layers(n_blocks); l++) t += model_layer(n_blocks, C, s, l).bytes;
    return t;
}

CompShape model_comp(int n_blocks, int C, int s) {
    CompShape c{};
    const int nout = s * s * 3;
    c.nb = (nout + 15) / 16 * 16;
    c.nstrip = 9;
    const size_t base = blob_layers_bytes(n_blocks, C, s);
    c.b_off = base;
    c.bias_off = base + align128((size_t)5 * (C / 16) * 2 * c.nstrip * c.nb * 16);
    c.aux_off = c.bias_off + align128((size_t)c.nb * 4);
    return c;
}

size_t model_packed_bytes(int n_blocks, int C, int s) {
    const CompShape c = model_comp(n_blocks, C, s);
    const size_t nout = (size_t)s * s * 3;
    const size_t aux = ((size_t)s * s * C * C * 9 + (size_t)s * s * C + (size_t)3 * C * 9 + 3 +
                        nout * C * 25 + nout) * 4;
    return c.aux_off + align128(aux);
}
}  // namespace ns

// ------------------------------------------------------------------ context
namespace {
constexpr int kStageSlots = 4;
constexpr size_t kStageBytes = 8u << 20;
constexpr int kMaxSN = 1 << 20;           // max streams x frames per call
constexpr int kMaxStreams = 65535;        // max streams per call (a grid dimension of the frame step)
constexpr int kMaxJobs = 1 << 20;
constexpr int kHostGroups = 8;            // stream groups per ns_enhance_streams_host call
// (NS_HOST_GROUPS in the environment overrides it: tuning experiments only)
static int host_groups() {
    static const int g = [] {
        const char *e = getenv("NS_HOST_GROUPS");
        const int v = e ? atoi(e) : 0;
        return v > 0 ? v : kHostGroups;
    }();
    return g;
}

// SR batch (jobs per arena); NS_SR_BATCH in the environment overrides it
// (tuning experiments only)
// stream parts of the SR / reconstruction overlap (1 = off); NS_OVERLAP_PARTS in
// the environment overrides it (tuning experiments only)
static int overlap_parts_default() {
    const char *e = getenv("NS_OVERLAP_PARTS");
    const int v = e ? atoi(e) : 0;
    return v > 0 ? v : 1;
}

// anchors per SR batch: 0 = per frame shape (sr_batch_jobs); NS_SR_BATCH in the
// environment fixes it (tuning experiments only)
static int sr_batch_default() {
    const char *e = getenv("NS_SR_BATCH");
    const int v = e ? atoi(e) : 0;
    return v > 0 ? v : 0;
}

struct ArenaEntry {
    int h, w, C, s, fmt, idx;   // idx: 0 / 1, the two arenas SR batches alternate between
    SrArena a;
};
}  // namespace

struct ns_model {
    ns_ctx *ctx;
    int n_blocks, C, s;
    uint8_t *packed;
    size_t bytes;
    bool has_weights;
};

struct ns_ctx {
    int device;
    uint8_t *pool = nullptr;
    size_t pool_bytes = 0, used = 0;
    uint8_t *stage_host[kStageSlots] = {};
    uint8_t *stage_dev[kStageSlots] = {};
    cudaEvent_t stage_ev[kStageSlots] = {};
    bool stage_used[kStageSlots] = {};
    int stage_next = 0;
    // device scratch (capacity kMaxSN)
    int64_t *score, *gain;
    int32_t *rank, *order, *grank, *pos_stream, *cut, *job_count;
    int32_t *acount;                     // [kMaxStreams] per-stream anchor counts / first job slots
    const uint8_t **asrc;                // [kMaxSN] HR rings: anchor sources (anchor cache)
    uint8_t *gsv;                        // [kMaxSN] HR rings: GOLDEN frames saved into hr_golden
    uint8_t *anchor;
    int16_t *gold;
    FrameDesc *fdesc;
    SrJob *jobs;
    uint16_t *blob_stage;  // device staging for host weight blobs
    size_t blob_stage_elems;
    int sr_batch = sr_batch_default();  // anchors per SR batch (arena size); 0 = per shape
    std::deque<ArenaEntry> arenas;   // deque: entries never move
    // host-input path (ns_enhance_streams_host): copy stream, two input staging
    // buffers (group ping-pong) and the anchor-LR gather staging, carved from
    // the pool on first use and grown (bump) if a later call needs more
    cudaStream_t cst = nullptr;
    cudaStream_t sst = nullptr;          // second SR stream: odd batches, so one batch's tail overlaps the next
    cudaStream_t rst = nullptr;          // reconstruction stream of the SR / reconstruction overlap
    cudaEvent_t ev_part[2] = {}, ev_rjoin = nullptr;
    int overlap_parts = overlap_parts_default();
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    cudaEvent_t ev_copied[2] = {}, ev_free[2] = {};
    bool hin_used[2] = {};
    uint8_t *hin[2] = {};
    size_t hin_cap = 0;
    uint8_t *lr_stage = nullptr;
    size_t lr_stage_cap = 0;
    const uint8_t **lr_src = nullptr;
    uint32_t *lr_len = nullptr;
    // ring mode: anchors' SR outputs wait here until their frame step (P:241
    // "caches it in memory"); carved from the pool on first use, grown on demand
    uint8_t *acache = nullptr;
    size_t acache_cap = 0;
    HybridEncoder *hybrid = nullptr;     // nvJPEG encoder (ns_encode_anchors), created on first use
};

static uint8_t *pool_take(ns_ctx *c, size_t bytes) {
    size_t off = (c->used + 255) / 256 * 256;
    if (off + bytes > c->pool_bytes) return nullptr;
    c->used = off + bytes;
    return c->pool + off;
}

// Stage a host buffer of `bytes` into device memory on `st`; returns the device address.
static ns_status stage_begin(ns_ctx *c, uint8_t **host, uint8_t **dev, int *slot) {
    const int i = c->stage_next;
    c->stage_next = (c->stage_next + 1) % kStageSlots;
    if (c->stage_used[i]) NS_CUDA(cudaEventSynchronize(c->stage_ev[i]));
    *host = c->stage_host[i];
    *dev = c->stage_dev[i];
    *slot = i;
    return NS_OK;
}
static ns_status stage_end(ns_ctx *c, int slot, size_t bytes, cudaStream_t st) {
    if (bytes) NS_CUDA(cudaMemcpyAsync(c->stage_dev[slot], c->stage_host[slot], bytes, cudaMemcpyHostToDevice, st));
    return NS_OK;
}
static ns_status stage_release(ns_ctx *c, int slot, cudaStream_t st) {
    NS_CUDA(cudaEventRecord(c->stage_ev[slot], st));
    c->stage_used[slot] = true;
    return NS_OK;
}

extern "C" ns_status ns_ctx_create(int device, size_t pool_bytes, ns_ctx **out) {
    if (!out) return fail(NS_EINVAL, "ns_ctx_create: out is NULL");
    *out = nullptr;
    int ndev = 0;
    NS_CUDA(cudaGetDeviceCount(&ndev));
    if (device < 0 || device >= ndev) return fail(NS_EINVAL, "ns_ctx_create: device %d out of range (%d)", device, ndev);
    cudaDeviceProp prop;
    NS_CUDA(cudaGetDeviceProperties(&prop, device));
    if (prop.major != 10 || prop.minor != 0)
        return fail(NS_EUNSUPPORTED, "ns_ctx_create: device %d is sm_%d%d, this build targets sm_100a", device,
                    prop.major, prop.minor);
    NS_CUDA(cudaSetDevice(device));
    ns_ctx *c = new ns_ctx();
    c->device = device;
    const size_t fixed = (size_t)kMaxSN * (8 + 8 + 4 + 4 + 4 + 4 + 1 + 2 + 2 + 8 + 1 + sizeof(FrameDesc)) +
                         (size_t)kMaxStreams * (2 + 4) +
                         (size_t)kMaxJobs * (sizeof(SrJob) + sizeof(uint8_t *) + sizeof(uint32_t)) +
                         kStageSlots * kStageBytes + (64u << 20) + 64 * 1024;
    if (pool_bytes < fixed + (64u << 20)) {
        delete c;
        return fail(NS_EINVAL, "ns_ctx_create: pool_bytes %zu too small (need >= %zu)", pool_bytes,
                    fixed + (64u << 20));
    }
    cudaError_t e = cudaMalloc(&c->pool, pool_bytes);
    if (e != cudaSuccess) {
        delete c;
        return cuda_fail(e, "cudaMalloc(pool)");
    }
    c->pool_bytes = pool_bytes;
    c->score = (int64_t *)pool_take(c, sizeof(int64_t) * kMaxSN);
    c->gain = (int64_t *)pool_take(c, sizeof(int64_t) * kMaxSN);
    c->rank = (int32_t *)pool_take(c, sizeof(int32_t) * kMaxSN);
    c->order = (int32_t *)pool_take(c, sizeof(int32_t) * kMaxSN);
    c->grank = (int32_t *)pool_take(c, sizeof(int32_t) * kMaxSN);
    c->pos_stream = (int32_t *)pool_take(c, sizeof(int32_t) * kMaxSN);
    c->anchor = (uint8_t *)pool_take(c, kMaxSN);
    c->gold = (int16_t *)pool_take(c, sizeof(int16_t) * ((size_t)kMaxSN + kMaxStreams));
    c->acount = (int32_t *)pool_take(c, sizeof(int32_t) * kMaxStreams);
    c->asrc = (const uint8_t **)pool_take(c, sizeof(uint8_t *) * kMaxSN);
    c->gsv = (uint8_t *)pool_take(c, kMaxSN);
    c->fdesc = (FrameDesc *)pool_take(c, sizeof(FrameDesc) * kMaxSN);
    c->cut = (int32_t *)pool_take(c, 256);
    c->job_count = (int32_t *)pool_take(c, sizeof(int32_t) * 4096);
    c->jobs = (SrJob *)pool_take(c, sizeof(SrJob) * kMaxJobs);
    c->blob_stage_elems = (64u << 20) / 2;
    c->blob_stage = (uint16_t *)pool_take(c, 64u << 20);
    for (int i = 0; i < kStageSlots; i++) {
        c->stage_dev[i] = pool_take(c, kStageBytes);
        if ((e = cudaHostAlloc(&c->stage_host[i], kStageBytes, cudaHostAllocDefault)) != cudaSuccess ||
            (e = cudaEventCreateWithFlags(&c->stage_ev[i], cudaEventDisableTiming)) != cudaSuccess) {
            ns_ctx_destroy(c);
            return cuda_fail(e, "staging");
        }
    }
    c->lr_src = (const uint8_t **)pool_take(c, sizeof(uint8_t *) * kMaxJobs);
    c->lr_len = (uint32_t *)pool_take(c, sizeof(uint32_t) * kMaxJobs);
    if ((e = cudaStreamCreateWithFlags(&c->cst, cudaStreamNonBlocking)) != cudaSuccess ||
        (e = cudaStreamCreateWithFlags(&c->sst, cudaStreamNonBlocking)) != cudaSuccess ||
        (e = cudaStreamCreateWithFlags(&c->rst, cudaStreamNonBlocking)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&c->ev_part[0], cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&c->ev_part[1], cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&c->ev_rjoin, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming)) != cudaSuccess ||
        (e = cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming)) != cudaSuccess) {
        ns_ctx_destroy(c);
        return cuda_fail(e, "streams");
    }
    for (int i = 0; i < 2; i++)
        if ((e = cudaEventCreateWithFlags(&c->ev_copied[i], cudaEventDisableTiming)) != cudaSuccess ||
            (e = cudaEventCreateWithFlags(&c->ev_free[i], cudaEventDisableTiming)) != cudaSuccess) {
            ns_ctx_destroy(c);
            return cuda_fail(e, "events");
        }
    *out = c;
    return NS_OK;
}

extern "C" ns_status ns_ctx_destroy(ns_ctx *c) {
    if (!c) return fail(NS_EINVAL, "ns_ctx_destroy: NULL");
    cudaSetDevice(c->device);
    cudaDeviceSynchronize();
    for (int i = 0; i < kStageSlots; i++) {
        if (c->stage_host[i]) cudaFreeHost(c->stage_host[i]);
        if (c->stage_ev[i]) cudaEventDestroy(c->stage_ev[i]);
    }
    for (int i = 0; i < 2; i++) {
        if (c->ev_copied[i]) cudaEventDestroy(c->ev_copied[i]);
        if (c->ev_free[i]) cudaEventDestroy(c->ev_free[i]);
    }
    hybrid_destroy(c->hybrid);
    if (c->cst) cudaStreamDestroy(c->cst);
    if (c->sst) cudaStreamDestroy(c->sst);
    if (c->rst) cudaStreamDestroy(c->rst);
    for (int i = 0; i < 2; i++)
        if (c->ev_part[i]) cudaEventDestroy(c->ev_part[i]);
    if (c->ev_rjoin) cudaEventDestroy(c->ev_rjoin);
    if (c->ev_fork) cudaEventDestroy(c->ev_fork);
    if (c->ev_join) cudaEventDestroy(c->ev_join);
    if (c->pool) cudaFree(c->pool);
    delete c;
    return NS_OK;
}

// ------------------------------------------------------------------ models
extern "C" size_t ns_model_blob_len(int B, int C, int s) {
    size_t n = (size_t)C * 3 * 9 + C;
    n += (size_t)2 * B * ((size_t)C * C * 9 + C);
    n += (size_t)C * C * 9 + C;
    n += (size_t)s * s * C * C * 9 + (size_t)s * s * C;
    n += (size_t)3 * C * 9 + 3;
    return n;
}

extern "C" ns_status ns_model_create(ns_ctx *c, int n_blocks, int n_ch, int scale, ns_model **out) {
    if (!c || !out) return fail(NS_EINVAL, "ns_model_create: NULL argument");
    if (n_blocks < 1 || n_blocks > 64) return fail(NS_EINVAL, "ns_model_create: n_blocks %d not in [1, 64]", n_blocks);
    if (n_ch != 16 && n_ch != 32) return fail(NS_EUNSUPPORTED, "ns_model_create: n_ch %d not in {16, 32}", n_ch);
    if (scale < 2 || scale > 4) return fail(NS_EINVAL, "ns_model_create: scale %d not in {2, 3, 4}", scale);
    const size_t bytes = model_packed_bytes(n_blocks, n_ch, scale);
    uint8_t *p = pool_take(c, bytes);
    if (!p) return fail(NS_ENOMEM, "ns_model_create: pool exhausted (%zu bytes needed)", bytes);
    ns_model *m = new ns_model{c, n_blocks, n_ch, scale, p, bytes, false};
    *out = m;
    return NS_OK;
}

extern "C" ns_status ns_model_set_weights(ns_model *m, const uint16_t *blob, size_t n, void *stream) {
    if (!m || !blob) return fail(NS_EINVAL, "ns_model_set_weights: NULL argument");
    const size_t need = ns_model_blob_len(m->n_blocks, m->C, m->s);
    if (n != need) return fail(NS_EINVAL, "ns_model_set_weights: blob has %zu entries, model needs %zu", n, need);
    ns_ctx *c = m->ctx;
    cudaStream_t st = (cudaStream_t)stream;
    NS_CUDA(cudaSetDevice(c->device));
    cudaPointerAttributes at;
    const uint16_t *src = blob;
    if (cudaPointerGetAttributes(&at, blob) != cudaSuccess || at.type != cudaMemoryTypeDevice) {
        cudaGetLastError();
        if (need > c->blob_stage_elems) return fail(NS_ENOMEM, "ns_model_set_weights: blob larger than staging");
        NS_CUDA(cudaMemcpyAsync(c->blob_stage, blob, need * 2, cudaMemcpyHostToDevice, st));
        src = c->blob_stage;
    }
    NS_CUDA(launch_repack(src, m->n_blocks, m->C, m->s, m->packed, st));
    if (src == c->blob_stage) NS_CUDA(cudaStreamSynchronize(st));  // host blob / staging reuse (not hot path)
    m->has_weights = true;
    return NS_OK;
}

extern "C" ns_status ns_model_destroy(ns_model *m) {
    if (!m) return fail(NS_EINVAL, "ns_model_destroy: NULL");
    // pool memory is released with the context (bump allocator, P:625 fragments)
    delete m;
    return NS_OK;
}

extern "C" uint64_t ns_launch_count(int reset) {
    return reset ? g_launches.exchange(0) : g_launches.load();
}
extern "C" const char *ns_last_error(void) { return g_err; }

extern "C" int ns_profile_enable(int on) {
    std::lock_guard<std::mutex> lk(g_pmu);
    if (on) {  // start: drop previous records; stop: keep them for ns_profile_read
        for (auto &r : g_recs) {
            g_evpool.push_back(r.e0);
            g_evpool.push_back(r.e1);
        }
        g_recs.clear();
    }
    g_prof.store(on != 0);
    return NS_OK;
}

extern "C" int ns_profile_read(ns_prof_entry *out, int max) {
    if (!out || max < (int)F_COUNT) return fail(NS_EINVAL, "ns_profile_read: need room for %d entries", (int)F_COUNT);
    std::lock_guard<std::mutex> lk(g_pmu);
    for (int f = 0; f < F_COUNT; f++) {
        memset(&out[f], 0, sizeof(ns_prof_entry));
        snprintf(out[f].name, sizeof(out[f].name), "%s", fam_name(f));
    }
    // total_ms = the union of the family's event intervals: launch groups of one
    // family on two streams (alternating SR batches) overlap, and the union is
    // the device time during which at least one of them ran (= the sum when
    // they do not overlap)
    std::vector<std::vector<std::pair<double, double>>> iv(F_COUNT);
    for (auto &r : g_recs) {
        float a = 0.f, b = 0.f;
        cudaError_t e = cudaEventSynchronize(r.e1);
        if (e == cudaSuccess) e = cudaEventElapsedTime(&a, g_recs[0].e0, r.e0);
        if (e == cudaSuccess) e = cudaEventElapsedTime(&b, g_recs[0].e0, r.e1);
        if (e != cudaSuccess) return cuda_fail(e, "ns_profile_read");
        out[r.fam].launches += (uint64_t)r.n;
        out[r.fam].scopes += 1;
        iv[r.fam].push_back({(double)a, (double)b});
    }
    for (int f = 0; f < F_COUNT; f++) {
        auto &v = iv[f];
        std::sort(v.begin(), v.end());
        double tot = 0.0, lo = 0.0, hi = -1e300;
        for (auto &x : v) {
            if (x.first > hi) {
                if (hi > lo) tot += hi - lo;
                lo = x.first;
                hi = x.second;
            } else if (x.second > hi) {
                hi = x.second;
            }
        }
        if (!v.empty() && hi > lo) tot += hi - lo;
        out[f].total_ms = tot;
    }
    if (max <= (int)F_COUNT) return (int)F_COUNT;
    // entry F_COUNT, "any": the union over every family -- the device time in
    // which at least one library scope was running (step time minus it = idle)
    std::vector<std::pair<double, double>> all;
    for (auto &v : iv) all.insert(all.end(), v.begin(), v.end());
    std::sort(all.begin(), all.end());
    double tot = 0.0, lo = 0.0, hi = -1e300;
    for (auto &x : all) {
        if (x.first > hi) {
            if (hi > lo) tot += hi - lo;
            lo = x.first;
            hi = x.second;
        } else if (x.second > hi) {
            hi = x.second;
        }
    }
    if (!all.empty() && hi > lo) tot += hi - lo;
    memset(&out[F_COUNT], 0, sizeof(ns_prof_entry));
    snprintf(out[F_COUNT].name, sizeof(out[F_COUNT].name), "any");
    for (int f = 0; f < F_COUNT; f++) { out[F_COUNT].launches += out[f].launches; out[F_COUNT].scopes += out[f].scopes; }
    out[F_COUNT].total_ms = tot;
    return (int)F_COUNT + 1;
}

// ------------------------------------------------------------------ validation
static bool al16(const void *p) { return ((uintptr_t)p & 15u) == 0; }
// elements per LR / residual frame and bytes per HR frame (all planes)
static size_t lr_frame_elems(const ns_chunk &k) {
    const size_t p = (size_t)k.h * k.w;
    return k.format == NS_FMT_I420 ? p * 3 / 2 : 3 * p;
}
static size_t hr_frame_bytes(const ns_chunk &k) {
    const size_t p = (size_t)k.h * k.scale * k.w * k.scale;
    return k.format == NS_FMT_I420 ? p * 3 / 2 : 3 * p;
}
// SR shape group: (h, w, C, s, B, format)
typedef std::tuple<int, int, int, int, int, int> GroupKey;

static ns_status check_chunks(const ns_chunk *ch, int S, bool need_model, int *n_out) {
    if (!ch) return fail(NS_EINVAL, "chunks is NULL");
    if (S < 1) return fail(NS_EINVAL, "S = %d < 1", S);
    if (S > kMaxStreams) return fail(NS_EINVAL, "S = %d exceeds %d streams per call", S, kMaxStreams);
    const int n = ch[0].n_frames;
    if (n < 1 || n > kMaxFrames) return fail(NS_EINVAL, "n_frames %d not in [1, %d]", n, kMaxFrames);
    if ((size_t)S * n > (size_t)kMaxSN) return fail(NS_EINVAL, "S * n = %zu exceeds %d", (size_t)S * n, kMaxSN);
    for (int s = 0; s < S; s++) {
        const ns_chunk &c = ch[s];
        if (c.n_frames != n) return fail(NS_EINVAL, "chunk %d: n_frames %d differs from chunk 0 (%d)", s, c.n_frames, n);
        if (c.w < 8 || c.h < 8 || c.w % 8 || c.h % 8)
            return fail(NS_EINVAL, "chunk %d: w=%d h=%d must be positive multiples of 8", s, c.w, c.h);
        if (c.w > 8192 || c.h > 8192) return fail(NS_EINVAL, "chunk %d: w/h > 8192", s);
        if (c.scale < 2 || c.scale > 4) return fail(NS_EINVAL, "chunk %d: scale %d not in {2,3,4}", s, c.scale);
        if (c.format != NS_FMT_444 && c.format != NS_FMT_I420)
            return fail(NS_EINVAL, "chunk %d: format %d not NS_FMT_444 / NS_FMT_I420", s, c.format);
        if (c.format == NS_FMT_I420 && (c.w % 16 || c.h % 16))
            return fail(NS_EINVAL, "chunk %d: 4:2:0 needs w, h multiples of 16 (8 x 8 chroma blocks), got %dx%d", s,
                        c.w, c.h);
        if (c.interp < NS_INTERP_BILINEAR || c.interp > NS_INTERP_SWITCHABLE)
            return fail(NS_EINVAL, "chunk %d: interp %d not an NS_INTERP_* value", s, c.interp);
        if (!c.lr || !c.res || !c.mv || !c.type) return fail(NS_EINVAL, "chunk %d: lr/res/mv/type must be non-NULL", s);
        if (!al16(c.res) || !al16(c.lr) || !al16(c.mv)) return fail(NS_EINVAL, "chunk %d: lr/res/mv must be 16-B aligned", s);
        if (c.gt && !al16(c.gt)) return fail(NS_EINVAL, "chunk %d: gt must be 16-B aligned", s);
        if ((c.hr_last && !al16(c.hr_last)) || (c.hr_golden && !al16(c.hr_golden)))
            return fail(NS_EINVAL, "chunk %d: hr_last/hr_golden must be 16-B aligned", s);
        if (c.hr_last && c.hr_last == c.hr_golden) return fail(NS_EINVAL, "chunk %d: hr_last aliases hr_golden", s);
        if (need_model) {
            if (!c.model) return fail(NS_EINVAL, "chunk %d: model is NULL", s);
            if (c.model->s != c.scale) return fail(NS_EINVAL, "chunk %d: model scale %d != chunk scale %d", s, c.model->s, c.scale);
            if (!c.model->has_weights) return fail(NS_EINVAL, "chunk %d: model has no weights (ns_model_set_weights)", s);
        }
    }
    *n_out = n;
    return NS_OK;
}

// hr_out[s][f]: non-NULL, 16-B aligned, distinct from hr_out[s][f-1] (the LAST
// reference frame f reads), from the stream's hr_last / hr_golden, and never
// shared with another stream.  A stream whose row repeats entries is an HR
// ring (ring[s] = 1): allowed only where `ring_ok` (ns_enhance_streams), and
// then it needs hr_golden (GOLDEN is saved there during the chunk) and no
// ground truth (the quality stats read every frame after the chunk).
static ns_status check_hr_table(const ns_chunk *ch, int S, int n, uint8_t *const *hr, bool ring_ok,
                                std::vector<int> *ring) {
    if (!hr) return fail(NS_EINVAL, "hr_out table is NULL");
    std::unordered_map<const uint8_t *, int> owner;
    owner.reserve((size_t)S * n * 2);
    if (ring) ring->assign(S, 0);
    for (int s = 0; s < S; s++)
        for (int f = 0; f < n; f++) {
            uint8_t *p = hr[(size_t)s * n + f];
            if (!p || !al16(p)) return fail(NS_EINVAL, "hr_out[%d][%d] is NULL or not 16-B aligned", s, f);
            if (f > 0 && p == hr[(size_t)s * n + f - 1]) return fail(NS_EINVAL, "hr_out[%d][%d] aliases hr_out[%d][%d]", s, f, s, f - 1);
            if (p == ch[s].hr_last || p == ch[s].hr_golden)
                return fail(NS_EINVAL, "hr_out[%d][%d] aliases the stream's hr_last/hr_golden", s, f);
            auto it = owner.emplace(p, s);
            if (!it.second) {
                if (it.first->second != s)
                    return fail(NS_EINVAL, "hr_out[%d][%d] is shared with another stream (%d)", s, f, it.first->second);
                if (!ring_ok)
                    return fail(NS_EINVAL, "hr_out[%d][%d] repeats an entry of its row: HR rings need ns_enhance_streams", s, f);
                if (ring) (*ring)[s] = 1;
            }
        }
    for (int s = 0; s < S && ring; s++) {
        if (!(*ring)[s]) continue;
        if (!ch[s].hr_golden) return fail(NS_EINVAL, "chunk %d: an HR ring needs hr_golden (GOLDEN is kept there)", s);
        if (ch[s].gt) return fail(NS_EINVAL, "chunk %d: quality stats vs gt need a full hr_out row, not a ring", s);
    }
    // state slots must not be shared between streams either
    for (int s = 0; s < S; s++)
        for (const uint8_t *q : {(const uint8_t *)ch[s].hr_last, (const uint8_t *)ch[s].hr_golden})
            if (q && owner.count(q)) return fail(NS_EINVAL, "chunk %d: a state slot is another stream's hr_out", s);
    return NS_OK;
}

// Builds StreamDesc[S] (+ optional hr table, cost, SR group stream lists) into
// a staging slot.
struct Staged {
    int slot;
    uint8_t *host, *dev;
    size_t used;
    StreamDesc *d_sd;
    uint8_t **d_hr;
    int64_t *d_cost;
    int32_t *d_glist, *d_goff;   // SR shape groups: streams of group g = glist[goff[g] .. goff[g+1])
    int16_t *d_prv, *d_nxt;      // HR rings: previous / next frame writing the same hr_out entry
};

static size_t a256(size_t v) { return (v + 255) / 256 * 256; }

// Per-stream batcher facts for stage_streams (all optional).
struct StreamPlan {
    const int *group = nullptr, *job_base = nullptr, *job_cap = nullptr, *job_goff = nullptr;
    uint8_t *const *acache = nullptr;    // per stream: its group's anchor cache (ring streams)
    const size_t *acache_stride = nullptr;
    const std::vector<int> *glist = nullptr, *goff = nullptr;
    const std::vector<int16_t> *prv = nullptr, *nxt = nullptr;   // [S*n] (HR rings)
};

static ns_status stage_streams(ns_ctx *c, const ns_chunk *ch, int S, int n, uint8_t *const *hr, const int64_t *cost,
                               bool use_res_size, Staged *out, const StreamPlan &pl = StreamPlan()) {
    const size_t sd_bytes = a256(sizeof(StreamDesc) * S);
    const size_t hr_bytes = hr ? a256(sizeof(uint8_t *) * (size_t)S * n) : 0;
    const size_t cost_bytes = cost ? a256(sizeof(int64_t) * S) : 0;
    const size_t gl_bytes = pl.glist ? a256(sizeof(int32_t) * pl.glist->size()) + a256(sizeof(int32_t) * pl.goff->size()) : 0;
    const size_t pn_bytes = pl.prv ? 2 * a256(sizeof(int16_t) * (size_t)S * n) : 0;
    if (sd_bytes + hr_bytes + cost_bytes + gl_bytes + pn_bytes > kStageBytes)
        return fail(NS_EINVAL, "too many streams x frames for one call (descriptor staging)");
    Staged g{};
    ns_status r = stage_begin(c, &g.host, &g.dev, &g.slot);
    if (r != NS_OK) return r;
    size_t off = 0;
    StreamDesc *sd = reinterpret_cast<StreamDesc *>(g.host);
    for (int s = 0; s < S; s++) {
        const ns_chunk &k = ch[s];
        StreamDesc d{};
        d.lr = k.lr; d.res = k.res; d.mv = k.mv; d.type = k.type; d.res_size = k.res_size;
        d.hr_last = k.hr_last; d.hr_golden = k.hr_golden; d.gt = k.gt;
        d.wts = k.model ? k.model->packed : nullptr;
        d.w = k.w; d.h = k.h; d.s = k.scale; d.n = k.n_frames;
        d.hr_base = s * n;
        d.group = pl.group ? pl.group[s] : 0;
        d.job_base = pl.job_base ? pl.job_base[s] : 0;
        d.job_cap = pl.job_cap ? pl.job_cap[s] : INT32_MAX;
        d.job_goff = pl.job_goff ? pl.job_goff[s] : 0;
        d.use_res_size = use_res_size ? 1 : 0;
        d.fmt = k.format;
        d.interp = k.interp;
        d.lr_frame = (int64_t)lr_frame_elems(k);
        d.hr_frame = (int64_t)hr_frame_bytes(k);
        d.acache = pl.acache ? pl.acache[s] : nullptr;
        d.acache_stride = pl.acache_stride ? pl.acache_stride[s] : 0;
        sd[s] = d;
    }
    g.d_sd = reinterpret_cast<StreamDesc *>(g.dev);
    off = sd_bytes;
    if (hr) {
        memcpy(g.host + off, hr, sizeof(uint8_t *) * (size_t)S * n);
        g.d_hr = reinterpret_cast<uint8_t **>(g.dev + off);
        off += hr_bytes;
    }
    if (cost) {
        memcpy(g.host + off, cost, sizeof(int64_t) * S);
        g.d_cost = reinterpret_cast<int64_t *>(g.dev + off);
        off += cost_bytes;
    }
    if (pl.glist) {
        memcpy(g.host + off, pl.glist->data(), sizeof(int32_t) * pl.glist->size());
        g.d_glist = reinterpret_cast<int32_t *>(g.dev + off);
        off += a256(sizeof(int32_t) * pl.glist->size());
        memcpy(g.host + off, pl.goff->data(), sizeof(int32_t) * pl.goff->size());
        g.d_goff = reinterpret_cast<int32_t *>(g.dev + off);
        off += a256(sizeof(int32_t) * pl.goff->size());
    }
    if (pl.prv) {
        memcpy(g.host + off, pl.prv->data(), sizeof(int16_t) * (size_t)S * n);
        g.d_prv = reinterpret_cast<int16_t *>(g.dev + off);
        off += a256(sizeof(int16_t) * (size_t)S * n);
        memcpy(g.host + off, pl.nxt->data(), sizeof(int16_t) * (size_t)S * n);
        g.d_nxt = reinterpret_cast<int16_t *>(g.dev + off);
        off += a256(sizeof(int16_t) * (size_t)S * n);
    }
    g.used = off;
    *out = g;
    return NS_OK;
}

static ns_status check_params(const ns_select_params *p, int S, int n) {
    if (!p) return fail(NS_EINVAL, "params is NULL");
    if (p->group_residual != NS_CARRY && p->group_residual != NS_FRESH)
        return fail(NS_EINVAL, "group_residual %d invalid", p->group_residual);
    if (p->selector != NS_SEL_NEUROSCALER && p->selector != NS_SEL_KEY && p->selector != NS_SEL_KEY_UNIFORM)
        return fail(NS_EINVAL, "selector %d invalid", p->selector);
    if (p->mode != NS_TOPK_PER_STREAM && p->selector != NS_SEL_NEUROSCALER)
        return fail(NS_EINVAL, "the baseline selectors are top-k only");
    if (p->mode != NS_GIVEN_ANCHORS && p->anchor_in)
        return fail(NS_EINVAL, "anchor_in is only read in NS_GIVEN_ANCHORS mode");
    if (p->mode == NS_TOPK_PER_STREAM) {
        if (p->k < 0 || p->k > n) return fail(NS_EINVAL, "k = %d not in [0, n = %d]", p->k, n);
    } else if (p->mode == NS_GLOBAL_BUDGET || p->mode == NS_GIVEN_ANCHORS) {
        if (p->mode == NS_GIVEN_ANCHORS && !p->anchor_in) return fail(NS_EINVAL, "given mode needs anchor_in");
        if (!p->cost) return fail(NS_EINVAL, "global / given mode needs cost[S]");
        if (p->budget < 0) return fail(NS_EINVAL, "budget < 0");
        for (int s = 0; s < S; s++)
            if (p->cost[s] < 1) return fail(NS_EINVAL, "cost[%d] = %lld < 1", s, (long long)p->cost[s]);
    } else {
        return fail(NS_EINVAL, "mode %d invalid", p->mode);
    }
    return NS_OK;
}

// select into (gain, rank, is_anchor); order/score in ctx scratch
static ns_status run_select(ns_ctx *c, const Staged &g, const ns_chunk *ch, int S, int n, const ns_select_params *p,
                            int64_t *gain, int32_t *rank, uint8_t *is_anchor, cudaStream_t st) {
    int maxv = 0;
    for (int s = 0; s < S; s++) maxv = std::max(maxv, (int)(lr_frame_elems(ch[s]) / 8));
    NS_CUDA(launch_score(g.d_sd, S, n, maxv, c->score, st));
    if (p->mode == NS_GIVEN_ANCHORS) {  // decided by ns_select_merge across GPUs
        if (is_anchor != p->anchor_in)
            NS_CUDA(cudaMemcpyAsync(is_anchor, p->anchor_in, (size_t)S * n, cudaMemcpyDeviceToDevice, st));
        return NS_OK;
    }
    const bool global = p->mode == NS_GLOBAL_BUDGET;
    NS_CUDA(launch_select(g.d_sd, c->score, S, n, global ? -1 : p->k, p->group_residual == NS_FRESH, p->selector,
                          gain, rank, is_anchor, global ? c->order : nullptr, st));
    if (global)
        NS_CUDA(launch_global(g.d_sd, S, n, gain, c->order, g.d_cost, p->budget, c->grank, c->pos_stream, c->cut,
                              rank, is_anchor, st));
    return NS_OK;
}

extern "C" ns_status ns_select_anchors(ns_ctx *c, const ns_chunk *ch, int S, const ns_select_params *p,
                                       int64_t *gain, int32_t *rank, uint8_t *is_anchor, void *stream) {
    if (!c) return fail(NS_EINVAL, "ns_select_anchors: ctx is NULL");
    int n = 0;
    ns_status r = check_chunks(ch, S, false, &n);
    if (r != NS_OK) return r;
    if ((r = check_params(p, S, n)) != NS_OK) return r;
    if (p->mode == NS_GIVEN_ANCHORS) return fail(NS_EINVAL, "ns_select_anchors: NS_GIVEN_ANCHORS selects nothing");
    if (!gain || !rank || !is_anchor) return fail(NS_EINVAL, "ns_select_anchors: outputs must be non-NULL");
    cudaStream_t st = (cudaStream_t)stream;
    NS_CUDA(cudaSetDevice(c->device));
    Staged g;
    if ((r = stage_streams(c, ch, S, n, nullptr, p->mode == NS_GLOBAL_BUDGET ? p->cost : nullptr,
                           p->use_res_size != 0, &g)) != NS_OK)
        return r;
    if ((r = stage_end(c, g.slot, g.used, st)) != NS_OK) return r;
    r = run_select(c, g, ch, S, n, p, gain, rank, is_anchor, st);
    stage_release(c, g.slot, st);
    return r;
}

extern "C" ns_status ns_select_merge(ns_ctx *c, int S, int n, const int64_t *gain, const int32_t *rank_in,
                                     const uint8_t *type, const int32_t *sid, const int64_t *cost, int64_t budget,
                                     int32_t *rank, uint8_t *is_anchor, void *stream) {
    if (!c) return fail(NS_EINVAL, "ns_select_merge: ctx is NULL");
    if (S < 1 || n < 1 || n > kMaxFrames) return fail(NS_EINVAL, "ns_select_merge: S = %d, n = %d", S, n);
    if ((size_t)S * n > (size_t)kMaxSN) return fail(NS_EINVAL, "S * n = %zu exceeds %d", (size_t)S * n, kMaxSN);
    if (budget < 0) return fail(NS_EINVAL, "budget < 0");
    if (!gain || !type || !sid || !cost || !rank || !is_anchor)
        return fail(NS_EINVAL, "ns_select_merge: NULL array");
    NS_CUDA(cudaSetDevice(c->device));
    NS_CUDA(launch_merge(S, n, gain, rank_in, type, sid, cost, budget, c->order, c->grank, c->pos_stream, c->cut, rank,
                         is_anchor, (cudaStream_t)stream));
    return NS_OK;
}

// ------------------------------------------------------------------ SR
// idx 0: the shape's first arena, sized for sr_batch_jobs (halved down to 16 if
// the pool cannot hold two of that size); idx 1: the second, with the first one's job count
// (batches alternate between them), or none if the pool has no room for it.
static ns_status get_arena(ns_ctx *c, int h, int w, int C, int s, int fmt, int idx, int nb_req, const SrArena **out) {
    for (auto &e : c->arenas)
        if (e.h == h && e.w == w && e.C == C && e.s == s && e.fmt == fmt && e.idx == idx) {
            *out = &e.a;
            return NS_OK;
        }
    int nb = nb_req;
    if (idx == 0) {
        int dev = 0, sms = 148;
        if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        nb = c->sr_batch > 0 ? c->sr_batch : sr_batch_jobs(h, w, sms);
        // (room for both arenas, so batches keep alternating between two streams)
        while (nb > 16 && c->used + 2 * sr_arena_bytes(h, w, C, s, nb, fmt) + 512 > c->pool_bytes) nb = std::max(16, nb / 2);
    }
    const size_t bytes = sr_arena_bytes(h, w, C, s, nb, fmt);
    if (idx > 0 && c->used + bytes + 256 > c->pool_bytes) {  // no room for a second arena: one stream
        *out = nullptr;
        return NS_OK;
    }
    uint8_t *mem = pool_take(c, bytes);
    if (!mem)
        return fail(NS_ENOMEM, "SR arena for %dx%d C%d x%d (%d jobs) needs %zu bytes; pool has %zu free", w, h, C, s,
                    nb, bytes, c->pool_bytes - c->used);
    ArenaEntry e{h, w, C, s, fmt, idx, {}};
    if (sr_arena_init(&e.a, h, w, C, s, nb, fmt, mem) != 0)
        return fail(NS_ECUDA, "cuTensorMapEncodeTiled failed for the SR arena");
    c->arenas.push_back(e);
    *out = &c->arenas.back().a;
    return NS_OK;
}

// jobs (device table) [0, max_jobs) of one shape; job_count (device) may be NULL.
// Batches alternate between `st` (arena 0) and the context's second SR stream
// (arena 1), forked from and joined back into `st`: a batch's last wave (each
// SR kernel's final partial wave of CTAs) overlaps the next batch's first.
static ns_status run_sr_group(ns_ctx *c, const GroupKey &key, const SrJob *d_jobs, int max_jobs,
                              const int32_t *job_count, cudaStream_t st) {
    int h, w, C, s, B, fmt;
    std::tie(h, w, C, s, B, fmt) = key;
    const SrArena *a[2] = {nullptr, nullptr};
    ns_status r = get_arena(c, h, w, C, s, fmt, 0, 0, &a[0]);
    if (r != NS_OK) return r;
    const int nbatch = (max_jobs + a[0]->nb - 1) / a[0]->nb;
    if (nbatch > 1 && (r = get_arena(c, h, w, C, s, fmt, 1, a[0]->nb, &a[1])) != NS_OK) return r;
    const bool two = a[1] != nullptr;
    if (two) {
        NS_CUDA(cudaEventRecord(c->ev_fork, st));
        NS_CUDA(cudaStreamWaitEvent(c->sst, c->ev_fork, 0));
    }
    for (int i = 0, j0 = 0; j0 < max_jobs; i++, j0 += a[0]->nb) {
        const int nj = std::min(a[0]->nb, max_jobs - j0);
        const bool odd = two && (i & 1);
        NS_CUDA(sr_run_batch(a[odd ? 1 : 0], B, d_jobs, j0, nj, job_count, odd ? c->sst : st));
    }
    if (two) {
        NS_CUDA(cudaEventRecord(c->ev_join, c->sst));
        NS_CUDA(cudaStreamWaitEvent(st, c->ev_join, 0));
    }
    return NS_OK;
}

extern "C" ns_status ns_sr_anchors(ns_ctx *c, const ns_sr_job *jobs, int n_jobs, void *stream) {
    if (!c) return fail(NS_EINVAL, "ns_sr_anchors: ctx is NULL");
    if (n_jobs < 0 || (n_jobs > 0 && !jobs)) return fail(NS_EINVAL, "ns_sr_anchors: bad job list");
    if (n_jobs == 0) return NS_OK;
    for (int j = 0; j < n_jobs; j++) {
        const ns_sr_job &J = jobs[j];
        if (!J.model || !J.lr || !J.hr_out) return fail(NS_EINVAL, "job %d: NULL model/lr/hr_out", j);
        if (!al16(J.lr) || !al16(J.hr_out)) return fail(NS_EINVAL, "job %d: lr/hr_out must be 16-B aligned", j);
        if (!J.model->has_weights) return fail(NS_EINVAL, "job %d: model has no weights", j);
        if (J.w < 8 || J.h < 8 || J.w % 8 || J.h % 8) return fail(NS_EINVAL, "job %d: w=%d h=%d must be multiples of 8", j, J.w, J.h);
    }
    cudaStream_t st = (cudaStream_t)stream;
    NS_CUDA(cudaSetDevice(c->device));
    // group by shape
    for (int j = 0; j < n_jobs; j++)
        if (jobs[j].format != NS_FMT_444 && jobs[j].format != NS_FMT_I420)
            return fail(NS_EINVAL, "job %d: format %d invalid", j, jobs[j].format);
        else if (jobs[j].format == NS_FMT_I420 && (jobs[j].w % 16 || jobs[j].h % 16))
            return fail(NS_EINVAL, "job %d: 4:2:0 needs w, h multiples of 16", j);
    std::map<GroupKey, std::vector<int>> groups;
    for (int j = 0; j < n_jobs; j++)
        groups[GroupKey(jobs[j].h, jobs[j].w, jobs[j].model->C, jobs[j].model->s, jobs[j].model->n_blocks,
                        jobs[j].format)]
            .push_back(j);
    ns_status r = NS_OK;
    for (auto &kv : groups) {  // every arena first: a pool that is too small fails with nothing launched
        int h, w, C, s, B, fmt;
        std::tie(h, w, C, s, B, fmt) = kv.first;
        const SrArena *a0 = nullptr, *a1 = nullptr;
        if ((r = get_arena(c, h, w, C, s, fmt, 0, 0, &a0)) != NS_OK) return r;
        if ((int)kv.second.size() > a0->nb && (r = get_arena(c, h, w, C, s, fmt, 1, a0->nb, &a1)) != NS_OK) return r;
    }
    for (auto &kv : groups) {
        const auto &idx = kv.second;
        if (idx.size() * sizeof(SrJob) > kStageBytes) return fail(NS_EINVAL, "too many SR jobs in one call");
        uint8_t *host, *dev;
        int slot;
        if ((r = stage_begin(c, &host, &dev, &slot)) != NS_OK) return r;
        SrJob *hj = reinterpret_cast<SrJob *>(host);
        for (size_t i = 0; i < idx.size(); i++) {
            const ns_sr_job &J = jobs[idx[i]];
            hj[i] = SrJob{J.lr, J.hr_out, J.model->packed};
        }
        if ((r = stage_end(c, slot, idx.size() * sizeof(SrJob), st)) != NS_OK) return r;
        r = run_sr_group(c, kv.first, reinterpret_cast<const SrJob *>(dev), (int)idx.size(), nullptr, st);
        stage_release(c, slot, st);
        if (r != NS_OK) return r;
    }
    return NS_OK;
}

// ------------------------------------------------------------------ reconstruct
// Reconstruction in three parts so that the whole path can overlap it with SR:
// the per-chunk descriptors (all streams), the frame steps of streams
// [s0, s0 + cnt), and the chunk-end state (all streams).
struct ReconGeom {
    int mw[5] = {0, 0, 0, 0, 0}, mh[5] = {0, 0, 0, 0, 0}, i420[5] = {0, 0, 0, 0, 0};
    int e8[5] = {0, 0, 0, 0, 0};   // bit 0: an 8-tap stream of that scale, bit 1: an 8-tap 4:2:0 one
    size_t maxhr = 0;
};
static ReconGeom recon_geom(const ns_chunk *ch, int s0, int cnt) {
    ReconGeom gm;
    for (int s = s0; s < s0 + cnt; s++) {
        gm.mw[ch[s].scale] = std::max(gm.mw[ch[s].scale], ch[s].w);
        gm.mh[ch[s].scale] = std::max(gm.mh[ch[s].scale], ch[s].h);
        gm.i420[ch[s].scale] |= ch[s].format == NS_FMT_I420;
        if (ch[s].interp != NS_INTERP_BILINEAR) gm.e8[ch[s].scale] |= ch[s].format == NS_FMT_I420 ? 3 : 1;
        gm.maxhr = std::max(gm.maxhr, hr_frame_bytes(ch[s]));
    }
    return gm;
}
static ns_status recon_prepare(ns_ctx *c, const Staged &g, int S, int n, const uint8_t *is_anchor,
                               const uint8_t *const *asrc, cudaStream_t st) {
    uint8_t *gsv = g.d_nxt ? c->gsv : nullptr;   // HR rings: GOLDEN saves
    NS_CUDA(launch_golden_index(g.d_sd, S, n, g.d_nxt, c->gold, gsv, st));
    NS_CUDA(launch_frame_desc(g.d_sd, S, n, is_anchor, g.d_hr, c->gold, gsv, asrc, c->fdesc, st));
    return NS_OK;
}
static ns_status recon_steps(ns_ctx *c, const ns_chunk *ch, int s0, int cnt, int n, cudaStream_t st) {
    const ReconGeom gm = recon_geom(ch, s0, cnt);
    for (int f = 0; f < n; f++) NS_CUDA(launch_recon_step(c->fdesc, cnt, n, f, gm.mw, gm.mh, gm.i420, gm.e8, st, s0));
    return NS_OK;
}
static ns_status recon_finish(ns_ctx *c, const Staged &g, const ns_chunk *ch, int S, int n, cudaStream_t st) {
    NS_CUDA(launch_state_copy(g.d_sd, S, n, g.d_hr, c->gold, g.d_nxt ? c->gsv : nullptr, recon_geom(ch, 0, S).maxhr,
                              st));
    return NS_OK;
}
static ns_status run_reconstruct(ns_ctx *c, const Staged &g, const ns_chunk *ch, int S, int n,
                                 const uint8_t *is_anchor, const uint8_t *const *asrc, cudaStream_t st) {
    ns_status r;
    if ((r = recon_prepare(c, g, S, n, is_anchor, asrc, st)) != NS_OK) return r;
    if ((r = recon_steps(c, ch, 0, S, n, st)) != NS_OK) return r;
    return recon_finish(c, g, ch, S, n, st);
}

extern "C" ns_status ns_reconstruct_chunk(ns_ctx *c, const ns_chunk *ch, int S, const uint8_t *is_anchor,
                                          uint8_t *const *hr_out, void *stream) {
    if (!c) return fail(NS_EINVAL, "ns_reconstruct_chunk: ctx is NULL");
    int n = 0;
    ns_status r = check_chunks(ch, S, false, &n);
    if (r != NS_OK) return r;
    if (!is_anchor) return fail(NS_EINVAL, "ns_reconstruct_chunk: is_anchor is NULL");
    if ((r = check_hr_table(ch, S, n, hr_out, false, nullptr)) != NS_OK) return r;
    cudaStream_t st = (cudaStream_t)stream;
    NS_CUDA(cudaSetDevice(c->device));
    Staged g;
    if ((r = stage_streams(c, ch, S, n, hr_out, nullptr, false, &g)) != NS_OK) return r;
    if ((r = stage_end(c, g.slot, g.used, st)) != NS_OK) return r;
    r = run_reconstruct(c, g, ch, S, n, is_anchor, nullptr, st);
    stage_release(c, g.slot, st);
    return r;
}

// ------------------------------------------------------------------ the whole path
// Optional host-input mode of enhance_impl: SR jobs read LR from a device copy
// gathered after selection (lr_stage, one frame of lr_stride bytes per job slot).
struct LrGather {
    uint8_t *stage;
    size_t stride;
};

static ns_status enhance_impl(ns_ctx *c, const ns_chunk *ch, int S, int n, const ns_select_params *p,
                              uint8_t *const *hr_out, uint8_t *anchor, double *stats, cudaStream_t st,
                              const LrGather *lg, uint64_t *gathered, const std::vector<int> &ring) {
    const bool topk = p->mode == NS_TOPK_PER_STREAM;
    // exactly k anchors per stream -> fixed job slots; otherwise (budget, given
    // map, Key SR with fewer key frames than k) slots are assigned per group
    const bool fixed = topk && p->selector != NS_SEL_KEY;
    // SR shape groups and job slots (multi-stream batcher)
    std::map<GroupKey, int> gid;
    std::vector<GroupKey> gkey;
    std::vector<int> group(S), job_base(S), job_goff(S), gcount, goff;
    std::vector<int> gstreams;
    int64_t min_cost = INT64_MAX;
    if (!topk)
        for (int s = 0; s < S; s++) min_cost = std::min(min_cost, p->cost[s]);
    for (int s = 0; s < S; s++) {
        const GroupKey key(ch[s].h, ch[s].w, ch[s].model->C, ch[s].scale, ch[s].model->n_blocks, ch[s].format);
        auto it = gid.find(key);
        if (it == gid.end()) {
            it = gid.emplace(key, (int)gkey.size()).first;
            gkey.push_back(key);
            gstreams.push_back(0);
        }
        group[s] = it->second;
        gstreams[it->second]++;
    }
    const int G = (int)gkey.size();
    gcount.resize(G);
    goff.resize(G);
    int total = 0;
    for (int gi = 0; gi < G; gi++) {
        int64_t mx = topk ? (int64_t)gstreams[gi] * p->k : (int64_t)gstreams[gi] * n;
        if (!topk) mx = std::min<int64_t>(mx, p->budget / std::max<int64_t>(min_cost, 1));
        gcount[gi] = (int)mx;
        goff[gi] = total;
        total += (int)mx;
    }
    if (total > kMaxJobs) return fail(NS_EINVAL, "too many SR jobs (%d)", total);
    if (lg && (size_t)total * lg->stride > c->lr_stage_cap)
        return fail(NS_EINVAL, "anchor LR staging too small (%d jobs)", total);
    // the streams of each group in stream order (deterministic slot assignment)
    std::vector<int> glist, gl_off(G + 1, 0);
    for (int s = 0; s < S; s++) gl_off[group[s] + 1]++;
    for (int gi = 0; gi < G; gi++) gl_off[gi + 1] += gl_off[gi];
    glist.resize(S);
    {
        std::vector<int> fill(gl_off.begin(), gl_off.end() - 1), local(G, 0);
        for (int s = 0; s < S; s++) {
            const int gi = group[s];
            glist[fill[gi]++] = s;
            job_base[s] = fixed ? goff[gi] + local[gi]++ * p->k : goff[gi];
            job_goff[s] = goff[gi];
        }
    }
    // every SR arena and the anchor cache are reserved before anything is
    // enqueued, so a pool that is too small fails with nothing launched
    ns_status r;
    if (total > 0)
        for (int gi = 0; gi < G; gi++) {
            int h, w, C, s, B, fmt;
            std::tie(h, w, C, s, B, fmt) = gkey[gi];
            const SrArena *a0 = nullptr, *a1 = nullptr;
            if ((r = get_arena(c, h, w, C, s, fmt, 0, 0, &a0)) != NS_OK) return r;
            if (gcount[gi] > a0->nb && (r = get_arena(c, h, w, C, s, fmt, 1, a0->nb, &a1)) != NS_OK) return r;
        }
    const bool any_ring = std::find(ring.begin(), ring.end(), 1) != ring.end();
    std::vector<uint8_t *> acache(S, nullptr);
    std::vector<size_t> astride(S, 0);
    if (any_ring && total > 0) {
        std::vector<size_t> gbase(G), gstride(G);
        size_t need = 0;
        for (int gi = 0; gi < G; gi++) {
            int h, w, C, s, B, fmt;
            std::tie(h, w, C, s, B, fmt) = gkey[gi];
            gstride[gi] = a256((size_t)h * s * w * s * (fmt == NS_FMT_I420 ? 3 : 6) / 2);
            gbase[gi] = need;
            need += gstride[gi] * gcount[gi];
        }
        if (need > c->acache_cap) {
            NS_CUDA(cudaStreamSynchronize(st));  // a smaller cache may still be read (not the steady state)
            if (!(c->acache = pool_take(c, need)))
                return fail(NS_ENOMEM, "HR ring: pool too small for the anchor cache (%zu bytes)", need);
            c->acache_cap = need;
        }
        for (int s = 0; s < S; s++) {
            acache[s] = c->acache + gbase[group[s]];
            astride[s] = gstride[group[s]];
        }
    }
    // HR rings: for every frame the previous / next frame of its stream that
    // writes the same hr_out entry (-1 / n: none)
    std::vector<int16_t> prv, nxt;
    if (any_ring) {
        prv.assign((size_t)S * n, -1);
        nxt.assign((size_t)S * n, (int16_t)n);
        std::unordered_map<const uint8_t *, int> last;
        for (int s = 0; s < S; s++) {
            last.clear();
            for (int f = 0; f < n; f++) {
                const size_t e = (size_t)s * n + f;
                auto it = last.find(hr_out[e]);
                if (it != last.end()) {
                    prv[e] = (int16_t)it->second;
                    nxt[(size_t)s * n + it->second] = (int16_t)f;
                    it->second = f;
                } else {
                    last.emplace(hr_out[e], f);
                }
            }
        }
    }
    if (gathered && lg) {  // exact in top-k mode (k frames per stream); upper bound otherwise
        uint64_t b = 0;
        for (int s = 0; s < S; s++) b += (uint64_t)lr_frame_elems(ch[s]) * (fixed ? p->k : 0);
        if (!fixed) b = (uint64_t)total * lg->stride;
        *gathered += b;
    }
    Staged g;
    std::vector<int> job_cap(S);
    for (int s = 0; s < S; s++) job_cap[s] = fixed ? p->k : gcount[group[s]];
    StreamPlan pl;
    pl.group = group.data();
    pl.job_base = job_base.data();
    pl.job_cap = job_cap.data();
    pl.job_goff = job_goff.data();
    pl.acache = acache.data();
    pl.acache_stride = astride.data();
    pl.glist = &glist;
    pl.goff = &gl_off;
    if (any_ring) {
        pl.prv = &prv;
        pl.nxt = &nxt;
    }
    if ((r = stage_streams(c, ch, S, n, hr_out, topk ? nullptr : p->cost, p->use_res_size != 0, &g, pl)) != NS_OK)
        return r;
    if ((r = stage_end(c, g.slot, g.used, st)) != NS_OK) return r;
    do {
        if ((r = run_select(c, g, ch, S, n, p, c->gain, c->rank, anchor, st)) != NS_OK) break;
        if (total > 0) {
            cudaError_t e = cudaSuccess;
            if (lg) e = cudaMemsetAsync(c->lr_len, 0, sizeof(uint32_t) * total, st);
            if (e == cudaSuccess)
                e = launch_compact(g.d_sd, S, n, anchor, g.d_hr, c->jobs, c->job_count, G, g.d_glist, g.d_goff,
                                   c->acount, fixed, g.d_prv, any_ring ? c->asrc : nullptr, st,
                                   lg ? lg->stage : nullptr,
                                   lg ? lg->stride : 0, c->lr_src, c->lr_len);
            if (e == cudaSuccess && lg) e = launch_lr_gather(c->jobs, c->lr_src, c->lr_len, total, lg->stride, st);
            if (e != cudaSuccess) { r = cuda_fail(e, "compact"); break; }
        }
        const uint8_t *const *asrc = any_ring && total > 0 ? c->asrc : nullptr;
        // SR of stream part p overlaps the reconstruction of part p - 1 (fixed top-k
        // job slots are contiguous per stream in each shape group): the frame steps
        // of a part run on the context's reconstruction stream once its anchors
        // are done; the chunk-end state and the stats wait for all of them.
        const int parts = (fixed && total > 0) ? std::max(1, std::min(c->overlap_parts, S)) : 1;
        if (parts == 1) {
            for (int gi = 0; gi < G && r == NS_OK && total > 0; gi++)
                r = run_sr_group(c, gkey[gi], c->jobs + goff[gi], gcount[gi], fixed ? nullptr : c->job_count + gi, st);
            if (r != NS_OK) break;
            if ((r = run_reconstruct(c, g, ch, S, n, anchor, asrc, st)) != NS_OK) break;
        } else {
            if ((r = recon_prepare(c, g, S, n, anchor, asrc, st)) != NS_OK) break;
            for (int pi = 0; pi < parts && r == NS_OK; pi++) {
                const int s0 = (int)((int64_t)S * pi / parts), s1 = (int)((int64_t)S * (pi + 1) / parts);
                for (int gi = 0; gi < G && r == NS_OK; gi++) {  // this part's job range of group gi
                    int lo = INT32_MAX, hi = -1;
                    for (int s = s0; s < s1; s++)
                        if (group[s] == gi) {
                            lo = std::min(lo, job_base[s]);
                            hi = std::max(hi, job_base[s] + p->k);
                        }
                    if (hi > lo) r = run_sr_group(c, gkey[gi], c->jobs + lo, hi - lo, nullptr, st);
                }
                if (r != NS_OK) break;
                cudaError_t e = cudaEventRecord(c->ev_part[pi & 1], st);
                if (e == cudaSuccess) e = cudaStreamWaitEvent(c->rst, c->ev_part[pi & 1], 0);
                if (e != cudaSuccess) { r = cuda_fail(e, "overlap fork"); break; }
                r = recon_steps(c, ch, s0, s1 - s0, n, c->rst);
            }
            if (r != NS_OK) break;
            NS_CUDA(cudaEventRecord(c->ev_rjoin, c->rst));
            NS_CUDA(cudaStreamWaitEvent(st, c->ev_rjoin, 0));
            if ((r = recon_finish(c, g, ch, S, n, st)) != NS_OK) break;
        }
        if (stats) {
            size_t maxhr = 0;
            for (int s = 0; s < S; s++) maxhr = std::max(maxhr, hr_frame_bytes(ch[s]));
            bool any_gt = false;
            for (int s = 0; s < S; s++) any_gt |= ch[s].gt != nullptr;
            cudaError_t e = launch_stats(g.d_sd, S, n, anchor, c->score, g.d_hr, any_gt ? maxhr : 0, stats, st);
            if (e != cudaSuccess) { r = cuda_fail(e, "stats"); break; }
        }
    } while (0);
    stage_release(c, g.slot, st);
    return r;
}

extern "C" ns_status ns_enhance_streams(ns_ctx *c, const ns_chunk *ch, int S, const ns_select_params *p,
                                        uint8_t *const *hr_out, uint8_t *is_anchor_out, double *stats, void *stream) {
    if (!c) return fail(NS_EINVAL, "ns_enhance_streams: ctx is NULL");
    int n = 0;
    ns_status r = check_chunks(ch, S, true, &n);
    if (r != NS_OK) return r;
    if ((r = check_params(p, S, n)) != NS_OK) return r;
    std::vector<int> ring;
    if ((r = check_hr_table(ch, S, n, hr_out, true, &ring)) != NS_OK) return r;
    NS_CUDA(cudaSetDevice(c->device));
    return enhance_impl(c, ch, S, n, p, hr_out, is_anchor_out ? is_anchor_out : c->anchor, stats,
                        (cudaStream_t)stream, nullptr, nullptr, ring);
}

// ------------------------------------------------------------------ host-input path
static bool host_mapped(const void *p) {
    if (!p) return true;
    cudaPointerAttributes at;
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    return at.type == cudaMemoryTypeHost && at.devicePointer == p;  // UVA: same address on the device
}

// bytes of one stream's uploaded inputs in a staging buffer (256-B aligned pieces)
static size_t host_stream_bytes(const ns_chunk &k) {
    const size_t n = (size_t)k.n_frames, px = (size_t)k.h * k.w;
    return a256(n * lr_frame_elems(k) * 2) + a256(n * (px / 64) * sizeof(ns_block_mv)) + a256(n) +
           (k.res_size ? a256(n * 4) : 0);
}

extern "C" ns_status ns_enhance_streams_host(ns_ctx *c, const ns_chunk *ch, int S, const ns_select_params *p,
                                             uint8_t *const *hr_out, uint8_t *is_anchor_out, double *stats,
                                             uint64_t *h2d_bytes, void *stream) {
    if (!c) return fail(NS_EINVAL, "ns_enhance_streams_host: ctx is NULL");
    int n = 0;
    ns_status r = check_chunks(ch, S, true, &n);
    if (r != NS_OK) return r;
    if ((r = check_params(p, S, n)) != NS_OK) return r;
    std::vector<int> ring;
    if ((r = check_hr_table(ch, S, n, hr_out, true, &ring)) != NS_OK) return r;
    for (int s = 0; s < S; s++)
        if (!host_mapped(ch[s].lr) || !host_mapped(ch[s].res) || !host_mapped(ch[s].mv) || !host_mapped(ch[s].type) ||
            !host_mapped(ch[s].res_size))
            return fail(NS_EINVAL, "chunk %d: lr/res/mv/type/res_size must be page-locked, device-mapped host memory", s);
    NS_CUDA(cudaSetDevice(c->device));
    cudaStream_t st = (cudaStream_t)stream;
    const bool topk = p->mode == NS_TOPK_PER_STREAM;
    // groups of consecutive streams, ~kHostGroups per call: the first group's
    // upload and the last group's compute are the unhidden fill and drain; global
    // budget mode needs all scores before selecting -> one group
    const int gs = topk ? std::max(1, (S + host_groups() - 1) / host_groups()) : S;
    // group sizes: gs each, the last one split into halves and quarters
    // (gs/2, gs/4, gs/4): the drain -- the last group's compute after the final
    // upload -- shrinks 4x, and compute (~0.55 of the upload time per stream)
    // still keeps ahead of the copy stream everywhere else
    std::vector<int> gsz;
    for (int left = S; left > 0; left -= gsz.back()) gsz.push_back(std::min(gs, left));
    if (topk && gsz.size() > 1 && gsz.back() >= 4) {
        const int last = gsz.back();
        gsz.pop_back();
        gsz.push_back(last / 2);
        gsz.push_back((last - last / 2) / 2);
        gsz.push_back(last - last / 2 - (last - last / 2) / 2);
    }
    size_t cap = 0, lr_stride = 0;
    int max_jobs = 0;
    for (int gi = 0, g0 = 0; gi < (int)gsz.size(); g0 += gsz[gi++]) {
        size_t b = 0;
        int jobs = 0;
        for (int s = g0; s < g0 + gsz[gi]; s++) {
            b += host_stream_bytes(ch[s]);
            jobs += topk ? p->k : n;
        }
        cap = std::max(cap, b);
        max_jobs = std::max(max_jobs, jobs);
    }
    for (int s = 0; s < S; s++) lr_stride = std::max(lr_stride, a256(lr_frame_elems(ch[s])));
    if (!topk) {  // one group; job slots as enhance_impl lays them out: per SR shape, min(streams * n, budget / min cost)
        int64_t min_cost = INT64_MAX;
        for (int s = 0; s < S; s++) min_cost = std::min(min_cost, p->cost[s]);
        std::map<GroupKey, int> cnt;
        for (int s = 0; s < S; s++)
            cnt[GroupKey(ch[s].h, ch[s].w, ch[s].model->C, ch[s].scale, ch[s].model->n_blocks, ch[s].format)]++;
        int64_t t = 0;
        for (auto &kv : cnt) t += std::min<int64_t>((int64_t)kv.second * n, p->budget / std::max<int64_t>(min_cost, 1));
        max_jobs = (int)std::min<int64_t>(t, kMaxJobs);
    }
    if (cap > c->hin_cap) {
        for (int i = 0; i < 2; i++) {
            if (c->hin_used[i]) NS_CUDA(cudaEventSynchronize(c->ev_free[i]));
            c->hin_used[i] = false;
            if (!(c->hin[i] = pool_take(c, cap)))
                return fail(NS_ENOMEM, "ns_enhance_streams_host: pool too small for input staging (%zu bytes x 2)", cap);
        }
        c->hin_cap = cap;
    }
    if ((size_t)max_jobs * lr_stride > c->lr_stage_cap) {
        const size_t need = (size_t)max_jobs * lr_stride;
        NS_CUDA(cudaStreamSynchronize(st));  // the old staging may still be read (not the steady state)
        if (!(c->lr_stage = pool_take(c, need)))
            return fail(NS_ENOMEM, "ns_enhance_streams_host: pool too small for anchor LR staging (%zu bytes)", need);
        c->lr_stage_cap = need;
    }
    uint8_t *anchor = is_anchor_out ? is_anchor_out : c->anchor;
    uint64_t moved = 0;
    std::vector<ns_chunk> dch(gs);
    for (int g0 = 0, gi = 0; gi < (int)gsz.size(); g0 += gsz[gi++]) {
        const int b = gi & 1, cnt = gsz[gi];
        // upload group gi into buffer b once the compute that last used b is done
        if (c->hin_used[b]) NS_CUDA(cudaStreamWaitEvent(c->cst, c->ev_free[b], 0));
        uint8_t *dst = c->hin[b];
        for (int i = 0; i < cnt; i++) {
            const ns_chunk &k = ch[g0 + i];
            const size_t nf = (size_t)k.n_frames, px = (size_t)k.h * k.w;
            dch[i] = k;
            const size_t rb = nf * lr_frame_elems(k) * 2, mb = nf * (px / 64) * sizeof(ns_block_mv);
            NS_CUDA(cudaMemcpyAsync(dst, k.res, rb, cudaMemcpyHostToDevice, c->cst));
            dch[i].res = reinterpret_cast<const int16_t *>(dst);
            dst += a256(rb);
            NS_CUDA(cudaMemcpyAsync(dst, k.mv, mb, cudaMemcpyHostToDevice, c->cst));
            dch[i].mv = reinterpret_cast<const ns_block_mv *>(dst);
            dst += a256(mb);
            NS_CUDA(cudaMemcpyAsync(dst, k.type, nf, cudaMemcpyHostToDevice, c->cst));
            dch[i].type = dst;
            dst += a256(nf);
            if (k.res_size) {
                NS_CUDA(cudaMemcpyAsync(dst, k.res_size, nf * 4, cudaMemcpyHostToDevice, c->cst));
                dch[i].res_size = reinterpret_cast<const uint32_t *>(dst);
                dst += a256(nf * 4);
                moved += nf * 4;
            }
            moved += rb + mb + nf;
        }
        NS_CUDA(cudaEventRecord(c->ev_copied[b], c->cst));
        NS_CUDA(cudaStreamWaitEvent(st, c->ev_copied[b], 0));
        LrGather lg{c->lr_stage, lr_stride};
        const std::vector<int> gring(ring.begin() + g0, ring.begin() + g0 + cnt);
        r = enhance_impl(c, dch.data(), cnt, n, p, hr_out + (size_t)g0 * n, anchor + (size_t)g0 * n,
                         stats ? stats + (size_t)8 * g0 : nullptr, st, &lg, &moved, gring);
        if (r != NS_OK) return r;
        NS_CUDA(cudaEventRecord(c->ev_free[b], st));
        c->hin_used[b] = true;
    }
    if (h2d_bytes) *h2d_bytes = moved;
    return NS_OK;
}

// ------------------------------------------------------------------ hybrid encoding (§6.1, NEXT-3)
extern "C" int ns_hybrid_quality(int n_anchors, int n_frames) { return hybrid_quality_table2(n_anchors, n_frames); }

extern "C" ns_status ns_encode_anchors(ns_ctx *c, const ns_chunk *ch, int S, const uint8_t *is_anchor,
                                       uint8_t *const *hr_out, int quality, uint8_t *out, size_t out_cap,
                                       size_t *out_len, void *stream) {
    if (!c) return fail(NS_EINVAL, "ns_encode_anchors: ctx is NULL");
    int n = 0;
    ns_status r = check_chunks(ch, S, false, &n);
    if (r != NS_OK) return r;
    if (!is_anchor || !hr_out || !out_len || (!out && out_cap)) return fail(NS_EINVAL, "ns_encode_anchors: NULL argument");
    if (quality < 0 || quality > 100) return fail(NS_EINVAL, "ns_encode_anchors: quality %d not in [0, 100]", quality);
    std::vector<int> q(S);
    for (int s = 0; s < S; s++) {
        int a = 0;
        for (int f = 0; f < n; f++) {
            a += is_anchor[(size_t)s * n + f] != 0;
            if (is_anchor[(size_t)s * n + f] && !hr_out[(size_t)s * n + f])
                return fail(NS_EINVAL, "ns_encode_anchors: hr_out[%d][%d] is NULL", s, f);
        }
        q[s] = quality ? quality : hybrid_quality_table2(a, n);
        if (q[s] < 1)
            return fail(NS_EUNSUPPORTED, "stream %d: anchor fraction %d/%d above 10%%: JPEG cannot meet the bitrate "
                                         "constraint (Table 2, P:679); pass an explicit quality", s, a, n);
    }
    NS_CUDA(cudaSetDevice(c->device));
    cudaStream_t st = (cudaStream_t)stream;
    char err[256];
    if (!c->hybrid && hybrid_create(c->device, st, &c->hybrid, err, sizeof(err)) != 0) return fail(NS_ECUDA, "%s", err);
    // every anchor, stream-major, frame order
    std::vector<HybridFrame> fr;
    for (int s = 0; s < S; s++)
        for (int f = 0; f < n; f++)
            if (is_anchor[(size_t)s * n + f])
                fr.push_back(HybridFrame{hr_out[(size_t)s * n + f], ch[s].h * ch[s].scale, ch[s].w * ch[s].scale,
                                         ch[s].format, q[s]});
    std::vector<std::vector<uint8_t>> bits;
    if (hybrid_encode_frames(c->hybrid, (int)fr.size(), fr.data(), bits, st, err, sizeof(err)) != 0)
        return fail(NS_ECUDA, "%s", err);
    size_t pos = 0, ai = 0;
    bool full = false;
    for (int s = 0; s < S; s++) {
        const size_t start = pos;
        for (int f = 0; f < n; f++) {
            ns_hybrid_header hd{};
            hd.magic = NS_HYBRID_MAGIC;
            hd.stream = (uint32_t)s;
            hd.frame = (uint16_t)f;
            hd.anchor = is_anchor[(size_t)s * n + f] ? 1 : 0;
            hd.quality = hd.anchor ? (uint8_t)q[s] : 0;
            const std::vector<uint8_t> *pl = hd.anchor ? &bits[ai++] : nullptr;
            hd.bytes = pl ? (uint32_t)pl->size() : 0u;
            const size_t need = sizeof(hd) + hd.bytes;
            if (!full && pos + need <= out_cap) {
                memcpy(out + pos, &hd, sizeof(hd));
                if (pl && !pl->empty()) memcpy(out + pos + sizeof(hd), pl->data(), pl->size());
            } else {
                full = true;
            }
            pos += need;
        }
        out_len[s] = pos - start;
    }
    if (full || pos > out_cap) return fail(NS_ENOMEM, "ns_encode_anchors: out_cap %zu < %zu bytes", out_cap, pos);
    return NS_OK;
}
