// k_select.cu -- anchor scoring (K1), zero-inference anchor selection (K2:
// Alg. 1 + Fig. 10 on one warp per stream), the global budget mode (§5.2) and
// SR job compaction (K3).
#include <cstdint>
#include "ns_internal.h"
#include <algorithm>

namespace ns {

constexpr int64_t kKeyGain = INT64_MAX;  // "equal anchor gain" of key frames

// ---------------------------------------------------------------- K1 score
// score[s][f] = sum_{c,y,x} |res[f][c][y][x]| ("total residual pixel value",
// P:191), or the encoded-size proxy res_size[f] when the stream asks for it.
// Grid (S*n, slabs); 16-B loads of 8 int16; one 64-bit atomic per CTA.
constexpr int kScoreThreads = 256, kScoreUnroll = 8;
__global__ void __launch_bounds__(kScoreThreads) k_score(const StreamDesc *sd, int n, int64_t *score) {
    const int sf = blockIdx.x, s = sf / n, f = sf % n;   // (stream, frame) on x: S*n may exceed 65535
    const StreamDesc d = sd[s];
    if (d.use_res_size && d.res_size) {
        if (blockIdx.y == 0 && threadIdx.x == 0) score[sf] = (int64_t)d.res_size[f];
        return;
    }
    const size_t nvec = (size_t)d.lr_frame / 8;   // 3 h w (4:4:4) or h w 3/2 (4:2:0): all planes
    const uint4 *r = reinterpret_cast<const uint4 *>(d.res + (size_t)f * d.lr_frame);
    const size_t base = (size_t)blockIdx.y * kScoreThreads * kScoreUnroll + threadIdx.x;
    if ((size_t)blockIdx.y * kScoreThreads * kScoreUnroll >= nvec) return;
    uint4 v[kScoreUnroll];
#pragma unroll
    for (int i = 0; i < kScoreUnroll; i++) {
        const size_t idx = base + (size_t)i * kScoreThreads;
        if (idx < nvec) v[i] = __ldg(r + idx);
        else v[i] = make_uint4(0, 0, 0, 0);
    }
    int acc = 0;
#pragma unroll
    for (int i = 0; i < kScoreUnroll; i++) {
        const uint32_t w4[4] = {v[i].x, v[i].y, v[i].z, v[i].w};
#pragma unroll
        for (int j = 0; j < 4; j++) {
            acc += abs((int)(int16_t)(w4[j] & 0xFFFFu)) + abs((int)(int16_t)(w4[j] >> 16));
        }
    }
    for (int off = 16; off; off >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, off);
    __shared__ int part[kScoreThreads / 32];
    if ((threadIdx.x & 31) == 0) part[threadIdx.x >> 5] = acc;
    __syncthreads();
    if (threadIdx.x == 0) {
        long long t = 0;
        for (int i = 0; i < kScoreThreads / 32; i++) t += part[i];
        atomicAdd(reinterpret_cast<unsigned long long *>(score + sf), (unsigned long long)t);
    }
}

cudaError_t launch_score(const StreamDesc *d_sd, int S, int n, int max_frame_vec8, int64_t *score,
                         cudaStream_t st) {
    KScope ks(F_SCORE, st);
    cudaError_t e = cudaMemsetAsync(score, 0, sizeof(int64_t) * S * n, st);
    if (e != cudaSuccess) return e;
    const int per = kScoreThreads * kScoreUnroll;
    dim3 g(S * n, (max_frame_vec8 + per - 1) / per);
    k_score<<<g, kScoreThreads, 0, st>>>(d_sd, n, score);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- K2 select
// One warp per stream; the frames of the chunk live in shared memory.
//   CalcResidual (Alg. 1 l.15-20) and the next-reset table: lane 0, serial.
//   EstimateGain (l.1-14): per iteration every lane evaluates Eq. 1
//     dRes(F[i]) = (k(i) - i) * Res[i] for its undone candidates, a warp
//     argmax picks the strict maximum (lowest frame on ties, Z5), then
//     UpdateResidual (l.21-25) and the next-reset table are updated in parallel.
//   Fig. 10 step 3 within the stream: rank = number of frames ordered before
//     f by (group, gain desc, frame asc); is_anchor = rank < k.
constexpr int kSelWarps = 4;
__global__ void __launch_bounds__(kSelWarps * 32)
    k_select(const StreamDesc *sd, const int64_t *score, int S, int n, int k, int fresh, int selector,
             int64_t *gain_out, int32_t *rank_out, uint8_t *anchor_out, int32_t *order_out) {
    __shared__ int64_t sR[kSelWarps][kMaxFrames];
    __shared__ int64_t sG[kSelWarps][kMaxFrames];
    __shared__ int16_t sNR[kSelWarps][kMaxFrames];
    __shared__ uint8_t sT[kSelWarps][kMaxFrames], sReset[kSelWarps][kMaxFrames], sDone[kSelWarps][kMaxFrames];
    const int wi = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int s = blockIdx.x * kSelWarps + wi;
    if (s >= S) return;  // warp-uniform; only __syncwarp below
    const StreamDesc d = sd[s];
    int64_t *R = sR[wi], *G = sG[wi];
    int16_t *NR = sNR[wi];
    uint8_t *T = sT[wi], *Reset = sReset[wi], *Done = sDone[wi];
    const int64_t *sc = score + (size_t)s * n;
    for (int f = lane; f < n; f += 32) {
        T[f] = d.type[f] & NS_TYPE_MASK;   // an invisible frame keeps its group
        G[f] = (T[f] == NS_KEY) ? kKeyGain : 0;
        Done[f] = 0;
    }
    __syncwarp();
    auto calc_residual = [&]() {
        if (lane == 0) {
            int64_t cur = 0;
            for (int f = 0; f < n; f++) {
                if (T[f] == NS_KEY) cur = 0;
                else cur += sc[f];
                R[f] = cur;
                Reset[f] = (T[f] == NS_KEY);
            }
            int nr = n;
            for (int f = n - 1; f >= 0; f--) {
                NR[f] = (int16_t)nr;
                if (Reset[f]) nr = f;
            }
        }
        __syncwarp();
    };
    auto estimate_gain = [&](int grp) {
        for (;;) {
            int64_t best = -1;
            int bi = n;
            for (int f = lane; f < n; f += 32) {
                if (T[f] == grp && !Done[f]) {
                    const int64_t g = (int64_t)(NR[f] - f) * R[f];
                    if (g > best || (g == best && f < bi)) { best = g; bi = f; }
                }
            }
            for (int off = 16; off; off >>= 1) {
                const int64_t ob = __shfl_xor_sync(0xffffffffu, best, off);
                const int oi = __shfl_xor_sync(0xffffffffu, bi, off);
                if (ob > best || (ob == best && oi < bi)) { best = ob; bi = oi; }
            }
            if (bi >= n) break;
            const int i = bi;
            const int64_t delta = R[i];
            const int kk = NR[i];
            __syncwarp();
            for (int f = lane; f < n; f += 32) {
                if (f >= i && f < kk) R[f] -= delta;
                if (f < i && NR[f] > i) NR[f] = (int16_t)i;
            }
            if (lane == 0) { Done[i] = 1; G[i] = best; Reset[i] = 1; }
            __syncwarp();
        }
    };
    if (selector == NS_SEL_NEUROSCALER) {
        calc_residual();
        estimate_gain(NS_ALTREF);
        if (fresh) calc_residual();
        estimate_gain(NS_NORMAL);
    } else {
        // The real-time baselines of §3.  Frames are re-classed so the
        // rank rule below orders them (class, frame): 0 = key, 1 = the equally
        // spaced frames U = {floor(j n / k)} (Key+Uniform, reading R5; f is in U
        // iff j = ceil(f k / n) < k has floor(j n / k) = f), 2 = the rest.
        int nkey = 0;
        for (int f = lane; f < n; f += 32) {
            int cls = 2;
            if (T[f] == NS_KEY) {
                cls = 0;
                nkey++;
            } else if (selector == NS_SEL_KEY_UNIFORM && k > 0) {
                const int j = (f * k + n - 1) / n;
                if (j < k && (j * n) / k == f) cls = 1;
            }
            T[f] = (uint8_t)cls;
        }
        nkey = __reduce_add_sync(0xffffffffu, nkey);
        if (selector == NS_SEL_KEY && k > nkey) k = nkey;  // Key SR: key frames only (reading R6)
        __syncwarp();
    }
    for (int f = lane; f < n; f += 32) {
        int cnt = 0;
        const int tf = T[f];
        const int64_t gf = G[f];
        for (int g = 0; g < n; g++) {
            const int tg = T[g];
            const int64_t gg = G[g];
            cnt += (tg < tf) || (tg == tf && (gg > gf || (gg == gf && g < f)));
        }
        const size_t o = (size_t)s * n + f;
        gain_out[o] = gf;
        rank_out[o] = cnt;
        if (k >= 0) anchor_out[o] = cnt < k ? 1 : 0;
        if (order_out) order_out[(size_t)s * n + cnt] = f;
    }
}

cudaError_t launch_select(const StreamDesc *d_sd, const int64_t *score, int S, int n, int k, int fresh,
                          int selector, int64_t *gain, int32_t *rank, uint8_t *is_anchor, int32_t *order,
                          cudaStream_t st) {
    KScope ks(F_SELECT, st);
    k_select<<<(S + kSelWarps - 1) / kSelWarps, kSelWarps * 32, 0, st>>>(d_sd, score, S, n, k, fresh, selector,
                                                                        gain, rank, is_anchor, order);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- global budget (§5.2)
// Global position of entry (s, f) in the merged order G_key -> G_altref ->
// G_normal, each by (gain desc, stream asc, frame asc): its rank inside its own
// stream plus, for every other stream, a binary search in that stream's
// sorted order for the entries that precede it.
// FLAT (ns_select_merge): types from a gathered [S][n] array and the stream key
// sid[s] (global stream ids of the streams of every GPU, reading R7).
template <bool FLAT>
__global__ void k_global_rank(const StreamDesc *sd, const uint8_t *type_flat, const int32_t *sid, int S, int n,
                              const int64_t *gain, const int32_t *order, const int32_t *rank_in, int32_t *grank,
                              int32_t *pos_stream) {
    const int e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= S * n) return;
    const int s = e / n, f = e % n;
    auto types = [&](int q) -> const uint8_t * { return FLAT ? type_flat + (size_t)q * n : sd[q].type; };
    auto key = [&](int q) -> int { return FLAT ? sid[q] : q; };
    const int t = types(s)[f] & NS_TYPE_MASK;
    const int ks = key(s);
    const int64_t g = gain[e];
    int cnt = rank_in[e];
    for (int s2 = 0; s2 < S; s2++) {
        if (s2 == s) continue;
        const uint8_t *T2 = types(s2);
        const int k2 = key(s2);
        const int32_t *O2 = order + (size_t)s2 * n;
        const int64_t *G2 = gain + (size_t)s2 * n;
        int lo = 0, hi = n;  // first position whose entry does NOT precede (s, f)
        while (lo < hi) {
            const int mid = (lo + hi) >> 1;
            const int f2 = O2[mid];
            const int t2 = T2[f2] & NS_TYPE_MASK;
            const int64_t g2 = G2[f2];
            const bool prec = (t2 < t) || (t2 == t && (g2 > g || (g2 == g && k2 < ks)));
            if (prec) lo = mid + 1;
            else hi = mid;
        }
        cnt += lo;
    }
    grank[e] = cnt;
    pos_stream[cnt] = s;
}

// Per-stream priority rank of every gathered entry, rebuilt from the entries
// themselves: the number of frames of the same stream ordered before (s, f) by
// (type asc, gain desc, frame asc) -- Fig. 10's per-stream order (KEY gain =
// INT64_MAX, so KEYs order by frame; reading Z5: within a stream this sort is
// the greedy pick order of Alg. 1).  It equals ns_select_anchors' rank in
// NS_TOPK_PER_STREAM / NS_SEL_NEUROSCALER mode, and it is a permutation of
// 0..n-1 for ANY input, so the merge never trusts a caller's rank array.
__global__ void k_stream_rank(int N, int n, const int64_t *gain, const uint8_t *type, int32_t *rank) {
    const int e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= N) return;
    const int s = e / n, f = e % n;
    const uint8_t *T = type + (size_t)s * n;
    const int64_t *G = gain + (size_t)s * n;
    const int t = T[f] & NS_TYPE_MASK;
    const int64_t g = G[f];
    int cnt = 0;
    for (int f2 = 0; f2 < n; f2++) {
        const int t2 = T[f2] & NS_TYPE_MASK;
        const int64_t g2 = G[f2];
        cnt += (t2 < t) || (t2 == t && (g2 > g || (g2 == g && f2 < f)));
    }
    rank[e] = cnt;
}

// order[s][rank[s][f]] = f: the per-stream priority order from the ranks.
__global__ void k_order_from_rank(int N, int n, const int32_t *rank_in, int32_t *order) {
    const int e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= N) return;
    const int s = e / n;
    order[(size_t)s * n + rank_in[e]] = e % n;
}

// Longest prefix of the global order whose summed cost stays <= budget
// (max N with sum_{i<=N} T_DNN(AF[i]) <= T_intv * M; Z7).
__global__ void __launch_bounds__(1024) k_global_cut(int N, const int32_t *pos_stream, const int64_t *cost,
                                                     int64_t budget, int32_t *cut) {
    __shared__ int64_t buf[1024];
    __shared__ int64_t carry;
    __shared__ int count;
    if (threadIdx.x == 0) { carry = 0; count = 0; }
    __syncthreads();
    for (int base = 0; base < N; base += 1024) {
        const int i = base + threadIdx.x;
        buf[threadIdx.x] = (i < N) ? cost[pos_stream[i]] : 0;
        __syncthreads();
        for (int off = 1; off < 1024; off <<= 1) {
            const int64_t v = threadIdx.x >= off ? buf[threadIdx.x - off] : 0;
            __syncthreads();
            buf[threadIdx.x] += v;
            __syncthreads();
        }
        const int64_t pre = carry + buf[threadIdx.x];
        const int ok = (i < N && pre <= budget) ? 1 : 0;
        const int tot = __syncthreads_count(ok);
        if (threadIdx.x == 0) { count += tot; carry += buf[1023]; }
        __syncthreads();
    }
    if (threadIdx.x == 0) *cut = count;
}

__global__ void k_global_mark(int N, const int32_t *grank, const int32_t *cut, int32_t *rank, uint8_t *is_anchor) {
    const int e = blockIdx.x * blockDim.x + threadIdx.x;
    if (e >= N) return;
    rank[e] = grank[e];
    is_anchor[e] = grank[e] < *cut ? 1 : 0;
}

cudaError_t launch_global(const StreamDesc *d_sd, int S, int n, const int64_t *gain, const int32_t *order,
                          const int64_t *cost, int64_t budget, int32_t *grank, int32_t *pos_stream,
                          int32_t *cut, int32_t *rank, uint8_t *is_anchor, cudaStream_t st) {
    KScope ks(F_GLOBAL, st, 3);
    const int N = S * n;
    // rank currently holds the per-stream rank (written by k_select)
    k_global_rank<false><<<(N + 255) / 256, 256, 0, st>>>(d_sd, nullptr, nullptr, S, n, gain, order, rank, grank,
                                                           pos_stream);
    k_global_cut<<<1, 1024, 0, st>>>(N, pos_stream, cost, budget, cut);
    k_global_mark<<<(N + 255) / 256, 256, 0, st>>>(N, grank, cut, rank, is_anchor);
    return cudaGetLastError();
}

cudaError_t launch_merge(int S, int n, const int64_t *gain, const int32_t *rank_in, const uint8_t *type,
                         const int32_t *sid, const int64_t *cost, int64_t budget, int32_t *order, int32_t *grank,
                         int32_t *pos_stream, int32_t *cut, int32_t *rank, uint8_t *is_anchor, cudaStream_t st) {
    (void)rank_in;  // not trusted: the per-stream ranks are rebuilt from (type, gain, frame) into `rank`
    KScope ks(F_GLOBAL, st, 5);
    const int N = S * n;
    k_stream_rank<<<(N + 255) / 256, 256, 0, st>>>(N, n, gain, type, rank);
    k_order_from_rank<<<(N + 255) / 256, 256, 0, st>>>(N, n, rank, order);
    k_global_rank<true><<<(N + 255) / 256, 256, 0, st>>>(nullptr, type, sid, S, n, gain, order, rank, grank,
                                                          pos_stream);
    k_global_cut<<<1, 1024, 0, st>>>(N, pos_stream, cost, budget, cut);
    k_global_mark<<<(N + 255) / 256, 256, 0, st>>>(N, grank, cut, rank, is_anchor);
    return cudaGetLastError();
}

// ---------------------------------------------------------------- K3 compaction
// Anchors of every stream -> SR job table of the stream's shape group.
// Top-k mode: stream s owns slots [job_base, job_base + k) in frame order.
// Other modes (global budget, a given anchor map, Key SR): the anchors of a
// group take consecutive slots stream by stream in the group's list order
// (k_anchor_count + k_group_scan: deterministic, no atomics); an anchor whose
// slot would pass the group's job_cap -- only possible for a given map that
// breaks its budget -- is demoted: is_anchor is cleared and the frame is
// reconstructed like any other (ns.h NS_GIVEN_ANCHORS).
// HR rings: an anchor whose hr_out entry an earlier frame of the stream also
// writes (prv >= 0) cannot be written before the reconstruction runs -- its SR
// output goes to the group's anchor cache and asrc[s][f] records where, for
// the frame step that copies it into place.  Every other anchor is SR'd
// straight into hr_out (always so without rings).
__global__ void k_anchor_count(int S, int n, const uint8_t *is_anchor, int32_t *acount) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= S) return;
    int c = 0;
    for (int f = 0; f < n; f++) c += is_anchor[(size_t)s * n + f] != 0;
    acount[s] = c;
}

// One CTA per group: exclusive scan of the anchor counts over the group's
// streams in list order -> acount[s] becomes the stream's first slot offset;
// job_count[g] = the slots the group fills (<= its cap).
__global__ void __launch_bounds__(1024) k_group_scan(const StreamDesc *sd, const int32_t *glist, const int32_t *goff,
                                                     int32_t *acount, int32_t *job_count) {
    __shared__ int32_t buf[1024];
    __shared__ int32_t carry;
    const int g = blockIdx.x, i0 = goff[g], i1 = goff[g + 1];
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (int base = i0; base < i1; base += 1024) {
        const int i = base + threadIdx.x;
        const int v = i < i1 ? acount[glist[i]] : 0;
        buf[threadIdx.x] = v;
        __syncthreads();
        for (int off = 1; off < 1024; off <<= 1) {
            const int32_t t = threadIdx.x >= off ? buf[threadIdx.x - off] : 0;
            __syncthreads();
            buf[threadIdx.x] += t;
            __syncthreads();
        }
        if (i < i1) acount[glist[i]] = carry + buf[threadIdx.x] - v;
        __syncthreads();
        if (threadIdx.x == 0) carry += buf[1023];
        __syncthreads();
    }
    if (threadIdx.x == 0 && i1 > i0) job_count[g] = min(carry, sd[glist[i0]].job_cap);
}

__global__ void k_compact(const StreamDesc *sd, int S, int n, uint8_t *is_anchor, uint8_t *const *hr_tab,
                          SrJob *jobs, const int32_t *start, int topk, const int16_t *prv, const uint8_t **asrc,
                          uint8_t *lr_stage,
                          size_t lr_stride, const uint8_t **lr_src, uint32_t *lr_len) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= S) return;
    const StreamDesc d = sd[s];
    const size_t lr_frame = (size_t)d.lr_frame;
    int claim = topk ? 0 : start[s];
    for (int f = 0; f < n; f++) {
        const size_t e = (size_t)s * n + f;
        if (asrc) asrc[e] = nullptr;
        if (!is_anchor[e]) continue;
        if (claim >= d.job_cap) {  // over the bound of a given anchor map: demoted (ns.h)
            is_anchor[e] = 0;
            continue;
        }
        const int slot = d.job_base + claim++;
        SrJob j;
        j.lr = d.lr + f * lr_frame;
        const bool direct = !prv || prv[e] < 0;
        j.hr = direct ? hr_tab[d.hr_base + f] : d.acache + (size_t)(slot - d.job_goff) * d.acache_stride;
        j.wts = d.wts;
        if (!direct) asrc[e] = j.hr;
        if (lr_stage) {  // host-resident LR: gather into device staging, SR reads the copy
            lr_src[slot] = j.lr;
            lr_len[slot] = (uint32_t)lr_frame;
            j.lr = lr_stage + (size_t)slot * lr_stride;
        }
        jobs[slot] = j;
    }
}

// One CTA row per job, CTAs stride over the frame in 16-B words: wide,
// coalesced reads of page-locked host memory over PCIe.
__global__ void k_lr_gather(const SrJob *jobs, const uint8_t *const *lr_src, const uint32_t *lr_len) {
    const int j = blockIdx.x;   // jobs on x (up to 2^20), CTAs of one job on y
    const uint32_t len = lr_len[j];
    if (len == 0) return;
    const uint4 *src = reinterpret_cast<const uint4 *>(lr_src[j]);
    uint4 *dst = reinterpret_cast<uint4 *>(const_cast<uint8_t *>(jobs[j].lr));
    const uint32_t nw = len / 16;
    for (uint32_t i = blockIdx.y * blockDim.x + threadIdx.x; i < nw; i += gridDim.y * blockDim.x) dst[i] = src[i];
}

cudaError_t launch_lr_gather(const SrJob *jobs, const uint8_t *const *lr_src, const uint32_t *lr_len, int max_jobs,
                             size_t max_len, cudaStream_t st) {
    KScope ks(F_COMPACT, st);
    const int bx = (int)std::min<size_t>((max_len / 16 + 1023) / 1024, 256);
    k_lr_gather<<<dim3(max_jobs, std::max(bx, 1)), 256, 0, st>>>(jobs, lr_src, lr_len);
    return cudaGetLastError();
}

cudaError_t launch_compact(const StreamDesc *d_sd, int S, int n, uint8_t *is_anchor, uint8_t *const *d_hr_table,
                           SrJob *jobs, int32_t *job_count, int n_groups, const int32_t *glist,
                           const int32_t *goff, int32_t *acount, int topk, const int16_t *prv,
                           const uint8_t **asrc, cudaStream_t st, uint8_t *lr_stage, size_t lr_stride,
                           const uint8_t **lr_src, uint32_t *lr_len) {
    KScope ks(F_COMPACT, st, topk ? 1 : 3);
    if (!topk) {
        cudaError_t e = cudaMemsetAsync(job_count, 0, sizeof(int32_t) * n_groups, st);
        if (e != cudaSuccess) return e;
        k_anchor_count<<<(S + 127) / 128, 128, 0, st>>>(S, n, is_anchor, acount);
        k_group_scan<<<n_groups, 1024, 0, st>>>(d_sd, glist, goff, acount, job_count);
    }
    k_compact<<<(S + 127) / 128, 128, 0, st>>>(d_sd, S, n, is_anchor, d_hr_table, jobs, acount, topk, prv, asrc,
                                               lr_stage, lr_stride, lr_src, lr_len);
    return cudaGetLastError();
}

}  // namespace ns
