// ns_hybrid.cu -- hybrid encoding of the super-resolved anchors (§6.1
// "Hybrid video encoding"): the ingest video
// is reused as is, only the SR anchor frames are compressed with an image
// codec -- JPEG here, through nvJPEG (a library call, like cuBLAS), at the
// quality Table 2 assigns to the chunk's anchor fraction -- and
// every frame gets a header (frame type, SR image for an anchor).
// Host-side glue; the encoder object lives in the context (created on first
// use, not on the hot path).
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <nvjpeg.h>
#include <algorithm>
#include <vector>
#include "ns_internal.h"

namespace ns {

// Table 2, JPEG column: quality by the fraction of anchor frames.
//   fraction <= 5% -> 95;  5% < f <= 7.5% -> 90;  7.5% < f <= 10% -> 80;
//   f > 10%: "JPEG ... cannot meet the bitrate constraint" -> -1.
// Exact integer comparisons of n_anchors / n_frames against 1/20, 3/40, 1/10.
int hybrid_quality_table2(int n_anchors, int n_frames) {
    if (n_frames < 1 || n_anchors < 0 || n_anchors > n_frames) return -1;
    const long a = n_anchors, n = n_frames;
    if (20 * a <= n) return 95;
    if (40 * a <= 3 * n) return 90;
    if (10 * a <= n) return 80;
    return -1;
}

// K encoder states on K streams: anchor i is encoded in slot i % K, so up to K
// encodes are in flight while the bitstream of the oldest one is retrieved (in
// anchor order).  nvJPEG retrieval synchronises its stream.
constexpr int kEncSlots = 4;
struct HybridEncoder {
    int device = -1;
    nvjpegHandle_t h = nullptr;
    nvjpegEncoderState_t st[kEncSlots] = {};
    nvjpegEncoderParams_t prm[kEncSlots] = {};
    cudaStream_t cs[kEncSlots] = {};
    cudaEvent_t ready = nullptr;
    int quality[kEncSlots] = {-1, -1, -1, -1};
    int css[kEncSlots] = {-1, -1, -1, -1};
};

static const char *nvj_err(nvjpegStatus_t s) {
    switch (s) {
        case NVJPEG_STATUS_SUCCESS: return "success";
        case NVJPEG_STATUS_NOT_INITIALIZED: return "not initialized";
        case NVJPEG_STATUS_INVALID_PARAMETER: return "invalid parameter";
        case NVJPEG_STATUS_BAD_JPEG: return "bad jpeg";
        case NVJPEG_STATUS_JPEG_NOT_SUPPORTED: return "not supported";
        case NVJPEG_STATUS_ALLOCATOR_FAILURE: return "allocator failure";
        case NVJPEG_STATUS_EXECUTION_FAILED: return "execution failed";
        case NVJPEG_STATUS_ARCH_MISMATCH: return "arch mismatch";
        case NVJPEG_STATUS_INTERNAL_ERROR: return "internal error";
        default: return "nvjpeg error";
    }
}

void hybrid_destroy(HybridEncoder *e) {
    if (!e) return;
    for (int i = 0; i < kEncSlots; i++) {
        if (e->prm[i]) nvjpegEncoderParamsDestroy(e->prm[i]);
        if (e->st[i]) nvjpegEncoderStateDestroy(e->st[i]);
        if (e->cs[i]) cudaStreamDestroy(e->cs[i]);
    }
    if (e->ready) cudaEventDestroy(e->ready);
    if (e->h) nvjpegDestroy(e->h);
    delete e;
}

// 0 on success, else writes a message into err.
int hybrid_create(int device, cudaStream_t stream, HybridEncoder **out, char *err, size_t errlen) {
    (void)stream;
    HybridEncoder *e = new HybridEncoder();
    e->device = device;
    nvjpegStatus_t s = nvjpegCreateSimple(&e->h);
    // optimized Huffman tables cost a second pass over the coefficients; off unless asked for
    // (NS_JPEG_OPT_HUFFMAN=1: a tuning experiment -- measured equal speed, 5% smaller files)
    const char *oh = getenv("NS_JPEG_OPT_HUFFMAN");
    for (int i = 0; i < kEncSlots && s == NVJPEG_STATUS_SUCCESS; i++) {
        if (cudaStreamCreateWithFlags(&e->cs[i], cudaStreamNonBlocking) != cudaSuccess) s = NVJPEG_STATUS_EXECUTION_FAILED;
        if (s == NVJPEG_STATUS_SUCCESS) s = nvjpegEncoderStateCreate(e->h, &e->st[i], e->cs[i]);
        if (s == NVJPEG_STATUS_SUCCESS) s = nvjpegEncoderParamsCreate(e->h, &e->prm[i], e->cs[i]);
        if (s == NVJPEG_STATUS_SUCCESS)
            s = nvjpegEncoderParamsSetOptimizedHuffman(e->prm[i], oh && atoi(oh) ? 1 : 0, e->cs[i]);
    }
    if (s == NVJPEG_STATUS_SUCCESS && cudaEventCreateWithFlags(&e->ready, cudaEventDisableTiming) != cudaSuccess)
        s = NVJPEG_STATUS_EXECUTION_FAILED;
    if (s != NVJPEG_STATUS_SUCCESS) {
        snprintf(err, errlen, "nvjpeg encoder setup: %s", nvj_err(s));
        hybrid_destroy(e);
        return -1;
    }
    *out = e;
    return 0;
}

// Encodes n frames (HR planes, device) in order; out[i] receives frame i's
// bitstream (host).  The encoder streams wait for `stream` first (the frames
// were produced there).  0 on success, -1 on an nvjpeg error.
int hybrid_encode_frames(HybridEncoder *e, int n, const HybridFrame *fr, std::vector<std::vector<uint8_t>> &out,
                         cudaStream_t stream, char *err, size_t errlen) {
    out.assign(n, {});
    if (n == 0) return 0;
    if (cudaEventRecord(e->ready, stream) != cudaSuccess) {
        snprintf(err, errlen, "hybrid encode: event record failed");
        return -1;
    }
    for (int i = 0; i < kEncSlots; i++) cudaStreamWaitEvent(e->cs[i], e->ready, 0);
    auto encode = [&](int i) -> nvjpegStatus_t {
        const int k = i % kEncSlots;
        const HybridFrame &f = fr[i];
        nvjpegStatus_t s = NVJPEG_STATUS_SUCCESS;
        if (f.quality != e->quality[k]) {
            s = nvjpegEncoderParamsSetQuality(e->prm[k], f.quality, e->cs[k]);
            e->quality[k] = f.quality;
        }
        const int css = f.fmt == NS_FMT_I420 ? (int)NVJPEG_CSS_420 : (int)NVJPEG_CSS_444;
        if (s == NVJPEG_STATUS_SUCCESS && css != e->css[k]) {
            s = nvjpegEncoderParamsSetSamplingFactors(e->prm[k], (nvjpegChromaSubsampling_t)css, e->cs[k]);
            e->css[k] = css;
        }
        if (s != NVJPEG_STATUS_SUCCESS) return s;
        nvjpegImage_t img{};
        const size_t plane = (size_t)f.H * f.W;
        if (f.fmt == NS_FMT_I420) {  // the codec's own planes: Y, then U, V at half resolution, coded as 4:2:0
            img.channel[0] = const_cast<uint8_t *>(f.hr);
            img.channel[1] = const_cast<uint8_t *>(f.hr) + plane;
            img.channel[2] = const_cast<uint8_t *>(f.hr) + plane + plane / 4;
            img.pitch[0] = (size_t)f.W;
            img.pitch[1] = img.pitch[2] = (size_t)f.W / 2;
            return nvjpegEncodeYUV(e->h, e->st[k], e->prm[k], &img, NVJPEG_CSS_420, f.W, f.H, e->cs[k]);
        }
        for (int c = 0; c < 3; c++) {
            img.channel[c] = const_cast<uint8_t *>(f.hr) + c * plane;
            img.pitch[c] = (size_t)f.W;
        }
        return nvjpegEncodeImage(e->h, e->st[k], e->prm[k], &img, NVJPEG_INPUT_RGB, f.W, f.H, e->cs[k]);
    };
    auto retrieve = [&](int i) -> nvjpegStatus_t {
        const int k = i % kEncSlots;
        size_t len = 0;
        nvjpegStatus_t s = nvjpegEncodeRetrieveBitstream(e->h, e->st[k], nullptr, &len, e->cs[k]);
        if (s != NVJPEG_STATUS_SUCCESS) return s;
        out[i].resize(len);
        s = nvjpegEncodeRetrieveBitstream(e->h, e->st[k], out[i].data(), &len, e->cs[k]);
        if (s == NVJPEG_STATUS_SUCCESS && cudaStreamSynchronize(e->cs[k]) != cudaSuccess)
            s = NVJPEG_STATUS_EXECUTION_FAILED;
        out[i].resize(len);
        return s;
    };
    for (int i = 0; i < n; i++) {
        if (i >= kEncSlots) {
            const nvjpegStatus_t s = retrieve(i - kEncSlots);
            if (s != NVJPEG_STATUS_SUCCESS) {
                snprintf(err, errlen, "nvjpegEncodeRetrieveBitstream: %s", nvj_err(s));
                return -1;
            }
        }
        const nvjpegStatus_t s = encode(i);
        if (s != NVJPEG_STATUS_SUCCESS) {
            snprintf(err, errlen, "nvjpeg encode %dx%d: %s", fr[i].W, fr[i].H, nvj_err(s));
            return -1;
        }
    }
    for (int i = std::max(0, n - kEncSlots); i < n; i++) {
        const nvjpegStatus_t s = retrieve(i);
        if (s != NVJPEG_STATUS_SUCCESS) {
            snprintf(err, errlen, "nvjpegEncodeRetrieveBitstream: %s", nvj_err(s));
            return -1;
        }
    }
    return 0;
}

}  // namespace ns
