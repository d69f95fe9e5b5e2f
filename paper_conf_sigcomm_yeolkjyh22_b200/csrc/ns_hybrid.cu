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

struct HybridEncoder {
    int device = -1;
    nvjpegHandle_t h = nullptr;
    nvjpegEncoderState_t st = nullptr;
    nvjpegEncoderParams_t prm = nullptr;
    int quality = -1;
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
    if (e->prm) nvjpegEncoderParamsDestroy(e->prm);
    if (e->st) nvjpegEncoderStateDestroy(e->st);
    if (e->h) nvjpegDestroy(e->h);
    delete e;
}

// 0 on success, else writes a message into err.
int hybrid_create(int device, cudaStream_t stream, HybridEncoder **out, char *err, size_t errlen) {
    HybridEncoder *e = new HybridEncoder();
    e->device = device;
    nvjpegStatus_t s = nvjpegCreateSimple(&e->h);
    if (s == NVJPEG_STATUS_SUCCESS) s = nvjpegEncoderStateCreate(e->h, &e->st, stream);
    if (s == NVJPEG_STATUS_SUCCESS) s = nvjpegEncoderParamsCreate(e->h, &e->prm, stream);
    // the three planes are full resolution (reading Z18): keep them so
    if (s == NVJPEG_STATUS_SUCCESS) s = nvjpegEncoderParamsSetSamplingFactors(e->prm, NVJPEG_CSS_444, stream);
    // optimized Huffman tables cost a second pass over the coefficients; off unless asked for
    // (NS_JPEG_OPT_HUFFMAN=1: a tuning experiment)
    const char *oh = getenv("NS_JPEG_OPT_HUFFMAN");
    if (s == NVJPEG_STATUS_SUCCESS) s = nvjpegEncoderParamsSetOptimizedHuffman(e->prm, oh && atoi(oh) ? 1 : 0, stream);
    if (s != NVJPEG_STATUS_SUCCESS) {
        snprintf(err, errlen, "nvjpeg encoder setup: %s", nvj_err(s));
        hybrid_destroy(e);
        return -1;
    }
    *out = e;
    return 0;
}

// Encodes one HR frame [3][H][W] (device, planar) at `quality` and appends the
// bitstream at dst (host) if it fits in cap; *len = its size.  Returns 0, 1 if
// it does not fit (len still set), -1 on an nvjpeg error.
int hybrid_encode_frame(HybridEncoder *e, const uint8_t *hr, int H, int W, int fmt, int quality, uint8_t *dst,
                        size_t cap, size_t *len, cudaStream_t stream, char *err, size_t errlen) {
    nvjpegStatus_t s = NVJPEG_STATUS_SUCCESS;
    if (quality != e->quality) {
        s = nvjpegEncoderParamsSetQuality(e->prm, quality, stream);
        if (s != NVJPEG_STATUS_SUCCESS) {
            snprintf(err, errlen, "nvjpegEncoderParamsSetQuality(%d): %s", quality, nvj_err(s));
            return -1;
        }
        e->quality = quality;
    }
    nvjpegImage_t img{};
    const size_t plane = (size_t)H * W;
    if (fmt == NS_FMT_I420) {  // the codec's own planes: Y, then U, V at half resolution, coded as 4:2:0
        img.channel[0] = const_cast<uint8_t *>(hr);
        img.channel[1] = const_cast<uint8_t *>(hr) + plane;
        img.channel[2] = const_cast<uint8_t *>(hr) + plane + plane / 4;
        img.pitch[0] = (size_t)W;
        img.pitch[1] = img.pitch[2] = (size_t)W / 2;
        s = nvjpegEncoderParamsSetSamplingFactors(e->prm, NVJPEG_CSS_420, stream);
        if (s == NVJPEG_STATUS_SUCCESS) s = nvjpegEncodeYUV(e->h, e->st, e->prm, &img, NVJPEG_CSS_420, W, H, stream);
        if (s == NVJPEG_STATUS_SUCCESS) s = nvjpegEncoderParamsSetSamplingFactors(e->prm, NVJPEG_CSS_444, stream);
    } else {
        for (int c = 0; c < 3; c++) {
            img.channel[c] = const_cast<uint8_t *>(hr) + c * plane;
            img.pitch[c] = (size_t)W;
        }
        s = nvjpegEncodeImage(e->h, e->st, e->prm, &img, NVJPEG_INPUT_RGB, W, H, stream);
    }
    if (s == NVJPEG_STATUS_SUCCESS) s = nvjpegEncodeRetrieveBitstream(e->h, e->st, nullptr, len, stream);
    if (s != NVJPEG_STATUS_SUCCESS) {
        snprintf(err, errlen, "nvjpegEncodeImage %dx%d: %s", W, H, nvj_err(s));
        return -1;
    }
    if (*len > cap) return 1;
    s = nvjpegEncodeRetrieveBitstream(e->h, e->st, dst, len, stream);
    if (s == NVJPEG_STATUS_SUCCESS && cudaStreamSynchronize(stream) != cudaSuccess) s = NVJPEG_STATUS_EXECUTION_FAILED;
    if (s != NVJPEG_STATUS_SUCCESS) {
        snprintf(err, errlen, "nvjpegEncodeRetrieveBitstream: %s", nvj_err(s));
        return -1;
    }
    return 0;
}

}  // namespace ns
