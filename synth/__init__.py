"""Seeded synthetic workload for the NeuroScaler hot path -- INPUTS ONLY.

This module is shared by the oracle tests, the GPU parity tests and bench.py.
It holds none of the method's arithmetic (no anchor gain, no selection, no SR,
no reconstruction).  It synthesises what the paper's modified VP9 decoder
exports (§7: "frame type, residual"; §2: "reference
index, motion vector, residual") plus per-stream content-aware DNN weights
(P:81), because the paper's videos, codecs and trained weights are not
available.

Recipe:
  * content = smooth gradient + band-limited noise + hard-edged rectangles,
    panned globally by a per-profile velocity (1/8 LR pel per frame), plus
    moving textured sprites (six Twitch content categories -> six
    motion/texture profiles);
  * a codec-like LR loop: 8x8-block motion vectors in 1/8 LR pel (true motion
    plus +-1/8 jitter), reference LAST / GOLDEN (~15%) / INTRA (~2%), LR
    motion-compensated prediction, residual quantised with step 4 (NORMAL),
    2 (ALTREF, "high-quality" reference) or 2 (KEY), decoded LR =
    clip(pred + res);
  * frame types: KEY at frame 0, ALTREF every ``altref_every`` frames
    (lag-in-frames 16), NORMAL otherwise.

The LR prediction inside the codec loop is the *encoder side* of the synthetic
codec; it is written independently of oracle/ and of the CUDA path.
"""
from __future__ import annotations

import dataclasses
import numpy as np

NS_KEY, NS_ALTREF, NS_NORMAL = 0, 1, 2
NS_REF_LAST, NS_REF_GOLDEN, NS_REF_INTRA = 0, 1, 2

# ns_block_mv in include/ns.h: { int16 mvx, mvy; uint8 ref; uint8 filter; uint8 pad[2]; }
MV_DTYPE = np.dtype([("mvx", "<i2"), ("mvy", "<i2"), ("ref", "u1"), ("filter", "u1"), ("pad", "u1", (2,))])

# Sub-pel interpolation of the synthetic codec (ns_chunk.interp): 0 = two-pass
# bilinear; 1 / 2 / 3 = VP9's 8-tap regular / smooth / sharp kernel for every
# block; 4 = per block (MV_DTYPE.filter: 0 regular, 1 smooth, 2 sharp).
INTERP_BILINEAR, INTERP_REGULAR, INTERP_SMOOTH, INTERP_SHARP, INTERP_SWITCHABLE = 0, 1, 2, 3, 4
# VP9's 8-tap kernels as published in libvpx (vp9_filter.c), phases 0..8; the
# codec mirrors them for phases 9..15 (phase 16-p = phase p reversed).
_VP9_HALF = {
    0: [[0, 0, 0, 128, 0, 0, 0, 0], [0, 1, -5, 126, 8, -3, 1, 0], [-1, 3, -10, 122, 18, -6, 2, 0],
        [-1, 4, -13, 118, 27, -9, 3, -1], [-1, 4, -16, 112, 37, -11, 4, -1], [-1, 5, -18, 105, 48, -14, 4, -1],
        [-1, 5, -19, 97, 58, -16, 5, -1], [-1, 6, -19, 88, 68, -18, 5, -1], [-1, 6, -19, 78, 78, -19, 6, -1]],
    1: [[0, 0, 0, 128, 0, 0, 0, 0], [-3, -1, 32, 64, 38, 1, -3, 0], [-2, -2, 29, 63, 41, 2, -3, 0],
        [-2, -2, 26, 63, 43, 4, -4, 0], [-2, -3, 24, 62, 46, 5, -4, 0], [-2, -3, 21, 60, 49, 7, -4, 0],
        [-1, -4, 18, 59, 51, 9, -4, 0], [-1, -4, 16, 57, 53, 12, -4, -1], [-1, -4, 14, 55, 55, 14, -4, -1]],
    2: [[0, 0, 0, 128, 0, 0, 0, 0], [-1, 3, -7, 127, 8, -3, 1, 0], [-2, 5, -13, 125, 17, -6, 3, -1],
        [-3, 7, -17, 121, 27, -10, 5, -2], [-4, 9, -20, 115, 37, -13, 6, -2], [-4, 10, -23, 108, 48, -16, 8, -3],
        [-4, 10, -24, 100, 59, -19, 9, -3], [-4, 11, -24, 90, 70, -21, 10, -4], [-4, 11, -23, 80, 80, -23, 11, -4]],
}
VP9_KERNELS = np.array([h + [r[::-1] for r in h[7:0:-1]] for h in (_VP9_HALF[0], _VP9_HALF[1], _VP9_HALF[2])],
                       np.int64)   # [kernel][phase 0..15][tap]

# Six motion/texture profiles named after the paper's six Twitch categories
# (P:275).  pan = (vx, vy) in 1/8 LR pel per frame; noise = amplitude of the
# band-limited texture; sprites = number of independently moving objects.
PROFILES = [
    dict(name="just_chatting", pan=(0, 0), noise=18.0, blur=3, sprites=2, spd=6),
    dict(name="gta_v", pan=(-12, 5), noise=30.0, blur=2, sprites=3, spd=10),
    dict(name="league_of_legends", pan=(8, 2), noise=24.0, blur=1, sprites=6, spd=12),
    dict(name="valorant", pan=(16, -6), noise=28.0, blur=2, sprites=2, spd=16),
    dict(name="fortnite", pan=(5, 5), noise=22.0, blur=2, sprites=4, spd=9),
    dict(name="minecraft", pan=(3, 1), noise=35.0, blur=0, sprites=3, spd=8),
]


@dataclasses.dataclass
class Chunk:
    """One stream's chunk (= GOP) as the decoder would export it."""
    w: int
    h: int
    scale: int
    lr: np.ndarray        # u8  [n][3][h][w]
    res: np.ndarray       # i16 [n][3][h][w]
    mv: np.ndarray        # MV_DTYPE [n][h/8][w/8]
    type: np.ndarray      # u8  [n]
    res_size: np.ndarray  # u32 [n] encoded-size proxy
    gt: np.ndarray | None = None  # u8 [n][3][s*h][s*w] (only with_gt=True)
    interp: int = INTERP_BILINEAR  # the codec's sub-pel filter (ns_chunk.interp)

    @property
    def n(self) -> int:
        return int(self.type.shape[0])


def default_types(n: int, altref_every: int | None = 16, altref_at=None) -> np.ndarray:
    t = np.full(n, NS_NORMAL, np.uint8)
    t[0] = NS_KEY
    if altref_at is not None:
        for a in altref_at:
            t[a] = NS_ALTREF
    elif altref_every:
        t[altref_every::altref_every] = NS_ALTREF
    return t


def _blur(a: np.ndarray, r: int, passes: int = 3) -> np.ndarray:
    """Separable box blur over the last two axes (repeated -> ~Gaussian)."""
    if r <= 0:
        return a
    for _ in range(passes):
        for ax in (1, 2):
            n = a.shape[ax]
            c = np.cumsum(a, axis=ax, dtype=np.float64)
            c = np.concatenate([np.zeros_like(np.take(c, [0], axis=ax)), c], axis=ax)
            hi = np.minimum(np.arange(n) + r + 1, n)
            lo = np.maximum(np.arange(n) - r, 0)
            shape = [1] * a.ndim
            shape[ax] = n
            a = ((np.take(c, hi, axis=ax) - np.take(c, lo, axis=ax)) / (hi - lo).reshape(shape)).astype(np.float32)
    return a


def _sample_bilinear(img: np.ndarray, ys: np.ndarray, xs: np.ndarray) -> np.ndarray:
    """Float bilinear sampling of img[c][Y][X] at (ys, xs) (broadcast 2-D grids)."""
    H, W = img.shape[1:]
    y0 = np.floor(ys).astype(np.int64)
    x0 = np.floor(xs).astype(np.int64)
    fy = (ys - y0).astype(np.float32)
    fx = (xs - x0).astype(np.float32)
    y0c = np.clip(y0, 0, H - 1); y1c = np.clip(y0 + 1, 0, H - 1)
    x0c = np.clip(x0, 0, W - 1); x1c = np.clip(x0 + 1, 0, W - 1)
    a = img[:, y0c, x0c]; b = img[:, y0c, x1c]
    c = img[:, y1c, x0c]; d = img[:, y1c, x1c]
    return (a * (1 - fx) + b * fx) * (1 - fy) + (c * (1 - fx) + d * fx) * fy


class _Scene:
    """Procedural scene: a panned base texture plus moving sprites."""

    def __init__(self, rng: np.random.Generator, w: int, h: int, n: int, prof: dict, up: int):
        self.w, self.h, self.up = w, h, up
        vx, vy = prof["pan"]
        self.v = (vx, vy)
        mx = abs(vx) * n // 8 + 4
        my = abs(vy) * n // 8 + 4
        self.mx, self.my = mx, my
        # base texture at LR resolution (+ margin for the pan); sampled at
        # sub-pixel positions for both LR and (upscaled) GT rendering.
        H, W = h + 2 * my, w + 2 * mx
        yy, xx = np.meshgrid(np.arange(H, dtype=np.float32), np.arange(W, dtype=np.float32), indexing="ij")
        base = np.empty((3, H, W), np.float32)
        for c in range(3):
            g = rng.uniform(-0.25, 0.25, 2) * 100.0 / max(H, W)
            base[c] = 128 + g[0] * (xx - W / 2) + g[1] * (yy - H / 2) + rng.uniform(-20, 20)
        noise = rng.standard_normal((3, H, W)).astype(np.float32)
        noise = _blur(noise, prof["blur"])
        noise *= prof["noise"] / max(float(noise.std()), 1e-6)
        base += noise
        for _ in range(max(2, (H * W) // 6000)):
            y0, x0 = rng.integers(0, H), rng.integers(0, W)
            hh, ww = rng.integers(4, max(5, H // 6)), rng.integers(4, max(5, W // 6))
            base[:, y0:y0 + hh, x0:x0 + ww] += rng.uniform(-40, 40, (3, 1, 1)).astype(np.float32)
        self.base = base
        self.sprites = []
        for _ in range(prof["sprites"]):
            sh_, sw_ = int(rng.integers(8, max(9, h // 4))), int(rng.integers(8, max(9, w // 4)))
            tex = rng.uniform(30, 225, (3, 1, 1)).astype(np.float32) + \
                8 * rng.standard_normal((3, sh_, sw_)).astype(np.float32)
            p0 = (float(rng.uniform(0, h - sh_)), float(rng.uniform(0, w - sw_)))
            spd = prof["spd"]
            u = (int(rng.integers(-spd, spd + 1)), int(rng.integers(-spd, spd + 1)))
            self.sprites.append((tex, p0, u))

    def pan_pos(self, f: int):
        return (f * self.v[1] / 8.0, f * self.v[0] / 8.0)

    def sprite_pos(self, k: int, f: int):
        tex, p0, u = self.sprites[k]
        return (p0[0] + f * u[1] / 8.0, p0[1] + f * u[0] / 8.0)

    def render(self, f: int, s: int) -> np.ndarray:
        """Render frame f at s x the LR resolution (float32 [3][s*h][s*w])."""
        py, px = self.pan_pos(f)
        if s == 1:
            # constant sub-pixel pan: lerp of four shifted slices
            iy, ix = int(np.floor(py)), int(np.floor(px))
            fy, fx = np.float32(py - iy), np.float32(px - ix)
            y0, x0 = self.my + iy, self.mx + ix
            b = self.base
            a00 = b[:, y0:y0 + self.h, x0:x0 + self.w]
            a01 = b[:, y0:y0 + self.h, x0 + 1:x0 + 1 + self.w]
            a10 = b[:, y0 + 1:y0 + 1 + self.h, x0:x0 + self.w]
            a11 = b[:, y0 + 1:y0 + 1 + self.h, x0 + 1:x0 + 1 + self.w]
            img = (a00 * (1 - fx) + a01 * fx) * (1 - fy) + (a10 * (1 - fx) + a11 * fx) * fy
        else:
            Y = (np.arange(self.h * s, dtype=np.float32) + 0.5) / s - 0.5
            X = (np.arange(self.w * s, dtype=np.float32) + 0.5) / s - 0.5
            img = _sample_bilinear(self.base, (Y + self.my + py)[:, None], (X + self.mx + px)[None, :])
        for k, (tex, _, _) in enumerate(self.sprites):
            sy, sx = self.sprite_pos(k, f)
            th, tw = tex.shape[1:]
            y0 = int(np.floor(sy * s)); x0 = int(np.floor(sx * s))
            y1 = y0 + th * s; x1 = x0 + tw * s
            cy0, cy1 = max(y0, 0), min(y1, self.h * s)
            cx0, cx1 = max(x0, 0), min(x1, self.w * s)
            if cy0 >= cy1 or cx0 >= cx1:
                continue
            ty = (np.arange(cy0, cy1, dtype=np.float32) - sy * s + 0.5) / s - 0.5
            tx = (np.arange(cx0, cx1, dtype=np.float32) - sx * s + 0.5) / s - 0.5
            img[:, cy0:cy1, cx0:cx1] = _sample_bilinear(tex, ty[:, None], tx[None, :])
        return img

    def block_motion(self, f: int, r: int, bh: int, bw: int) -> tuple[np.ndarray, np.ndarray]:
        """True motion (1/8 LR pel) of each 8x8 block of frame f w.r.t. frame r:
        pred(x) = ref(x + mv)."""
        mvx = np.full((bh, bw), (f - r) * self.v[0], np.int32)
        mvy = np.full((bh, bw), (f - r) * self.v[1], np.int32)
        cy = np.arange(bh) * 8 + 4
        cx = np.arange(bw) * 8 + 4
        for k, (tex, _, u) in enumerate(self.sprites):
            sy, sx = self.sprite_pos(k, f)
            th, tw = tex.shape[1:]
            iny = (cy >= sy) & (cy < sy + th)
            inx = (cx >= sx) & (cx < sx + tw)
            m = iny[:, None] & inx[None, :]
            mvx[m] = -(f - r) * u[0]
            mvy[m] = -(f - r) * u[1]
        return mvx, mvy


def _codec_predict(ref: np.ndarray, mvx_b: np.ndarray, mvy_b: np.ndarray) -> np.ndarray:
    """Encoder-side LR motion-compensated prediction of the synthetic codec
    (two-pass bilinear at 1/8 pel, edge-replicated borders, libvpx-style
    rounding), computed block by block on 9x9 windows of an edge-padded ref."""
    C, H, W = ref.shape
    bh, bw = mvx_b.shape
    ix = np.floor_divide(mvx_b, 8).astype(np.int64); fx = (mvx_b - 8 * ix).astype(np.int32)
    iy = np.floor_divide(mvy_b, 8).astype(np.int64); fy = (mvy_b - 8 * iy).astype(np.int32)
    m = int(max(np.abs(ix).max(initial=0), np.abs(iy).max(initial=0))) + 2
    pad = np.pad(ref, ((0, 0), (m, m), (m, m)), mode="edge").astype(np.int32)
    win = np.lib.stride_tricks.sliding_window_view(pad, (9, 9), axis=(1, 2))  # [C][Y][X][9][9]
    oy = (np.arange(bh) * 8)[:, None] + iy + m
    ox = (np.arange(bw) * 8)[None, :] + ix + m
    wv = win[:, oy, ox]                                   # [C][bh][bw][9][9]
    fx_ = fx[None, :, :, None, None]; fy_ = fy[None, :, :, None, None]
    hrow = (wv[..., :, :8] * (8 - fx_) + wv[..., :, 1:] * fx_ + 4) >> 3   # [C][bh][bw][9][8]
    out = (hrow[..., :8, :] * (8 - fy_) + hrow[..., 1:, :] * fy_ + 4) >> 3  # [C][bh][bw][8][8]
    return out.transpose(0, 1, 3, 2, 4).reshape(C, H, W).astype(np.int64)


def _quant(d: np.ndarray, q: int) -> np.ndarray:
    return np.clip(np.round(d / q) * q, -255, 255).astype(np.int16)


def _box_down(img: np.ndarray, s: int) -> np.ndarray:
    C, H, W = img.shape
    return img.reshape(C, H // s, s, W // s, s).mean(axis=(2, 4))


def make_chunk(seed: int, w: int, h: int, scale: int, n: int, *, types=None,
               altref_every: int | None = 16, profile: int | None = None,
               intra_frac: float = 0.02, golden_frac: float = 0.15,
               jitter: float = 0.3, with_gt: bool = False, interp: int = INTERP_BILINEAR) -> Chunk:
    """Generate one stream's chunk.  Seeds follow SURVEY.md §8(d):
    seed = stream_id + 1000 * config.  interp: the codec's sub-pel filter
    (INTERP_*); the default stream is bilinear and draws no extra randoms."""
    assert w % 8 == 0 and h % 8 == 0 and n >= 1
    rng = np.random.default_rng(seed)
    prof = PROFILES[(seed % len(PROFILES)) if profile is None else profile]
    if types is None:
        types = default_types(n, altref_every)
    types = np.asarray(types, np.uint8)
    assert types.shape == (n,)
    scene = _Scene(rng, w, h, n, prof, scale)
    bh, bw = h // 8, w // 8
    lr = np.empty((n, 3, h, w), np.uint8)
    res = np.empty((n, 3, h, w), np.int16)
    mv = np.zeros((n, bh, bw), MV_DTYPE)
    gt = np.empty((n, 3, h * scale, w * scale), np.uint8) if with_gt else None
    golden = -1
    for f in range(n):
        if with_gt:
            g = np.clip(np.round(scene.render(f, scale)), 0, 255)
            gt[f] = g.astype(np.uint8)
            target = _box_down(g, scale)
        else:
            target = scene.render(f, 1)
        target = np.clip(np.round(target), 0, 255)
        if types[f] == NS_KEY:
            q = 2
            rq = _quant(target - 128.0, q)
            lr[f] = np.clip(128 + rq.astype(np.int32), 0, 255)
            res[f] = rq
            mv[f]["ref"] = NS_REF_INTRA
        else:
            q = 2 if types[f] == NS_ALTREF else 4
            u = rng.random((bh, bw))
            ref = np.where(u < intra_frac, NS_REF_INTRA,
                           np.where(u < intra_frac + golden_frac, NS_REF_GOLDEN, NS_REF_LAST)).astype(np.uint8)
            if golden < 0 or f == 0:
                ref[ref == NS_REF_GOLDEN] = NS_REF_LAST
            if f == 0:
                # chunk without a leading KEY: the synthetic codec predicts
                # from a mid-grey previous frame
                ref[:] = NS_REF_INTRA
            mvx_l, mvy_l = scene.block_motion(f, f - 1, bh, bw)
            mvx_g, mvy_g = scene.block_motion(f, max(golden, 0), bh, bw)
            mvx = np.where(ref == NS_REF_GOLDEN, mvx_g, mvx_l)
            mvy = np.where(ref == NS_REF_GOLDEN, mvy_g, mvy_l)
            jm = rng.random((bh, bw)) < jitter
            mvx = mvx + jm * rng.integers(-1, 2, (bh, bw))
            jm = rng.random((bh, bw)) < jitter
            mvy = mvy + jm * rng.integers(-1, 2, (bh, bw))
            mvx = np.clip(mvx, -32768, 32767)
            mvy = np.clip(mvy, -32768, 32767)
            mvx[ref == NS_REF_INTRA] = 0
            mvy[ref == NS_REF_INTRA] = 0
            if interp:
                kb = _block_kernels(rng, interp, bh, bw)
                mv[f]["filter"] = kb if interp == INTERP_SWITCHABLE else 0

                def predict(r_):
                    return _codec_predict8(r_, mvx, mvy, kb, 8, 2)
            else:
                predict = lambda r_: _codec_predict(r_, mvx, mvy)  # noqa: E731
            pred_l = predict(lr[f - 1]) if f > 0 else np.full((3, h, w), 128, np.int64)
            pred_g = predict(lr[golden]) if golden >= 0 and (ref == NS_REF_GOLDEN).any() else pred_l
            refpx = np.repeat(np.repeat(ref, 8, 0), 8, 1)[None]
            pred = np.where(refpx == NS_REF_GOLDEN, pred_g, pred_l)
            pred = np.where(refpx == NS_REF_INTRA, 128, pred)
            rq = _quant(target - pred, q)
            lr[f] = np.clip(pred + rq.astype(np.int64), 0, 255)
            res[f] = rq
            mv[f]["mvx"] = mvx
            mv[f]["mvy"] = mvy
            mv[f]["ref"] = ref
        if types[f] in (NS_KEY, NS_ALTREF):
            golden = f
    # encoded-size proxy: ~bytes to code the quantised residual; >= 1
    nz = np.abs(res.reshape(n, -1).astype(np.int64))
    res_size = (1 + (np.log2(1 + nz).sum(axis=1) / 8.0)).astype(np.uint32)
    return Chunk(w=w, h=h, scale=scale, lr=lr, res=res, mv=mv, type=types,
                 res_size=res_size, gt=gt, interp=interp)


def _codec_predict16(ref: np.ndarray, mvx_b: np.ndarray, mvy_b: np.ndarray) -> np.ndarray:
    """Encoder-side 4:2:0 chroma prediction of the synthetic codec: the block's
    luma vector read in 1/16 chroma pel (VP9's 4:2:0 rule), two-pass bilinear
    with 16 phases on the 4x4 chroma block, edge-replicated borders."""
    C, H, W = ref.shape
    bh, bw = mvx_b.shape
    ix = np.floor_divide(mvx_b, 16).astype(np.int64); fx = (mvx_b - 16 * ix).astype(np.int32)
    iy = np.floor_divide(mvy_b, 16).astype(np.int64); fy = (mvy_b - 16 * iy).astype(np.int32)
    m = int(max(np.abs(ix).max(initial=0), np.abs(iy).max(initial=0))) + 2
    pad = np.pad(ref, ((0, 0), (m, m), (m, m)), mode="edge").astype(np.int32)
    win = np.lib.stride_tricks.sliding_window_view(pad, (5, 5), axis=(1, 2))
    oy = (np.arange(bh) * 4)[:, None] + iy + m
    ox = (np.arange(bw) * 4)[None, :] + ix + m
    wv = win[:, oy, ox]                                   # [C][bh][bw][5][5]
    fx_ = fx[None, :, :, None, None]; fy_ = fy[None, :, :, None, None]
    hrow = (wv[..., :, :4] * (16 - fx_) + wv[..., :, 1:] * fx_ + 8) >> 4
    out = (hrow[..., :4, :] * (16 - fy_) + hrow[..., 1:, :] * fy_ + 8) >> 4
    return out.transpose(0, 1, 3, 2, 4).reshape(C, H, W).astype(np.int64)


def _codec_predict8(ref: np.ndarray, mvx_b: np.ndarray, mvy_b: np.ndarray, kern_b: np.ndarray, bs: int,
                    q4: int) -> np.ndarray:
    """Encoder-side 8-tap prediction of the synthetic codec (libvpx convolve8
    semantics): the block's vector times q4 gives its offset in 1/16 pel (2 for
    luma vectors in 1/8 pel, 1 for a 4:2:0 chroma plane), taps at -3..+4 around
    the integer position, each pass rounded by 7 bits and clipped to a byte,
    edge-replicated borders; blocks of bs x bs pixels, kernel per block."""
    C, H, W = ref.shape
    bh, bw = mvx_b.shape
    ox16 = mvx_b.astype(np.int64) * q4
    oy16 = mvy_b.astype(np.int64) * q4
    ix, px = np.floor_divide(ox16, 16), np.mod(ox16, 16)
    iy, py = np.floor_divide(oy16, 16), np.mod(oy16, 16)
    m = int(max(np.abs(ix).max(initial=0), np.abs(iy).max(initial=0))) + 8
    pad = np.pad(ref, ((0, 0), (m, m), (m, m)), mode="edge").astype(np.int64)
    win = np.lib.stride_tricks.sliding_window_view(pad, (bs + 7, bs + 7), axis=(1, 2))
    oy = (np.arange(bh) * bs)[:, None] + iy - 3 + m
    ox = (np.arange(bw) * bs)[None, :] + ix - 3 + m
    wv = win[:, oy, ox]                                    # [C][bh][bw][bs+7][bs+7]
    fx = VP9_KERNELS[kern_b, px]                            # [bh][bw][8]
    fy = VP9_KERNELS[kern_b, py]
    taps = np.lib.stride_tricks.sliding_window_view(wv, 8, axis=4)   # [C][bh][bw][bs+7][bs][8]
    hrow = np.clip(((taps * fx[None, :, :, None, None, :]).sum(-1) + 64) >> 7, 0, 255)   # [C][bh][bw][bs+7][bs]
    vt = np.lib.stride_tricks.sliding_window_view(hrow, 8, axis=3)   # [C][bh][bw][bs][bs][8]
    out = np.clip(((vt * fy[None, :, :, None, None, :]).sum(-1) + 64) >> 7, 0, 255)
    return out.transpose(0, 1, 3, 2, 4).reshape(C, H, W).astype(np.int64)


def _block_kernels(rng, interp: int, bh: int, bw: int) -> np.ndarray:
    if interp == INTERP_SWITCHABLE:
        return rng.integers(0, 3, (bh, bw)).astype(np.uint8)
    return np.full((bh, bw), max(interp - 1, 0), np.uint8)


@dataclasses.dataclass
class ChunkI420:
    """One stream's chunk in YUV 4:2:0 (NEXT-2): per frame Y [h][w] then U, V
    [h/2][w/2], flattened; the rest as Chunk."""
    w: int
    h: int
    scale: int
    lr: np.ndarray        # u8  [n][h*w*3/2]
    res: np.ndarray       # i16 [n][h*w*3/2]
    mv: np.ndarray        # MV_DTYPE [n][h/8][w/8] (luma vectors, 1/8 LR luma pel)
    type: np.ndarray
    res_size: np.ndarray
    gt: np.ndarray | None = None   # u8 [n][s*h*s*w*3/2]
    fmt: str = "i420"
    interp: int = INTERP_BILINEAR

    @property
    def n(self) -> int:
        return int(self.type.shape[0])


def to_i420(planes: np.ndarray) -> np.ndarray:
    """[3][H][W] -> flat Y | U | V with chroma = rounded 2x2 box average (input
    conversion of the synthetic source only)."""
    y = planes[0].astype(np.int64)
    c = planes[1:].astype(np.int64)
    cs = (c[:, 0::2, 0::2] + c[:, 1::2, 0::2] + c[:, 0::2, 1::2] + c[:, 1::2, 1::2] + 2) >> 2
    return np.concatenate([y.ravel(), cs.reshape(-1)])


def make_chunk_i420(seed: int, w: int, h: int, scale: int, n: int, *, types=None, altref_every: int | None = 16,
                    profile: int | None = None, intra_frac: float = 0.02, golden_frac: float = 0.15,
                    jitter: float = 0.3, with_gt: bool = False, interp: int = INTERP_BILINEAR) -> ChunkI420:
    """The synthetic codec loop of make_chunk in YUV 4:2:0: luma exactly as
    there, chroma planes at half resolution predicted with the block's luma
    vector read in 1/16 chroma pel (_codec_predict16)."""
    assert w % 8 == 0 and h % 8 == 0 and n >= 1
    rng = np.random.default_rng(seed)
    prof = PROFILES[(seed % len(PROFILES)) if profile is None else profile]
    if types is None:
        types = default_types(n, altref_every)
    types = np.asarray(types, np.uint8)
    scene = _Scene(rng, w, h, n, prof, scale)
    bh, bw = h // 8, w // 8
    P = h * w
    lr = np.empty((n, P * 3 // 2), np.uint8)
    res = np.empty((n, P * 3 // 2), np.int16)
    mv = np.zeros((n, bh, bw), MV_DTYPE)
    gt = np.empty((n, scale * scale * P * 3 // 2), np.uint8) if with_gt else None

    def planes(flat):
        y = flat[:P].reshape(1, h, w)
        c = flat[P:].reshape(2, h // 2, w // 2)
        return y, c

    golden = -1
    for f in range(n):
        if with_gt:
            g = np.clip(np.round(scene.render(f, scale)), 0, 255)
            gt[f] = to_i420(g)
            target = _box_down(g, scale)
        else:
            target = scene.render(f, 1)
        tflat = to_i420(np.clip(np.round(target), 0, 255)).astype(np.float64)
        if types[f] == NS_KEY:
            rq = _quant(tflat - 128.0, 2)
            lr[f] = np.clip(128 + rq.astype(np.int32), 0, 255)
            res[f] = rq
            mv[f]["ref"] = NS_REF_INTRA
        else:
            q = 2 if types[f] == NS_ALTREF else 4
            u = rng.random((bh, bw))
            ref = np.where(u < intra_frac, NS_REF_INTRA,
                           np.where(u < intra_frac + golden_frac, NS_REF_GOLDEN, NS_REF_LAST)).astype(np.uint8)
            if golden < 0 or f == 0:
                ref[ref == NS_REF_GOLDEN] = NS_REF_LAST
            if f == 0:
                ref[:] = NS_REF_INTRA
            mvx_l, mvy_l = scene.block_motion(f, f - 1, bh, bw)
            mvx_g, mvy_g = scene.block_motion(f, max(golden, 0), bh, bw)
            mvx = np.where(ref == NS_REF_GOLDEN, mvx_g, mvx_l)
            mvy = np.where(ref == NS_REF_GOLDEN, mvy_g, mvy_l)
            jm = rng.random((bh, bw)) < jitter
            mvx = mvx + jm * rng.integers(-1, 2, (bh, bw))
            jm = rng.random((bh, bw)) < jitter
            mvy = mvy + jm * rng.integers(-1, 2, (bh, bw))
            mvx = np.clip(mvx, -32768, 32767)
            mvy = np.clip(mvy, -32768, 32767)
            mvx[ref == NS_REF_INTRA] = 0
            mvy[ref == NS_REF_INTRA] = 0
            if interp:
                kb = _block_kernels(rng, interp, bh, bw)
                mv[f]["filter"] = kb if interp == INTERP_SWITCHABLE else 0
            pred = np.empty(P * 3 // 2, np.int64)
            refpx_y = np.repeat(np.repeat(ref, 8, 0), 8, 1)
            refpx_c = np.repeat(np.repeat(ref, 4, 0), 4, 1)
            for which, rp_ in ((NS_REF_LAST, f - 1), (NS_REF_GOLDEN, golden)):
                if rp_ < 0 or not (ref == which).any():
                    continue
                ry, rc = planes(lr[rp_])
                if interp:
                    py = _codec_predict8(ry, mvx, mvy, kb, 8, 2)[0]
                    pc = _codec_predict8(rc, mvx, mvy, kb, 4, 1)
                else:
                    py = _codec_predict(ry, mvx, mvy)[0]
                    pc = _codec_predict16(rc, mvx, mvy)
                cur = np.concatenate([py.ravel(), pc.reshape(-1)])
                sel = np.concatenate([(refpx_y == which).ravel(), np.tile((refpx_c == which).ravel(), 2)])
                pred[sel] = cur[sel]
            intra = np.concatenate([(refpx_y == NS_REF_INTRA).ravel(), np.tile((refpx_c == NS_REF_INTRA).ravel(), 2)])
            pred[intra] = 128
            rq = _quant(tflat - pred, q)
            lr[f] = np.clip(pred + rq.astype(np.int64), 0, 255)
            res[f] = rq
            mv[f]["mvx"] = mvx
            mv[f]["mvy"] = mvy
            mv[f]["ref"] = ref
        if types[f] in (NS_KEY, NS_ALTREF):
            golden = f
    nz = np.abs(res.astype(np.int64))
    res_size = (1 + (np.log2(1 + nz).sum(axis=1) / 8.0)).astype(np.uint32)
    return ChunkI420(w=w, h=h, scale=scale, lr=lr, res=res, mv=mv, type=types, res_size=res_size, gt=gt,
                     interp=interp)


def _to_bf16_bits(x: np.ndarray) -> np.ndarray:
    """float32 -> bf16 bit pattern, round-to-nearest-even."""
    u = np.ascontiguousarray(x, np.float32).view(np.uint32).astype(np.uint64)
    u = u + 0x7FFF + ((u >> 16) & 1)
    return (u >> 16).astype(np.uint16)


def weight_shapes(n_blocks: int, n_ch: int, scale: int):
    """(name, cout, cin) in the documented blob order (include/ns.h):
    head, blocks x (conv1, conv2), end, up, tail; each [Cout][Cin][3][3] + bias[Cout]."""
    C = n_ch
    out = [("head", C, 3)]
    for b in range(n_blocks):
        out += [(f"b{b}.conv1", C, C), (f"b{b}.conv2", C, C)]
    out += [("end", C, C), ("up", scale * scale * C, C), ("tail", 3, C)]
    return out


def blob_len(n_blocks: int, n_ch: int, scale: int) -> int:
    return sum(co * ci * 9 + co for _, co, ci in weight_shapes(n_blocks, n_ch, scale))


# Multipliers on He-normal init (std = sqrt(2 / (9*Cin))), SURVEY.md §8(d):
# body x0.1 keeps the net unsaturated; the tail multiplier is fixed so that the
# output correction t has a std of a few LSB on this generator's content.
W_MULT = dict(head=0.5, body=0.1, end=0.1, up=0.1, tail=0.8)


def make_weights(seed: int, n_blocks: int, n_ch: int, scale: int, gain: float = 1.0) -> np.ndarray:
    """Seeded bf16 weight blob (uint16 bit patterns) of one content-aware DNN."""
    rng = np.random.default_rng(seed + 7_777_777)
    parts = []
    for name, co, ci in weight_shapes(n_blocks, n_ch, scale):
        kind = name.split(".")[0] if "." not in name else "body"
        he = np.sqrt(2.0 / (9 * ci))
        wt = rng.standard_normal((co, ci, 3, 3)).astype(np.float32) * np.float32(he * W_MULT[kind] * gain)
        b = rng.uniform(-0.01, 0.01, co).astype(np.float32) * np.float32(gain)
        parts += [wt.ravel(), b]
    return _to_bf16_bits(np.concatenate(parts))


def bf16_bits_to_f32(bits: np.ndarray) -> np.ndarray:
    return (np.asarray(bits, np.uint16).astype(np.uint32) << 16).view(np.float32)


# Configurations of BASELINE.json "configs".
CONFIGS = {
    1: dict(name="c1", w=128, h=72, scale=2, n=8, n_blocks=4, n_ch=16, k=2, altref_every=None),
    2: dict(name="c2", w=640, h=360, scale=3, n=60, n_blocks=8, n_ch=32, k=6, altref_every=16),
    3: dict(name="c3", w=1280, h=720, scale=3, n=60, n_blocks=8, n_ch=32, k=5, altref_every=16),
    4: dict(name="c4", w=1280, h=720, scale=3, n=60, n_blocks=8, n_ch=32, k=5, altref_every=16, streams=64),
    5: dict(name="c5", w=None, h=None, scale=3, n=60, n_blocks=8, n_ch=32, k=5, altref_every=16, streams=512),
}
