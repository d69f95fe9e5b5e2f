"""Pins of the YUV 4:2:0 oracle (NEXT-2; oracle/ns_oracle.c or_reconstruct_i420,
oracle.sr_forward_i420; readings R9, R10 in DESIGN.md §3).  Each pin checks the
oracle against something other than itself: the synthetic codec's own decoder
(written separately, numpy), the 4:4:4 oracle on the luma plane, closed forms
(identity, exact integer translation) and fp64 bilinear sampling."""
import numpy as np
import pytest

import oracle
import synth


def _planes(flat, h, w):
    return oracle.i420_planes(flat, h, w)


@pytest.mark.parametrize("seed,w,h,n,types", [
    (5, 32, 24, 6, None),
    (11, 48, 32, 10, [0, 2, 2, 1, 2, 2, 2, 1, 2, 2]),       # ALTREFs: GOLDEN references in chroma
    (17, 64, 16, 8, [0, 2, 2, 2, 0, 2, 1, 2]),               # a KEY inside the chunk
])
def test_s1_equals_codec_decode(seed, w, h, n, types):
    """At s = 1 reconstruction IS decoding: the oracle must reproduce the
    synthetic 4:2:0 codec's decoded LR frames byte for byte.  This pins the
    chroma MV derivation (luma vector in 1/16 chroma pel), the 16-phase
    bilinear, LAST / GOLDEN / INTRA / KEY handling and the rounding."""
    t = synth.default_types(n, 3) if types is None else np.array(types, np.uint8)
    c = synth.make_chunk_i420(seed, w, h, 1, n, types=t)
    assert (c.mv["ref"] == synth.NS_REF_GOLDEN).any() or types is None
    grey = np.full(h * w * 3 // 2, 128, np.uint8)
    hr = np.zeros((n, h * w * 3 // 2), np.uint8)
    out, _, _ = oracle.reconstruct_i420(c, [0] * n, hr, grey, grey, s=1)
    assert np.array_equal(out, c.lr)


@pytest.mark.parametrize("s", [2, 3, 4])
def test_luma_plane_is_the_444_oracle(s):
    """The luma plane of a 4:2:0 chunk follows O7/O6/O8 exactly as the 4:4:4
    oracle's plane 0 does (same vectors, references, types, anchors)."""
    n, w, h = 7, 40, 24
    c = synth.make_chunk_i420(31 + s, w, h, s, n, types=synth.default_types(n, 3))
    P = h * w
    c444 = synth.Chunk(w=w, h=h, scale=s, lr=np.zeros((n, 3, h, w), np.uint8), res=np.zeros((n, 3, h, w), np.int16),
                       mv=c.mv.copy(), type=c.type.copy(), res_size=c.res_size.copy())
    c444.lr[:, 0] = c.lr[:, :P].reshape(n, h, w)
    c444.res[:, 0] = c.res[:, :P].reshape(n, h, w)
    rng = np.random.default_rng(s)
    ia = [1, 0, 0, 1, 0, 0, 0]
    H, W = s * h, s * w
    a420 = rng.integers(0, 256, (n, H * W * 3 // 2)).astype(np.uint8)
    a444 = np.zeros((n, 3, H, W), np.uint8)
    a444[:, 0] = a420[:, :H * W].reshape(n, H, W)
    last = rng.integers(0, 256, H * W * 3 // 2).astype(np.uint8)
    l444 = np.zeros((3, H, W), np.uint8)
    l444[0] = last[:H * W].reshape(H, W)
    o420, _, _ = oracle.reconstruct_i420(c, ia, a420, last, last.copy())
    o444, _, _ = oracle.reconstruct(c444, ia, a444, l444, l444.copy())
    assert np.array_equal(o420[:, :H * W].reshape(n, H, W), o444[:, 0])


def _one_block_chunk(w, h, s, mvx, mvy, ref=synth.NS_REF_LAST):
    c = synth.make_chunk_i420(3, w, h, s, 2, types=np.array([2, 2], np.uint8))
    c.res[:] = 0
    c.mv["mvx"] = mvx
    c.mv["mvy"] = mvy
    c.mv["ref"] = ref
    return c


def test_zero_motion_zero_residual_is_identity():
    w, h, s = 32, 16, 3
    c = _one_block_chunk(w, h, s, 0, 0)
    rng = np.random.default_rng(1)
    last = rng.integers(0, 256, s * s * h * w * 3 // 2).astype(np.uint8)
    out, elast, _ = oracle.reconstruct_i420(c, [0, 0], np.zeros((2, last.size), np.uint8), last, last.copy())
    assert np.array_equal(out[0], last) and np.array_equal(out[1], last) and np.array_equal(elast, last)


@pytest.mark.parametrize("mv", [(16, 0), (-32, 48), (16 * 5, -16 * 3)])
def test_integer_chroma_shift_is_exact_translation(mv):
    """s * mv a multiple of 16 (s = 2: mv multiple of 8) moves the chroma planes
    by whole HR chroma pixels: an edge-padded translation, exactly (and luma by
    whole HR luma pixels: s * mv / 8)."""
    w, h, s = 32, 16, 2
    mvx, mvy = mv[0] // s, mv[1] // s
    c = _one_block_chunk(w, h, s, mvx, mvy)
    H, W = s * h, s * w
    rng = np.random.default_rng(2)
    last = rng.integers(0, 256, H * W * 3 // 2).astype(np.uint8)
    out, _, _ = oracle.reconstruct_i420(c, [0, 0], np.zeros((2, last.size), np.uint8), last, last.copy())
    Y, U, V = _planes(last, H, W)
    oY, oU, oV = _planes(out[0], H, W)
    dx, dy = s * mvx // 16, s * mvy // 16

    def shifted(p, ddx, ddy):
        m = 64
        pad = np.pad(p, m, mode="edge")
        return pad[m + ddy:m + ddy + p.shape[0], m + ddx:m + ddx + p.shape[1]]
    assert np.array_equal(oU, shifted(U, dx, dy)) and np.array_equal(oV, shifted(V, dx, dy))
    assert np.array_equal(oY, shifted(Y, 2 * dx, 2 * dy))


def test_fractional_chroma_within_one_of_fp64_bilinear():
    w, h, s = 48, 32, 3
    rng = np.random.default_rng(4)
    for _ in range(5):
        mvx, mvy = (int(v) for v in rng.integers(-40, 41, 2))
        c = _one_block_chunk(w, h, s, mvx, mvy)
        H, W = s * h, s * w
        last = rng.integers(0, 256, H * W * 3 // 2).astype(np.uint8)
        out, _, _ = oracle.reconstruct_i420(c, [0, 0], np.zeros((2, last.size), np.uint8), last, last.copy())
        _, U, _ = _planes(last, H, W)
        _, oU, _ = _planes(out[0], H, W)
        ch, cw = U.shape
        yy = np.clip(np.arange(ch)[:, None] + s * mvy / 16.0, 0, ch - 1)
        xx = np.clip(np.arange(cw)[None, :] + s * mvx / 16.0, 0, cw - 1)
        y0 = np.floor(yy).astype(int); x0 = np.floor(xx).astype(int)
        y1 = np.minimum(y0 + 1, ch - 1); x1 = np.minimum(x0 + 1, cw - 1)
        fy, fx = yy - y0, xx - x0
        Uf = U.astype(np.float64)
        ref = (Uf[y0, x0] * (1 - fx) + Uf[y0, x1] * fx) * (1 - fy) + (Uf[y1, x0] * (1 - fx) + Uf[y1, x1] * fx) * fy
        assert np.abs(oU.astype(np.float64) - ref).max() <= 1.0


def test_sr_i420_constant_frame_with_zero_tail():
    """With the HR tail at zero the net adds nothing (O5: out = up_s(LR) + t),
    so a constant-colour 4:2:0 anchor must stay exactly constant per plane
    through the chroma upsample, the net and the 2x2 chroma average."""
    B, C, s, h, w = 1, 16, 2, 16, 24
    blob = synth.make_weights(8, B, C, s).copy()
    tail = 3 * C * 9 + 3
    blob[-tail:] = 0
    lr = np.concatenate([np.full(h * w, 77), np.full(h * w // 4, 140), np.full(h * w // 4, 9)]).astype(np.uint8)
    out = oracle.sr_forward_i420(lr, blob, B, C, s, h, w)
    Y, U, V = _planes(out, s * h, s * w)
    assert (Y == 77).all() and (U == 140).all() and (V == 9).all()
