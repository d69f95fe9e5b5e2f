"""Pins for the numeric oracle (oracle/ns_oracle.c) -- CPU only.

  conv3x3 / pixel shuffle : brute-force 7-loop Python on tiny tensors, and
                            torch.nn.functional (fp64, CPU) as an independent
                            library implementation;
  SR net (O5)             : an independent torch fp64 module with the same
                            weights (t within 1e-9), the zero-tail special case
                            (out == up_s(LR) exactly);
  upsample (O6)           : x2 == fp64 bilinear (align_corners=False) with the
                            same final rounding, exactly (dyadic Q7 weights);
                            x3 within +-1 (u8) / +-2 (i16); constants preserved;
  warp (O7)               : zero MV == copy; integer MV == np.pad(edge)+slice;
                            fractional MV within 1 of fp64 bilinear sampling;
  reconstruct (O8)        : zero MV + zero residual reproduces the reference
                            exactly (north-star invariant); at s = 1 it equals
                            the synthetic codec's own decoded LR byte for byte.
  score (O2)              : numpy |res| sum; the proxy replaces it when given.
"""
import numpy as np
import pytest
import torch
import torch.nn.functional as F

import oracle
import synth


def test_score():
    c = synth.make_chunk(11, 64, 48, 2, 5)
    s = oracle.score(c.res)
    assert list(s) == [int(np.abs(c.res[f].astype(np.int64)).sum()) for f in range(5)]
    assert list(oracle.score(c.res, c.res_size)) == [int(v) for v in c.res_size]


def _brute_conv(x, w, b):
    cin, h, wd = x.shape
    cout = w.shape[0]
    out = np.zeros((cout, h, wd))
    for co in range(cout):
        for y in range(h):
            for xx in range(wd):
                acc = b[co]
                for ci in range(cin):
                    for ky in range(3):
                        for kx in range(3):
                            yy, xs = y + ky - 1, xx + kx - 1
                            if 0 <= yy < h and 0 <= xs < wd:
                                acc += w[co, ci, ky, kx] * x[ci, yy, xs]
                out[co, y, xx] = acc
    return out


def test_conv3x3_brute_force_and_torch():
    rng = np.random.default_rng(0)
    x = rng.standard_normal((2, 5, 4))
    w = rng.standard_normal((3, 2, 3, 3))
    b = rng.standard_normal(3)
    got = oracle.conv3x3(x, w, b)
    assert np.allclose(got, _brute_conv(x, w, b), atol=1e-12)
    x = rng.standard_normal((7, 13, 17))
    w = rng.standard_normal((5, 7, 3, 3))
    b = rng.standard_normal(5)
    ref = F.conv2d(torch.from_numpy(x)[None], torch.from_numpy(w), torch.from_numpy(b), padding=1)[0].numpy()
    assert np.allclose(oracle.conv3x3(x, w, b), ref, atol=1e-10)
    # asymmetric kernel catches a transposed (convolution vs correlation) tap
    w = np.zeros((1, 1, 3, 3)); w[0, 0, 0, 2] = 1.0
    x = np.arange(20.0).reshape(1, 4, 5)
    out = oracle.conv3x3(x, w, None)
    assert out[0, 1, 1] == x[0, 0, 2]


def test_pixel_shuffle_torch():
    rng = np.random.default_rng(1)
    for s in (2, 3, 4):
        x = rng.standard_normal((2 * s * s, 3, 5))
        ref = F.pixel_shuffle(torch.from_numpy(x)[None], s)[0].numpy()
        assert np.array_equal(oracle.pixel_shuffle(x, s), ref)


def _torch_sr_t(lr, blob, B, C, s):
    """Independent fp64 torch implementation of O5 up to t (before the skip)."""
    wf = torch.from_numpy(synth.bf16_bits_to_f32(blob).astype(np.float64))
    pos = 0

    def take(co, ci):
        nonlocal pos
        n = co * ci * 9
        w = wf[pos:pos + n].reshape(co, ci, 3, 3)
        b = wf[pos + n:pos + n + co]
        pos += n + co
        return w, b

    x = torch.from_numpy(lr.astype(np.float64) - 128.0)[None]
    w, b = take(C, 3)
    h0 = F.conv2d(x, w, b, padding=1)
    h = h0
    for _ in range(B):
        w1, b1 = take(C, C)
        w2, b2 = take(C, C)
        h = h + F.conv2d(F.relu(F.conv2d(h, w1, b1, padding=1)), w2, b2, padding=1)
    w, b = take(C, C)
    h = h0 + F.conv2d(h, w, b, padding=1)
    w, b = take(s * s * C, C)
    u = F.pixel_shuffle(F.conv2d(h, w, b, padding=1), s)
    w, b = take(3, C)
    t = F.conv2d(u, w, b, padding=1)[0].numpy()
    assert pos == blob.size
    return t


@pytest.mark.parametrize("B,C,s,h,w", [(2, 16, 2, 16, 24), (1, 32, 3, 16, 16), (1, 8, 4, 8, 16)])
def test_sr_forward_matches_torch(B, C, s, h, w):
    c = synth.make_chunk(21, w, h, s, 1)
    blob = synth.make_weights(21, B, C, s, gain=2.0)
    out, t = oracle.sr_forward(c.lr[0], blob, B, C, s, want_t=True)
    t_ref = _torch_sr_t(c.lr[0], blob, B, C, s)
    assert np.allclose(t, t_ref, atol=1e-9, rtol=0)
    up = np.stack([oracle.upsample(c.lr[0, p], s) for p in range(3)])
    exp = np.clip(np.floor(up + t_ref + 0.5), 0, 255)
    near_half = np.abs((up + t_ref) - np.floor(up + t_ref) - 0.5) < 1e-7
    assert np.array_equal(out[~near_half], exp[~near_half])
    assert t.std() > 0.3          # the net is not degenerate on this content


def test_sr_zero_tail_is_bilinear():
    B, C, s = 2, 16, 2
    c = synth.make_chunk(22, 32, 16, s, 1)
    blob = synth.make_weights(22, B, C, s).copy()
    n_tail = 3 * C * 9 + 3
    blob[-n_tail:] = 0
    out = oracle.sr_forward(c.lr[0], blob, B, C, s)
    up = np.stack([oracle.upsample(c.lr[0, p], s) for p in range(3)])
    assert np.array_equal(out, up.astype(np.uint8))


def _torch_bilinear(plane, s):
    x = torch.from_numpy(plane.astype(np.float64))[None, None]
    return F.interpolate(x, scale_factor=s, mode="bilinear", align_corners=False)[0, 0].numpy()


def test_upsample_x2_exact():
    rng = np.random.default_rng(3)
    for dt, lo, hi in ((np.uint8, 0, 256), (np.int16, -255, 256)):
        p = rng.integers(lo, hi, (13, 19)).astype(dt)
        got = oracle.upsample(p, 2)
        ref = np.floor(_torch_bilinear(p, 2) + 0.5)
        assert np.array_equal(got, ref)


def test_upsample_weights_and_bounds():
    rng = np.random.default_rng(4)
    for s in (3, 4):
        for dt, lo, hi, tol in ((np.uint8, 0, 256, 1), (np.int16, -255, 256, 2)):
            p = rng.integers(lo, hi, (11, 17)).astype(dt)
            got = oracle.upsample(p, s)
            ref = np.floor(_torch_bilinear(p, s) + 0.5)
            assert np.abs(got - ref).max() <= tol
    for s in (2, 3, 4):
        for v in (0, 7, 255, -255):
            assert np.all(oracle.upsample(np.full((4, 8), v, np.int32), s) == v)


def test_upsample_s3_tap_weights():
    # a single 1 at LR x=2 in a long row: HR outputs near it are the Q7 taps
    p = np.zeros((1, 8), np.int32); p[0, 2] = 1 << 14
    r = oracle.upsample(p, 3)[0]
    # X = 6,7,8 sit at source positions 5/3-..: centre X = 3*2+1 = 7 -> exactly the pixel
    assert r[7] == 1 << 14
    # X = 6 -> u = 12+1-3 = 10, x0 = 1, rem = 4, w1 = 85: weight of x=2 is 85/128
    assert r[6] == (85 * (1 << 14) * 128 + 8192) // 16384
    # X = 8 -> u = 14, x0 = 2, rem = 2, w1 = 43: weight of x=2 is (128-43)/128
    assert r[8] == ((128 - 43) * (1 << 14) * 128 + 8192) // 16384


def _mv_field(h, w, mvx, mvy, ref=synth.NS_REF_LAST):
    mv = np.zeros((h // 8, w // 8), synth.MV_DTYPE)
    mv["mvx"], mv["mvy"], mv["ref"] = mvx, mvy, ref
    return mv


def test_warp_zero_and_integer():
    rng = np.random.default_rng(5)
    s, h, w = 3, 16, 24
    ref = rng.integers(0, 256, (s * h, s * w)).astype(np.uint8)
    assert np.array_equal(oracle.warp_plane(ref, _mv_field(h, w, 0, 0), s), ref)
    for mvx, mvy in ((8, 0), (-16, 8), (24, -40), (-8, -8)):
        got = oracle.warp_plane(ref, _mv_field(h, w, mvx, mvy), s)
        dx, dy = s * mvx // 8, s * mvy // 8
        m = 64
        pad = np.pad(ref, m, mode="edge")
        exp = pad[m + dy:m + dy + s * h, m + dx:m + dx + s * w]
        assert np.array_equal(got, exp)


def test_warp_fractional_close_to_bilinear():
    rng = np.random.default_rng(6)
    s, h, w = 2, 16, 16
    ref = rng.integers(0, 256, (s * h, s * w)).astype(np.uint8)
    mv = np.zeros((h // 8, w // 8), synth.MV_DTYPE)
    mv["mvx"] = rng.integers(-20, 21, mv.shape)
    mv["mvy"] = rng.integers(-20, 21, mv.shape)
    got = oracle.warp_plane(ref, mv, s).astype(np.float64)
    H, W = ref.shape
    Y, X = np.mgrid[0:H, 0:W]
    m_x = s * np.repeat(np.repeat(mv["mvx"], 8 * s, 0), 8 * s, 1) / 8.0
    m_y = s * np.repeat(np.repeat(mv["mvy"], 8 * s, 0), 8 * s, 1) / 8.0
    sx, sy = X + m_x, Y + m_y
    x0, y0 = np.floor(sx).astype(int), np.floor(sy).astype(int)
    fx, fy = sx - x0, sy - y0
    cl = lambda a, n: np.clip(a, 0, n - 1)
    r = ref.astype(np.float64)
    v = (r[cl(y0, H), cl(x0, W)] * (1 - fx) + r[cl(y0, H), cl(x0 + 1, W)] * fx) * (1 - fy) + \
        (r[cl(y0 + 1, H), cl(x0, W)] * (1 - fx) + r[cl(y0 + 1, H), cl(x0 + 1, W)] * fx) * fy
    assert np.abs(got - v).max() <= 1.0


def test_reconstruct_zero_motion_zero_residual_is_identity():
    s, h, w, n = 2, 16, 24, 6
    c = synth.make_chunk(31, w, h, s, n, types=synth.default_types(n, None))
    c.res[:] = 0
    c.mv["mvx"] = 0
    c.mv["mvy"] = 0
    c.mv["ref"][1:] = synth.NS_REF_LAST
    rng = np.random.default_rng(7)
    hr0 = rng.integers(0, 256, (3, s * h, s * w)).astype(np.uint8)
    hr = np.zeros((n, 3, s * h, s * w), np.uint8)
    hr[0] = hr0
    ia = [1] + [0] * (n - 1)
    out, last, gold = oracle.reconstruct(c, ia, hr, hr_last=np.zeros_like(hr0), hr_golden=np.zeros_like(hr0))
    for f in range(n):
        assert np.array_equal(out[f], hr0)
    assert np.array_equal(last, hr0) and np.array_equal(gold, hr0)


@pytest.mark.parametrize("seed,types", [(41, None), (42, [0, 2, 2, 1, 2, 2, 2, 2, 1, 2, 2, 2])])
def test_reconstruct_s1_equals_codec_decode(seed, types):
    """At s = 1 every anchor is its own LR frame and reconstruction must replay
    the synthetic codec's decoder exactly (independent numpy implementation,
    synth._codec_predict): LAST/GOLDEN/INTRA handling, block indexing, sub-pel
    rounding and clamping all pinned at once."""
    n = 12
    t = synth.default_types(n, 4) if types is None else np.array(types, np.uint8)
    c = synth.make_chunk(seed, 40, 32, 1, n, types=t)
    hr = np.zeros((n, 3, 32, 40), np.uint8)
    ia = [0] * n
    ia[0] = 1
    hr[0] = c.lr[0]
    out, _, _ = oracle.reconstruct(c, ia, hr, s=1)
    assert np.array_equal(out, c.lr)
    # with some anchors in the middle (SR := identity at s = 1)
    ia = [1 if f in (0, 5, 9) else 0 for f in range(n)]
    hr = np.zeros_like(hr)
    for f in (0, 5, 9):
        hr[f] = c.lr[f]
    out, _, _ = oracle.reconstruct(c, ia, hr, s=1)
    assert np.array_equal(out, c.lr)


def test_reconstruct_key_and_intra_use_upsampled_lr():
    s, h, w, n = 3, 16, 16, 3
    c = synth.make_chunk(51, w, h, s, n, types=np.array([0, 2, 0], np.uint8))
    c.mv["ref"][1] = synth.NS_REF_INTRA
    hr = np.zeros((n, 3, s * h, s * w), np.uint8)
    out, _, _ = oracle.reconstruct(c, [0, 0, 0], hr)
    for f in range(n):
        up = np.stack([oracle.upsample(c.lr[f, p], s) for p in range(3)])
        assert np.array_equal(out[f], up)
