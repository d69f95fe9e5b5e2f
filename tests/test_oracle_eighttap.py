"""Pins of the oracle's 8-tap motion compensation (NEXT-2, reading R13 in
DESIGN.md §3; oracle/ns_oracle.c warp_px8, or_reconstruct(.., interp)).

Each pin checks the oracle against something other than itself:
  * the kernel tables: properties VP9's published kernels have (rows sum to
    128 = 2^FILTER_BITS, phase 0 is the identity, phase 16-p is phase p
    reversed), and agreement with the synthetic codec's separate transcription
    (synth.VP9_KERNELS, written as half tables + mirror);
  * s = 1: reconstruction is decoding -- the oracle must reproduce the
    synthetic codec's decoded LR frames (synth._codec_predict8, vectorised
    numpy, written separately) byte for byte, 4:4:4 and 4:2:0, every kernel
    and the per-block (switchable) mode;
  * integer motion: 8-tap at phase 0 and the bilinear of O7 are both exact
    translations, so the two reconstructions agree;
  * a uniform fractional motion reduces to scipy.ndimage.correlate1d with
    edge replication (mode="nearest") per pass;
  * a constant reference stays constant (unit DC gain), switchable blocks equal
    the per-kernel reconstructions block by block, invalid modes are rejected.
"""
import numpy as np
import pytest
from scipy import ndimage

import oracle
import synth


@pytest.mark.parametrize("kernel", [0, 1, 2])
def test_kernel_tables(kernel):
    F = oracle.filter8(kernel)
    assert F.shape == (16, 8)
    assert (F.sum(axis=1) == 128).all()
    assert list(F[0]) == [0, 0, 0, 128, 0, 0, 0, 0]
    for p in range(1, 16):
        assert list(F[16 - p]) == list(F[p][::-1]), p
    assert np.array_equal(F, synth.VP9_KERNELS[kernel])


@pytest.mark.parametrize("interp", [1, 2, 3, 4])
@pytest.mark.parametrize("types", [None, [0, 2, 2, 1, 2, 2, 0, 2, 1, 2]])
def test_s1_equals_codec_decode_444(interp, types):
    n = 10
    t = synth.default_types(n, 3) if types is None else np.array(types, np.uint8)
    c = synth.make_chunk(300 + interp, 48, 32, 1, n, types=t, interp=interp)
    assert (c.mv["ref"] == synth.NS_REF_GOLDEN).any()
    if interp == 4:
        assert len(np.unique(c.mv["filter"][1:])) == 3
    hr = np.zeros((n, 3, 32, 48), np.uint8)
    hr[0] = c.lr[0]
    out, _, _ = oracle.reconstruct(c, [1] + [0] * (n - 1), hr, s=1)
    assert np.array_equal(out, c.lr)


@pytest.mark.parametrize("interp", [1, 2, 3, 4])
def test_s1_equals_codec_decode_i420(interp):
    n = 8
    c = synth.make_chunk_i420(400 + interp, 48, 32, 1, n, types=np.array([0, 2, 2, 1, 2, 2, 2, 2], np.uint8),
                              interp=interp)
    grey = np.full(32 * 48 * 3 // 2, 128, np.uint8)
    out, _, _ = oracle.reconstruct_i420(c, [0] * n, np.zeros((n, grey.size), np.uint8), grey, grey, s=1)
    assert np.array_equal(out, c.lr)


def _two_frame(w, h, s, mvx, mvy, interp, seed=3):
    """Two NORMAL frames, zero residual, every block LAST with the given motion:
    frame 0 predicts from hr_last (frame 1 from frame 0)."""
    c = synth.make_chunk(seed, w, h, s, 2, types=np.array([2, 2], np.uint8))
    c.res[:] = 0
    c.mv["mvx"], c.mv["mvy"], c.mv["ref"] = mvx, mvy, synth.NS_REF_LAST
    c.interp = interp
    return c


@pytest.mark.parametrize("s", [2, 3, 4])
def test_integer_motion_equals_bilinear(s):
    w, h = 32, 24
    rng = np.random.default_rng(s)
    H, W = s * h, s * w
    last = rng.integers(0, 256, (3, H, W)).astype(np.uint8)
    for _ in range(4):
        # s * mv a multiple of 8: whole HR pixels, phase 0 in both filters
        step = 8 // np.gcd(8, s)
        mvx = step * rng.integers(-12, 13, (h // 8, w // 8))
        mvy = step * rng.integers(-12, 13, (h // 8, w // 8))
        outs = []
        for interp in (0, 1, 3):
            c = _two_frame(w, h, s, mvx, mvy, interp)
            outs.append(oracle.reconstruct(c, [0, 0], np.zeros((2, 3, H, W), np.uint8), last, last.copy())[0])
        assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], outs[2])


@pytest.mark.parametrize("kernel", [0, 1, 2])
def test_uniform_motion_is_scipy_correlate(kernel):
    """Every block moves by the same (mvx, mvy): each pass is a 1-D
    correlation with edge replication, ROUND_POWER_OF_TWO(., 7), clip."""
    s, w, h = 2, 32, 24
    H, W = s * h, s * w
    rng = np.random.default_rng(10 + kernel)
    last = rng.integers(0, 256, (3, H, W)).astype(np.uint8)
    F = synth.VP9_KERNELS[kernel]
    for mvx, mvy in ((3, -5), (-7, 2), (1, 1), (-11, 9)):
        c = _two_frame(w, h, s, mvx, mvy, kernel + 1)
        out = oracle.reconstruct(c, [0, 0], np.zeros((2, 3, H, W), np.uint8), last, last.copy())[0][0]
        qx, qy = 2 * s * mvx, 2 * s * mvy              # 1/16 HR pel
        dx, px = qx // 16, qx % 16
        dy, py = qy // 16, qy % 16
        # correlate1d: out[i] = sum_j w[j] in[i + j - 4 - origin]; taps at i + d - 3 + j
        hp = ndimage.correlate1d(last.astype(np.int64), F[px], axis=2, mode="nearest", origin=-1 - dx)
        hp = np.clip((hp + 64) >> 7, 0, 255)
        vp = ndimage.correlate1d(hp, F[py], axis=1, mode="nearest", origin=-1 - dy)
        exp = np.clip((vp + 64) >> 7, 0, 255).astype(np.uint8)
        assert np.array_equal(out, exp), (mvx, mvy)


def test_constant_reference_stays_constant():
    s, w, h = 3, 24, 16
    H, W = s * h, s * w
    last = np.empty((3, H, W), np.uint8)
    last[0], last[1], last[2] = 0, 255, 77
    rng = np.random.default_rng(4)
    for interp in (1, 2, 3):
        c = _two_frame(w, h, s, rng.integers(-300, 300, (h // 8, w // 8)), rng.integers(-300, 300, (h // 8, w // 8)),
                       interp)
        out = oracle.reconstruct(c, [0, 0], np.zeros((2, 3, H, W), np.uint8), last, last.copy())[0]
        assert np.array_equal(out[0], last) and np.array_equal(out[1], last)


def test_switchable_is_per_block_kernel():
    s, w, h = 2, 40, 32
    H, W = s * h, s * w
    rng = np.random.default_rng(8)
    last = rng.integers(0, 256, (3, H, W)).astype(np.uint8)
    mvx = rng.integers(-40, 41, (h // 8, w // 8))
    mvy = rng.integers(-40, 41, (h // 8, w // 8))
    kb = rng.integers(0, 3, (h // 8, w // 8)).astype(np.uint8)
    c = _two_frame(w, h, s, mvx, mvy, 4)
    c.mv["filter"] = kb
    got = oracle.reconstruct(c, [0, 0], np.zeros((2, 3, H, W), np.uint8), last, last.copy())[0][0]
    per = [oracle.reconstruct(_two_frame(w, h, s, mvx, mvy, k + 1), [0, 0], np.zeros((2, 3, H, W), np.uint8),
                              last, last.copy())[0][0] for k in range(3)]
    B = 8 * s
    for by in range(h // 8):
        for bx in range(w // 8):
            sl = (slice(None), slice(by * B, by * B + B), slice(bx * B, bx * B + B))
            assert np.array_equal(got[sl], per[kb[by, bx]][sl])


def test_invalid_interp_rejected_and_filter_byte_range():
    c = _two_frame(16, 16, 2, 0, 0, 5)
    with pytest.raises(RuntimeError):
        oracle.reconstruct(c, [0, 0], np.zeros((2, 3, 32, 32), np.uint8), np.zeros((3, 32, 32), np.uint8))
    # a switchable block's filter byte above 2 reads as EIGHTTAP (include/ns.h)
    rng = np.random.default_rng(2)
    last = rng.integers(0, 256, (3, 32, 32)).astype(np.uint8)
    c = _two_frame(16, 16, 2, 3, 1, 4)
    c.mv["filter"] = 7
    a = oracle.reconstruct(c, [0, 0], np.zeros((2, 3, 32, 32), np.uint8), last, last.copy())[0]
    b = oracle.reconstruct(_two_frame(16, 16, 2, 3, 1, 1), [0, 0], np.zeros((2, 3, 32, 32), np.uint8), last,
                           last.copy())[0]
    assert np.array_equal(a, b)
