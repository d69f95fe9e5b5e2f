"""GPU parity at full size and at every seam the kernels introduce.

The SR kernels split a frame into CTA strips and x-tiles:
  * fused res-block: strips of NS_RB_ROWS = 240 LR rows, two 126-px tiles per
    CTA (CTA x-seams every 252 px);
  * rotated convs (head, end) and the composed upsampler+tail: strips of 180
    rows, 128-px tiles (uptail2: two per CTA, seams every 256 px);
  * the exact frame-border fix-up on the HR border ring.
An interior strip start (rows y0-2, y0-1 are in-frame data, not padding) and a
CTA x-seam are where ordering bugs live, so the oracle is evaluated on windows
that straddle every one of them at c3 size, on whole frames at c2 size, and on
one whole c3 frame.  Reconstruction is checked bit-exactly on adversarial
inputs: residuals spanning [-255, 255], MVs at the int16 extremes and far out of
frame, every reference kind, ragged widths and heights (partial CTAs).

Bars (BASELINE.json north_star): SR max-abs <= 2/255 per pixel and mean PSNR
difference <= 0.05 dB; reconstruction bit-exact given identical SR bytes.
"""
import numpy as np
import pytest

import oracle
import synth
from helpers import alloc_hr, dev_chunk, oracle_sr_crops, psnr

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ns = pytest.importorskip("paper_conf_sigcomm_yeolkjyh22_b200")

DEV = "cuda:0"
SR_MAX_ABS = 2
SR_PSNR_DB = 0.05

# strip starts / tile seams of the SR kernels (csrc/k_sr.cu: kRbRows, kRotRows,
# kTile, kRbOut): the windows below are centred on them
RB_ROWS, ROT_ROWS, TILE, RB_OUT = 240, 180, 128, 126


@pytest.fixture(scope="module")
def ctx():
    c = ns.Context(0, pool_bytes=16 << 30)
    yield c
    c.close()


def _model(ctx, B, C, s, seed):
    m = ctx.model(B, C, s)
    blob = synth.make_weights(seed, B, C, s)
    m.set_weights(blob)
    return m, blob


def _seam_windows(w, h, hh=16, ww=24):
    """LR windows (y0, x0, hh, ww) centred on every strip start and CTA x-seam
    of the SR kernels inside a w x h frame (plus the frame corners)."""
    ys = sorted({y for y in range(RB_ROWS, h, RB_ROWS)} | {y for y in range(ROT_ROWS, h, ROT_ROWS)})
    xs = sorted({x for x in range(2 * RB_OUT, w, 2 * RB_OUT)} | {x for x in range(TILE, w, TILE)})
    # merge x seams closer than a window
    merged = []
    for x in xs:
        if merged and x - merged[-1] < ww // 2:
            merged[-1] = (merged[-1] + x) // 2
        else:
            merged.append(x)
    wins = []
    for y in ys:
        for x in merged:
            wins.append((min(max(y - hh // 2, 0), h - hh), min(max(x - ww // 2, 0), w - ww), hh, ww))
    wins += [(0, 0, hh, ww), (0, w - ww, hh, ww), (h - hh, 0, hh, ww), (h - hh, w - ww, hh, ww)]
    return wins


def test_seam_windows_cover_every_seam():
    """The window list itself: every res-block strip start (240, 480), every
    rotated-conv / uptail strip start (180, 360, 540) and every CTA x-seam of
    a 1280 x 720 frame lies strictly inside some window."""
    w, h = 1280, 720
    wins = _seam_windows(w, h)
    for y in (180, 240, 360, 480, 540):
        for x in (128, 252, 256, 504, 512, 756, 768, 1008, 1024, 1152, 1260):
            assert any(y0 < y < y0 + hh and x0 < x < x0 + ww for (y0, x0, hh, ww) in wins), (y, x)


@pytest.mark.slow
def test_c3_sr_seam_windows(ctx):
    """c3 (720p -> 4K, B8/C32, x3): two anchors through ns_sr_anchors in one
    batch; every strip start and x-seam window against the oracle."""
    cfg = synth.CONFIGS[3]
    B, C, s, w, h = cfg["n_blocks"], cfg["n_ch"], cfg["scale"], cfg["w"], cfg["h"]
    m, blob = _model(ctx, B, C, s, seed=3301)
    c = synth.make_chunk(3301, w, h, s, 2)
    lr = torch.from_numpy(c.lr).to(DEV)
    hr = torch.zeros((2, 3, s * h, s * w), dtype=torch.uint8, device=DEV)
    ctx.sr_anchors([(m, lr[i], hr[i]) for i in range(2)])
    torch.cuda.synchronize()
    got = hr.cpu().numpy()
    wins = _seam_windows(w, h)
    worst, n_px = 0, 0
    for i in range(2):
        for (Y0, X0, HH, WW), patch in oracle_sr_crops(c.lr[i], blob, B, C, s, wins):
            g = got[i][:, Y0:Y0 + HH, X0:X0 + WW]
            d = np.abs(g.astype(int) - patch.astype(int))
            worst = max(worst, int(d.max()))
            n_px += d.size
            assert d.max() <= SR_MAX_ABS, (i, (Y0 // s, X0 // s), int(d.max()))
    print(f"c3 seam windows: {len(wins)} per frame, {n_px} px, worst max-abs {worst}")


@pytest.mark.slow
def test_c2_whole_chunk_vs_oracle(ctx):
    """c2 (360p -> 1080p, B8/C32, x3, n = 60, k = 6) through ns_enhance_streams:
    every anchor's WHOLE SR frame against the oracle (max-abs <= 2), and the
    chunk's PSNR against ground truth within 0.05 dB of the oracle's own
    enhanced chunk (oracle SR anchors + oracle reconstruction)."""
    cfg = synth.CONFIGS[2]
    B, C, s, n, k, w, h = cfg["n_blocks"], cfg["n_ch"], cfg["scale"], cfg["n"], cfg["k"], cfg["w"], cfg["h"]
    c = synth.make_chunk(2201, w, h, s, n, types=synth.default_types(n, 16), with_gt=True)
    m, blob = _model(ctx, B, C, s, seed=2201)
    dc = dev_chunk(ns, c, DEV, model=m, state=True)
    hr = alloc_hr(n, c, DEV)
    ia = torch.zeros((1, n), dtype=torch.uint8, device=DEV)
    ctx.enhance_streams([dc], [hr], is_anchor_out=ia, k=k)
    torch.cuda.synchronize()
    ia = [int(v) for v in ia.cpu().numpy()[0]]
    sc = [int(v) for v in oracle.score(c.res)]
    assert ia == oracle.select_topk(list(c.type), sc, k)[2]
    got = np.stack([t.cpu().numpy() for t in hr])
    ora = np.zeros_like(got)
    worst = 0
    for f in range(n):
        if ia[f]:
            ora[f] = oracle.sr_forward(c.lr[f], blob, B, C, s)
            d = int(np.abs(got[f].astype(int) - ora[f].astype(int)).max())
            worst = max(worst, d)
            assert d <= SR_MAX_ABS, (f, d)
    ora, _, _ = oracle.reconstruct(c, ia, ora, np.zeros_like(got[0]), np.zeros_like(got[0]))
    p_gpu, p_ora = psnr(got, c.gt), psnr(ora, c.gt)
    print(f"c2 whole chunk: worst anchor max-abs {worst}, PSNR gpu {p_gpu:.4f} oracle {p_ora:.4f} dB")
    assert abs(p_gpu - p_ora) <= SR_PSNR_DB
    # and the reuse path is bit-exact given the GPU's own anchor bytes
    exp, _, _ = oracle.reconstruct(c, ia, got, np.zeros_like(got[0]), np.zeros_like(got[0]))
    assert np.array_equal(got, exp)


@pytest.mark.slow
def test_c3_whole_frame_vs_oracle(ctx):
    """One whole c3 anchor (1280 x 720 -> 3840 x 2160): every pixel against the
    oracle, every strip and seam included; PSNR vs ground truth within 0.05 dB."""
    cfg = synth.CONFIGS[3]
    B, C, s, w, h = cfg["n_blocks"], cfg["n_ch"], cfg["scale"], cfg["w"], cfg["h"]
    m, blob = _model(ctx, B, C, s, seed=3401)
    c = synth.make_chunk(3401, w, h, s, 1, with_gt=True)
    lr = torch.from_numpy(c.lr[0]).to(DEV)
    hr = torch.zeros((3, s * h, s * w), dtype=torch.uint8, device=DEV)
    ctx.sr_anchors([(m, lr, hr)])
    torch.cuda.synchronize()
    got = hr.cpu().numpy()
    exp = oracle.sr_forward(c.lr[0], blob, B, C, s)
    d = np.abs(got.astype(int) - exp.astype(int))
    print(f"c3 whole frame: max-abs {d.max()}, mean {d.mean():.5f}, "
          f"PSNR gpu {psnr(got, c.gt[0]):.4f} oracle {psnr(exp, c.gt[0]):.4f}")
    assert d.max() <= SR_MAX_ABS
    assert abs(psnr(got, c.gt[0]) - psnr(exp, c.gt[0])) <= SR_PSNR_DB


# ---------------------------------------------------------------- adversarial reconstruction
def _adversarial_chunk(seed, w, h, s, n):
    """A synth chunk whose metadata is then replaced by contract-range extremes:
    residuals uniform in [-255, 255] with whole +-255 blocks; MVs mixing small
    sub-pel motion, large displacements, far out of frame and the int16
    extremes; references LAST / GOLDEN / INTRA at random; KEY and ALTREF frames
    in the middle of the chunk."""
    types = np.full(n, synth.NS_NORMAL, np.uint8)
    types[0] = synth.NS_KEY
    types[n // 3] = synth.NS_ALTREF
    types[(2 * n) // 3] = synth.NS_KEY
    c = synth.make_chunk(seed, w, h, s, n, types=types)
    rng = np.random.default_rng(seed)
    c.res[:] = rng.integers(-255, 256, c.res.shape, dtype=np.int16)
    bh, bw = h // 8, w // 8
    for f in range(n):
        for _ in range(max(1, bh * bw // 6)):
            by, bx = rng.integers(0, bh), rng.integers(0, bw)
            c.res[f, :, 8 * by:8 * by + 8, 8 * bx:8 * bx + 8] = rng.choice([-255, 255])
    kind = rng.integers(0, 4, (n, bh, bw))
    small = rng.integers(-64, 65, (n, bh, bw, 2))
    large = rng.integers(-4000, 4001, (n, bh, bw, 2))
    ext = rng.choice(np.array([-32768, -32767, 32767, 32766], np.int64), (n, bh, bw, 2))
    mv = np.where(kind[..., None] == 0, small, np.where(kind[..., None] == 1, large, ext))
    mv = np.where(kind[..., None] == 3, rng.integers(-8, 9, (n, bh, bw, 2)), mv)
    c.mv["mvx"] = mv[..., 0].astype(np.int16)
    c.mv["mvy"] = mv[..., 1].astype(np.int16)
    c.mv["ref"] = rng.choice(np.array([synth.NS_REF_LAST, synth.NS_REF_GOLDEN, synth.NS_REF_INTRA], np.uint8),
                             (n, bh, bw), p=[0.5, 0.35, 0.15])
    return c


@pytest.mark.parametrize("s,w,h", [
    (2, 72, 40),     # 9 block columns: one partial CTA; 80 HR rows (not a multiple of 32)
    (3, 264, 48),    # 33 block columns: a second CTA with one valid column
    (3, 40, 16),     # tiny frame: every window clamps on both sides
    (4, 136, 24),    # x4, 17 block columns
    (2, 520, 8),     # one block row, 65 block columns
])
def test_reconstruct_adversarial(ctx, s, w, h):
    n = 9
    c = _adversarial_chunk(4000 + 31 * s + w + h, w, h, s, n)
    rng = np.random.default_rng(w * h + s)
    ia = [0] * n
    ia[1] = ia[n // 3] = 1          # a NORMAL anchor and the ALTREF as anchor
    hr_anchor = np.zeros((n, 3, s * h, s * w), np.uint8)
    for f in range(n):
        if ia[f]:
            hr_anchor[f] = rng.choice(np.array([0, 255, 1, 254, 128], np.uint8), hr_anchor[f].shape)
    last0 = rng.integers(0, 256, hr_anchor[0].shape).astype(np.uint8)
    gold0 = rng.choice(np.array([0, 255], np.uint8), hr_anchor[0].shape)
    exp, elast, egold = oracle.reconstruct(c, ia, hr_anchor, last0, gold0)
    dc = dev_chunk(ns, c, DEV)
    dc.hr_last = torch.from_numpy(last0).to(DEV)
    dc.hr_golden = torch.from_numpy(gold0).to(DEV)
    hr = [torch.from_numpy(hr_anchor[f]).to(DEV) for f in range(n)]
    ctx.reconstruct_chunk([dc], torch.tensor([ia], dtype=torch.uint8, device=DEV), [hr])
    torch.cuda.synchronize()
    for f in range(n):
        g = hr[f].cpu().numpy()
        assert np.array_equal(g, exp[f]), (f, int(np.abs(g.astype(int) - exp[f]).max()),
                                           int((g != exp[f]).sum()))
    assert np.array_equal(dc.hr_last.cpu().numpy(), elast)
    assert np.array_equal(dc.hr_golden.cpu().numpy(), egold)


def test_reconstruct_adversarial_multistream(ctx):
    """Several adversarial streams of different shapes and scales in ONE call
    (frame steps batched over streams, one launch per scale per step)."""
    shapes = [(2, 72, 40), (3, 264, 48), (3, 40, 16), (4, 136, 24), (2, 48, 16)]
    n = 7
    cs, dcs, hrs, exps = [], [], [], []
    ia_all = np.zeros((len(shapes), n), np.uint8)
    for i, (s, w, h) in enumerate(shapes):
        c = _adversarial_chunk(5000 + i, w, h, s, n)
        rng = np.random.default_rng(i)
        ia = [0] * n
        ia[int(rng.integers(1, n))] = 1
        ia_all[i] = ia
        hra = np.zeros((n, 3, s * h, s * w), np.uint8)
        for f in range(n):
            if ia[f]:
                hra[f] = rng.integers(0, 256, hra[f].shape)
        last0 = rng.integers(0, 256, hra[0].shape).astype(np.uint8)
        gold0 = rng.integers(0, 256, hra[0].shape).astype(np.uint8)
        exps.append(oracle.reconstruct(c, ia, hra, last0, gold0)[0])
        dc = dev_chunk(ns, c, DEV)
        dc.hr_last = torch.from_numpy(last0).to(DEV)
        dc.hr_golden = torch.from_numpy(gold0).to(DEV)
        dcs.append(dc)
        hrs.append([torch.from_numpy(hra[f]).to(DEV) for f in range(n)])
    ctx.reconstruct_chunk(dcs, torch.from_numpy(ia_all).to(DEV), hrs)
    torch.cuda.synchronize()
    for i in range(len(shapes)):
        for f in range(n):
            assert np.array_equal(hrs[i][f].cpu().numpy(), exps[i][f]), (i, f)
