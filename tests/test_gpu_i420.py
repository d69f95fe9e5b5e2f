"""YUV 4:2:0 streams (NS_FMT_I420, readings R9 / R10)
through the C ABI against the 4:2:0 oracle (oracle.reconstruct_i420,
oracle.sr_forward_i420; pinned in tests/test_oracle_i420.py).

Bars as for 4:4:4: selection and reconstruction bit-exact (reconstruction given
identical SR anchor bytes), SR within max-abs 2/255 per pixel."""
import io

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ns = pytest.importorskip("paper_conf_sigcomm_yeolkjyh22_b200")

DEV = "cuda:0"
SR_MAX_ABS = 2


@pytest.fixture(scope="module")
def ctx():
    c = ns.Context(0, pool_bytes=8 << 30)
    yield c
    c.close()


def _dev(c, model=None, last=None, gold=None, gt=False):
    d = ns.DeviceChunk.from_numpy(c.lr, c.res, c.mv, c.type, c.w, c.h, c.scale, DEV, model=model,
                                  gt=c.gt if gt else None, format=ns.NS_FMT_I420)
    if last is not None:
        d.hr_last = torch.from_numpy(last).to(DEV)
        d.hr_golden = torch.from_numpy(gold).to(DEV)
    return d


def _hr_size(c):
    return c.scale * c.h * c.scale * c.w * 3 // 2


def _adversarial(c, seed):
    rng = np.random.default_rng(seed)
    n, bh, bw = c.n, c.h // 8, c.w // 8
    c.res[:] = rng.integers(-255, 256, c.res.shape, dtype=np.int16)
    kind = rng.integers(0, 3, (n, bh, bw))
    mv = np.where(kind[..., None] == 0, rng.integers(-64, 65, (n, bh, bw, 2)),
                  np.where(kind[..., None] == 1, rng.integers(-4000, 4001, (n, bh, bw, 2)),
                           rng.choice(np.array([-32768, 32767]), (n, bh, bw, 2))))
    c.mv["mvx"] = mv[..., 0].astype(np.int16)
    c.mv["mvy"] = mv[..., 1].astype(np.int16)
    c.mv["ref"] = rng.choice(np.array([0, 1, 2], np.uint8), (n, bh, bw), p=[0.5, 0.35, 0.15])
    return c


@pytest.mark.parametrize("s,w,h,adv", [(2, 64, 48, False), (3, 48, 32, False), (4, 32, 16, False),
                                       (3, 272, 48, True), (2, 80, 32, True), (4, 288, 16, True)])
def test_reconstruct_i420_bit_exact(ctx, s, w, h, adv):
    n = 9
    types = synth.default_types(n, 4)
    types[6] = synth.NS_KEY
    c = synth.make_chunk_i420(600 + s + w, w, h, s, n, types=types)
    if adv:
        c = _adversarial(c, w + h)
    rng = np.random.default_rng(s + w)
    ia = [1 if f in (2, 4) else 0 for f in range(n)]
    hra = np.zeros((n, _hr_size(c)), np.uint8)
    for f in range(n):
        if ia[f]:
            hra[f] = rng.integers(0, 256, hra.shape[1])
    last0 = rng.integers(0, 256, hra.shape[1]).astype(np.uint8)
    gold0 = rng.integers(0, 256, hra.shape[1]).astype(np.uint8)
    exp, elast, egold = oracle.reconstruct_i420(c, ia, hra, last0, gold0)
    dc = _dev(c, last=last0, gold=gold0)
    hr = [torch.from_numpy(hra[f]).to(DEV) for f in range(n)]
    ctx.reconstruct_chunk([dc], torch.tensor([ia], dtype=torch.uint8, device=DEV), [hr])
    torch.cuda.synchronize()
    for f in range(n):
        g = hr[f].cpu().numpy()
        assert np.array_equal(g, exp[f]), (f, int((g != exp[f]).sum()))
    assert np.array_equal(dc.hr_last.cpu().numpy(), elast)
    assert np.array_equal(dc.hr_golden.cpu().numpy(), egold)


@pytest.mark.parametrize("B,C,s,w,h", [(2, 16, 2, 64, 48), (1, 32, 3, 144, 32), (1, 16, 4, 32, 16),
                                       (1, 32, 3, 272, 256)])
def test_sr_i420_vs_oracle(ctx, B, C, s, w, h):
    """ns_sr_anchors on 4:2:0 frames: the net on (Y, up2 U, up2 V), HR chroma
    by the rounded 2x2 average (R10); 264 x 256 spans several res-block and
    upsampler strips and CTA x-seams."""
    m = ctx.model(B, C, s)
    blob = synth.make_weights(40 + B + C + s, B, C, s)
    m.set_weights(blob)
    c = synth.make_chunk_i420(41 + w, w, h, s, 2)
    lr = torch.from_numpy(c.lr).to(DEV)
    hr = torch.zeros((2, _hr_size(c)), dtype=torch.uint8, device=DEV)
    ctx.sr_anchors([(m, lr[i], hr[i], w, h, ns.NS_FMT_I420) for i in range(2)])
    torch.cuda.synchronize()
    got = hr.cpu().numpy()
    for i in range(2):
        exp = oracle.sr_forward_i420(c.lr[i], blob, B, C, s, h, w)
        d = np.abs(got[i].astype(int) - exp.astype(int))
        assert d.max() <= SR_MAX_ABS, (i, int(d.max()), np.argwhere(d > SR_MAX_ABS)[:4])


def test_enhance_i420_and_444_mixed(ctx):
    """One ns_enhance_streams call over 4:2:0 and 4:4:4 streams: SR groups are
    split by format, frame steps run the luma kernel for both and the chroma
    kernel for the 4:2:0 ones; every stream against its oracle."""
    n, k = 10, 3
    specs = [("i420", 64, 32, 2), ("444", 64, 32, 2), ("i420", 48, 32, 3), ("i420", 64, 32, 2)]
    dcs, hrs, refs = [], [], []
    rng = np.random.default_rng(9)
    for i, (fmt, w, h, s) in enumerate(specs):
        m = ctx.model(1, 16, s)
        blob = synth.make_weights(90 + i, 1, 16, s)
        m.set_weights(blob)
        types = synth.default_types(n, 4)
        if fmt == "i420":
            c = synth.make_chunk_i420(900 + i, w, h, s, n, types=types, with_gt=True)
            size = _hr_size(c)
            last = rng.integers(0, 256, size).astype(np.uint8)
            gold = rng.integers(0, 256, size).astype(np.uint8)
            dcs.append(_dev(c, model=m, last=last, gold=gold, gt=True))
            hrs.append([torch.zeros(size, dtype=torch.uint8, device=DEV) for _ in range(n)])
        else:
            c = synth.make_chunk(900 + i, w, h, s, n, types=types, with_gt=True)
            shp = (3, s * h, s * w)
            last = rng.integers(0, 256, shp).astype(np.uint8)
            gold = rng.integers(0, 256, shp).astype(np.uint8)
            d = ns.DeviceChunk.from_numpy(c.lr, c.res, c.mv, c.type, w, h, s, DEV, model=m, gt=c.gt)
            d.hr_last, d.hr_golden = torch.from_numpy(last).to(DEV), torch.from_numpy(gold).to(DEV)
            dcs.append(d)
            hrs.append([torch.zeros(shp, dtype=torch.uint8, device=DEV) for _ in range(n)])
        refs.append((fmt, c, blob, last, gold))
    ia = torch.zeros((len(specs), n), dtype=torch.uint8, device=DEV)
    stats = torch.zeros((len(specs), 8), dtype=torch.float64, device=DEV)
    ctx.enhance_streams(dcs, hrs, is_anchor_out=ia, stats=stats, k=k)
    torch.cuda.synchronize()
    ia = ia.cpu().numpy()
    st = stats.cpu().numpy()
    for si, (fmt, c, blob, last, gold) in enumerate(refs):
        sc = [int(v) for v in oracle.score(c.res.reshape(n, 3, 1, -1) if fmt == "i420" else c.res)]
        _, _, ea = oracle.select_topk(list(c.type), sc, k)
        assert list(ia[si]) == ea, si
        got = np.stack([t.cpu().numpy() for t in hrs[si]])
        if fmt == "i420":
            for f in range(n):
                if ea[f]:
                    e = oracle.sr_forward_i420(c.lr[f], blob, 1, 16, c.scale, c.h, c.w)
                    assert np.abs(got[f].astype(int) - e.astype(int)).max() <= SR_MAX_ABS, (si, f)
            exp, elast, egold = oracle.reconstruct_i420(c, ea, got, last, gold)
        else:
            exp, elast, egold = oracle.reconstruct(c, ea, got, last, gold)
        assert np.array_equal(got, exp), si
        assert np.array_equal(dcs[si].hr_last.cpu().numpy(), elast)
        assert np.array_equal(dcs[si].hr_golden.cpu().numpy(), egold)
        # stats: frames, anchors, total score, PSNR of exactly these bytes
        assert st[si, 0] == n and st[si, 1] == sum(ea) and st[si, 3] == float(sum(sc))
        d = got.astype(np.float64) - c.gt.reshape(got.shape).astype(np.float64)
        mse = float((d * d).mean())
        assert abs(st[si, 5] - (100.0 if mse == 0 else min(100.0, 10 * np.log10(255.0 ** 2 / mse)))) < 1e-6


def test_ring_i420_equals_full_table(ctx):
    n, R, k = 11, 3, 3
    c = synth.make_chunk_i420(977, 48, 32, 3, n, types=synth.default_types(n, 3))
    m = ctx.model(1, 16, 3)
    m.set_weights(synth.make_weights(977, 1, 16, 3))
    size = _hr_size(c)
    outs = []
    for ring in (0, R):
        rng = np.random.default_rng(3)
        last = rng.integers(0, 256, size).astype(np.uint8)
        dc = _dev(c, model=m, last=last, gold=last[::-1].copy())
        slots = [torch.full((size,), 7, dtype=torch.uint8, device=DEV) for _ in range(ring or n)]
        row = [slots[f % len(slots)] for f in range(n)]
        ctx.enhance_streams([dc], [row], k=k)
        torch.cuda.synchronize()
        outs.append(([t.cpu().numpy() for t in slots], dc.hr_last.cpu().numpy(), dc.hr_golden.cpu().numpy()))
    full, ring_ = outs
    for r in range(R):
        f_last = max(f for f in range(n) if f % R == r)
        assert np.array_equal(ring_[0][r], full[0][f_last]), r
    assert np.array_equal(ring_[1], full[1]) and np.array_equal(ring_[2], full[2])


def test_hybrid_encode_i420(ctx):
    """4:2:0 anchors go out as 4:2:0 JPEGs (nvjpegEncodeYUV); the decoded luma
    matches the HR luma plane."""
    Image = pytest.importorskip("PIL.Image")
    n, k = 20, 2
    c = synth.make_chunk_i420(978, 64, 48, 2, n, types=synth.default_types(n, 8))
    m = ctx.model(1, 16, 2)
    m.set_weights(synth.make_weights(978, 1, 16, 2))
    size = _hr_size(c)
    dc = _dev(c, model=m, last=np.zeros(size, np.uint8), gold=np.zeros(size, np.uint8))
    hr = [torch.zeros(size, dtype=torch.uint8, device=DEV) for _ in range(n)]
    ia = torch.zeros((1, n), dtype=torch.uint8, device=DEV)
    ctx.enhance_streams([dc], [hr], is_anchor_out=ia, k=k)
    torch.cuda.synchronize()
    pk = ctx.encode_anchors([dc], ia.cpu().numpy(), [hr])
    H, W = 2 * c.h, 2 * c.w
    for h_, payload in ns.parse_hybrid(pk[0]):
        if not h_.anchor:
            continue
        im = Image.open(io.BytesIO(payload))
        im.draft("YCbCr", im.size)
        y = np.asarray(im.convert("YCbCr"))[..., 0] if im.mode != "YCbCr" else np.asarray(im)[..., 0]
        ref = hr[h_.frame].cpu().numpy()[:H * W].reshape(H, W)
        d = y.astype(np.float64) - ref
        assert 10 * np.log10(255.0 ** 2 / max(float((d * d).mean()), 1e-9)) >= 30.0


def test_i420_shape_rejected(ctx):
    """4:2:0 frames need whole 8x8 chroma blocks: w, h multiples of 16."""
    c = synth.make_chunk_i420(990, 40, 16, 3, 4, types=synth.default_types(4, None))
    dc = _dev(c, last=np.zeros(_hr_size(c), np.uint8), gold=np.zeros(_hr_size(c), np.uint8))
    hr = [torch.zeros(_hr_size(c), dtype=torch.uint8, device=DEV) for _ in range(4)]
    with pytest.raises(ns.NsError) as ei:
        ctx.reconstruct_chunk([dc], torch.zeros((1, 4), dtype=torch.uint8, device=DEV), [hr])
    assert ei.value.status == ns.NS_EINVAL and "16" in str(ei.value)
