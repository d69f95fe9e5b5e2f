"""GPU parity of the 8-tap motion compensation (NEXT-2, reading R13;
k_recon8 in csrc/k_recon.cu) against the oracle (warp_px8 in
oracle/ns_oracle.c): reconstruction bit-exact for every kernel and the
per-block switchable mode, 4:4:4 and 4:2:0, on the synthetic codec's streams and
on contract-range adversarial inputs (+-255 residuals, int16-extreme and
far-out-of-frame vectors, every reference kind, ragged CTAs), streams of
different filters, formats and scales in one call, and the whole path."""
import numpy as np
import pytest

import oracle
import synth
from helpers import alloc_hr, dev_chunk
from test_gpu_parity_full import _adversarial_chunk

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ns = pytest.importorskip("paper_conf_sigcomm_yeolkjyh22_b200")

DEV = "cuda:0"


@pytest.fixture(scope="module")
def ctx():
    c = ns.Context(0, pool_bytes=8 << 30)
    yield c
    c.close()


def _i420_dev(c, last, gold):
    d = ns.DeviceChunk.from_numpy(c.lr, c.res, c.mv, c.type, c.w, c.h, c.scale, DEV, format=ns.NS_FMT_I420,
                                  interp=c.interp)
    d.hr_last = torch.from_numpy(last).to(DEV)
    d.hr_golden = torch.from_numpy(gold).to(DEV)
    return d


def _case(c, ia, seed, i420=False):
    """(device chunk, HR table, expected HR frames, expected state) for given anchors."""
    n, s = c.n, c.scale
    rng = np.random.default_rng(seed)
    shape = (s * c.h * s * c.w * 3 // 2,) if i420 else (3, s * c.h, s * c.w)
    hra = np.zeros((n,) + shape, np.uint8)
    for f in range(n):
        if ia[f]:
            hra[f] = rng.integers(0, 256, shape)
    last0 = rng.integers(0, 256, shape).astype(np.uint8)
    gold0 = rng.integers(0, 256, shape).astype(np.uint8)
    if i420:
        exp, elast, egold = oracle.reconstruct_i420(c, ia, hra, last0, gold0)
        dc = _i420_dev(c, last0, gold0)
    else:
        exp, elast, egold = oracle.reconstruct(c, ia, hra, last0, gold0)
        dc = dev_chunk(ns, c, DEV)
        dc.hr_last = torch.from_numpy(last0).to(DEV)
        dc.hr_golden = torch.from_numpy(gold0).to(DEV)
    hr = [torch.from_numpy(hra[f]).to(DEV) for f in range(n)]
    return dc, hr, exp, elast, egold


def _check(dc, hr, exp, elast, egold):
    for f in range(len(hr)):
        g = hr[f].cpu().numpy()
        assert np.array_equal(g, exp[f]), (f, int(np.abs(g.astype(int) - exp[f]).max()), int((g != exp[f]).sum()))
    assert np.array_equal(dc.hr_last.cpu().numpy(), elast)
    assert np.array_equal(dc.hr_golden.cpu().numpy(), egold)


@pytest.mark.parametrize("interp", [1, 2, 3, 4])
@pytest.mark.parametrize("s", [2, 3, 4])
def test_reconstruct_8tap_bit_exact(ctx, s, interp):
    n = 10
    c = synth.make_chunk(700 + 10 * s + interp, 64, 40, s, n, types=synth.default_types(n, 4), interp=interp)
    ia = [1 if f in (0, 5) else 0 for f in range(n)]
    dc, hr, *exp = _case(c, ia, s + interp)
    ctx.reconstruct_chunk([dc], torch.tensor([ia], dtype=torch.uint8, device=DEV), [hr])
    torch.cuda.synchronize()
    _check(dc, hr, *exp)


@pytest.mark.parametrize("interp", [1, 3, 4])
@pytest.mark.parametrize("s,w,h", [(2, 72, 40), (3, 264, 48), (3, 40, 16), (4, 136, 24), (2, 520, 8)])
def test_reconstruct_8tap_adversarial(ctx, s, w, h, interp):
    n = 8
    c = _adversarial_chunk(4100 + 31 * s + w + h + interp, w, h, s, n)
    c.interp = interp
    rng = np.random.default_rng(w + h + interp)
    c.mv["filter"] = rng.integers(0, 6, c.mv.shape)   # switchable: bytes above 2 read as EIGHTTAP
    ia = [0] * n
    ia[1] = ia[n // 3] = 1
    dc, hr, *exp = _case(c, ia, w * h + s)
    ctx.reconstruct_chunk([dc], torch.tensor([ia], dtype=torch.uint8, device=DEV), [hr])
    torch.cuda.synchronize()
    _check(dc, hr, *exp)


@pytest.mark.parametrize("interp", [1, 4])
@pytest.mark.parametrize("s,w,h,adv", [(2, 64, 48, False), (3, 48, 32, False), (4, 32, 16, False),
                                       (3, 272, 48, True), (4, 288, 16, True)])
def test_reconstruct_8tap_i420(ctx, s, w, h, adv, interp):
    from test_gpu_i420 import _adversarial
    n = 8
    types = synth.default_types(n, 3)
    types[5] = synth.NS_KEY
    c = synth.make_chunk_i420(650 + s + w + interp, w, h, s, n, types=types, interp=interp)
    if adv:
        c = _adversarial(c, w + h + interp)
        c.mv["filter"] = np.random.default_rng(w).integers(0, 4, c.mv.shape)
    ia = [1 if f in (2, 4) else 0 for f in range(n)]
    dc, hr, *exp = _case(c, ia, s + w, i420=True)
    ctx.reconstruct_chunk([dc], torch.tensor([ia], dtype=torch.uint8, device=DEV), [hr])
    torch.cuda.synchronize()
    _check(dc, hr, *exp)


def test_mixed_filters_formats_scales_one_call(ctx):
    """Bilinear and 8-tap streams, 4:4:4 and 4:2:0, three scales: one call,
    each stream equal to its own oracle reconstruction."""
    specs = [(2, 64, 32, 0, False), (3, 48, 32, 1, False), (3, 64, 48, 4, True), (4, 32, 16, 3, False),
             (2, 48, 32, 0, True), (3, 80, 16, 2, False)]
    n = 7
    dcs, hrs, exps = [], [], []
    ia_all = np.zeros((len(specs), n), np.uint8)
    for i, (s, w, h, interp, i420) in enumerate(specs):
        types = synth.default_types(n, 3)
        mk = synth.make_chunk_i420 if i420 else synth.make_chunk
        c = mk(820 + i, w, h, s, n, types=types, interp=interp)
        ia = [0] * n
        ia[1 + i % 5] = 1
        ia_all[i] = ia
        dc, hr, *exp = _case(c, ia, i, i420=i420)
        dcs.append(dc)
        hrs.append(hr)
        exps.append(exp)
    ctx.reconstruct_chunk(dcs, torch.from_numpy(ia_all).to(DEV), hrs)
    torch.cuda.synchronize()
    for i in range(len(specs)):
        _check(dcs[i], hrs[i], *exps[i])


def test_whole_path_8tap(ctx):
    """ns_enhance_streams on an 8-tap (switchable) stream next to a bilinear
    one: anchors are Alg. 1's, every non-anchor frame is the oracle's
    reconstruction from the GPU's own SR anchors, byte for byte."""
    n, k = 12, 3
    m = ctx.model(1, 16, 2)
    blob = synth.make_weights(5, 1, 16, 2)
    m.set_weights(blob)
    cs = [synth.make_chunk(870 + i, 48, 24, 2, n, types=synth.default_types(n, 5), interp=interp)
          for i, interp in enumerate((4, 0))]
    dcs = [dev_chunk(ns, c, DEV, model=m, state=True) for c in cs]
    hrs = [alloc_hr(n, c, DEV) for c in cs]
    ia = torch.zeros((2, n), dtype=torch.uint8, device=DEV)
    ctx.enhance_streams(dcs, hrs, is_anchor_out=ia, k=k)
    torch.cuda.synchronize()
    for i, c in enumerate(cs):
        anchors = list(ia.cpu().numpy()[i])
        assert anchors == oracle.enhance_chunk(c, blob, 1, 16, k)["is_anchor"]
        got = np.stack([t.cpu().numpy() for t in hrs[i]])
        z = np.zeros_like(got[0])
        exp, _, _ = oracle.reconstruct(c, anchors, got, z, z)
        assert np.array_equal(got, exp)


def test_interp_out_of_range_rejected(ctx):
    c = synth.make_chunk(5, 16, 16, 2, 2)
    dc = dev_chunk(ns, c, DEV)
    dc.interp = 5
    hr = alloc_hr(2, c, DEV, fill=7)
    before = ns.launch_count()
    with pytest.raises(ns.NsError) as e:
        ctx.reconstruct_chunk([dc], torch.ones((1, 2), dtype=torch.uint8, device=DEV), [hr])
    assert e.value.status == ns.NS_EINVAL and "interp" in ns.last_error()
    assert ns.launch_count() == before
    assert all(int(t.min()) == 7 == int(t.max()) for t in hr)
