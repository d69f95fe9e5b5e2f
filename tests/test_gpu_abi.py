"""C-ABI argument validation on a real context (SURVEY.md §4.2 "ABI tests";
include/ns.h conventions): every invalid call returns the documented negative
ns_status, sets ns_last_error(), launches nothing (ns_launch_count unchanged)
and leaves every output untouched."""
import ctypes

import numpy as np
import pytest

import synth
from helpers import dev_chunk

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ns = pytest.importorskip("paper_conf_sigcomm_yeolkjyh22_b200")

DEV = "cuda:0"


@pytest.fixture(scope="module")
def ctx():
    c = ns.Context(0, pool_bytes=4 << 30)
    yield c
    c.close()


@pytest.fixture(scope="module")
def model(ctx):
    m = ctx.model(1, 16, 2)
    m.set_weights(synth.make_weights(5, 1, 16, 2))
    return m


def _chunk(model, w=32, h=16, s=2, n=4, seed=1):
    c = synth.make_chunk(seed, w, h, s, n, types=synth.default_types(n, None))
    return c, dev_chunk(ns, c, DEV, model=model, state=True)


def _expect(status, fn, *args, msg=None, **kw):
    torch.cuda.synchronize()
    before = ns.launch_count()
    with pytest.raises(ns.NsError) as ei:
        fn(*args, **kw)
    assert ei.value.status == status, (ei.value.status, str(ei.value))
    if msg:
        assert msg in str(ei.value), str(ei.value)
    assert ns.launch_count() == before, "a rejected call launched kernels"
    torch.cuda.synchronize()
    return str(ei.value)


def _outs(n, c, fill=77):
    hr = [torch.full((3, c.scale * c.h, c.scale * c.w), fill, dtype=torch.uint8, device=DEV) for _ in range(n)]
    ia = torch.full((1, n), 7, dtype=torch.uint8, device=DEV)
    return hr, ia


def _untouched(hr, ia, fill=77):
    torch.cuda.synchronize()
    assert all(bool((t == fill).all()) for t in hr)
    assert bool((ia == 7).all())


def test_shape_and_scale_rejected(ctx, model):
    c, dc = _chunk(model)
    hr, ia = _outs(c.n, c)
    bad = dict(vars(dc))
    for field, val, msg in (("w", 36, "multiples of 8"), ("h", 12, "multiples of 8"), ("scale", 5, "scale"),
                            ("scale", 1, "scale")):
        d2 = ns.DeviceChunk(**{**bad, field: val})
        _expect(ns.NS_EINVAL, ctx.enhance_streams, [d2], [hr], is_anchor_out=ia, k=1, msg=msg)
    # model scale != chunk scale
    m3 = ctx.model(1, 16, 3)
    m3.set_weights(synth.make_weights(6, 1, 16, 3))
    d3 = ns.DeviceChunk(**{**bad, "model": m3})
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [d3], [hr], is_anchor_out=ia, k=1, msg="model scale")
    # a model without weights
    m0 = ctx.model(1, 16, 2)
    d0 = ns.DeviceChunk(**{**bad, "model": m0})
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [d0], [hr], is_anchor_out=ia, k=1, msg="no weights")
    _untouched(hr, ia)


def test_k_and_params_rejected(ctx, model):
    c, dc = _chunk(model)
    hr, ia = _outs(c.n, c)
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [dc], [hr], is_anchor_out=ia, k=c.n + 1, msg="k =")
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [dc], [hr], is_anchor_out=ia, k=-1)
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [dc], [hr], is_anchor_out=ia, mode=7)
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [dc], [hr], is_anchor_out=ia, k=1, selector=9)
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [dc], [hr], is_anchor_out=ia, mode=ns.NS_GLOBAL_BUDGET, budget=3)
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [dc], [hr], is_anchor_out=ia, mode=ns.NS_GLOBAL_BUDGET, budget=3,
            cost=[0])
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [dc], [hr], is_anchor_out=ia, mode=ns.NS_GIVEN_ANCHORS, budget=3,
            cost=[1])
    gain = torch.zeros((1, c.n), dtype=torch.int64, device=DEV)
    rank = torch.zeros((1, c.n), dtype=torch.int32, device=DEV)
    _expect(ns.NS_EINVAL, ctx.select_anchors, [dc], gain, rank, ia, mode=ns.NS_GIVEN_ANCHORS, anchor_in=ia,
            cost=[1], budget=1)
    _expect(ns.NS_EINVAL, ctx.select_anchors, [dc], gain, rank, ia, k=c.n + 1)
    _untouched(hr, ia)


def test_chunk_mismatch_and_alignment_rejected(ctx, model):
    c, dc = _chunk(model)
    c2, dc2 = _chunk(model, n=5, seed=2)
    hr, ia = _outs(c.n, c)
    hr2, _ = _outs(c2.n, c2)
    _expect(ns.NS_EINVAL, ctx.select_anchors, [dc, dc2], torch.zeros((2, 4), dtype=torch.int64, device=DEV),
            torch.zeros((2, 4), dtype=torch.int32, device=DEV), torch.zeros((2, 4), dtype=torch.uint8, device=DEV),
            k=1, msg="n_frames")
    flat = torch.zeros(dc.lr.numel() + 16, dtype=torch.uint8, device=DEV)
    mis = ns.DeviceChunk(**{**vars(dc), "lr": flat[1:1 + dc.lr.numel()]})
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [mis], [hr], is_anchor_out=ia, k=1, msg="16-B aligned")
    _untouched(hr, ia)


def test_hr_aliasing_rejected(ctx, model):
    c, dc = _chunk(model)
    hr, ia = _outs(c.n, c)
    # frame f writes over the LAST reference it reads (f - 1)
    alias = list(hr)
    alias[2] = alias[1]
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [dc], [alias], is_anchor_out=ia, k=1, msg="aliases")
    _expect(ns.NS_EINVAL, ctx.reconstruct_chunk, [dc], ia, [alias], msg="aliases")
    # an output frame is the stream's own state slot
    alias = list(hr)
    alias[3] = dc.hr_last
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [dc], [alias], is_anchor_out=ia, k=1, msg="hr_last")
    alias = list(hr)
    alias[0] = dc.hr_golden
    _expect(ns.NS_EINVAL, ctx.reconstruct_chunk, [dc], ia, [alias], msg="hr_golden")
    # hr_last == hr_golden
    d2 = ns.DeviceChunk(**{**vars(dc), "hr_golden": dc.hr_last})
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [d2], [hr], is_anchor_out=ia, k=1)
    # two streams sharing an output frame
    c2, dcb = _chunk(model, seed=3)
    hrb, _ = _outs(c2.n, c2)
    hrb[1] = hr[1]
    ia2 = torch.full((2, c.n), 7, dtype=torch.uint8, device=DEV)
    _expect(ns.NS_EINVAL, ctx.enhance_streams, [dc, dcb], [hr, hrb], is_anchor_out=ia2, k=1, msg="another stream")
    _untouched(hr, ia)


def test_sr_jobs_rejected(ctx, model):
    lr = torch.zeros((3, 16, 36), dtype=torch.uint8, device=DEV)
    hr = torch.zeros((3, 32, 72), dtype=torch.uint8, device=DEV)
    _expect(ns.NS_EINVAL, ctx.sr_anchors, [(model, lr, hr)], msg="multiples of 8")
    lr_buf = torch.zeros(3 * 16 * 32 + 4, dtype=torch.uint8, device=DEV)
    hr_ok = torch.zeros((3, 32, 64), dtype=torch.uint8, device=DEV)
    _expect(ns.NS_EINVAL, ctx.sr_anchors, [(model, lr_buf[4:].view(3, 16, 32), hr_ok)], msg="aligned")
    L = ns.lib()
    assert L.ns_sr_anchors(ctypes.c_void_p(ctx.handle), None, 2, None) == ns.NS_EINVAL


def test_model_args_rejected(ctx):
    with pytest.raises(ns.NsError) as ei:
        ctx.model(1, 24, 2)
    assert ei.value.status == ns.NS_EUNSUPPORTED
    for args in ((0, 16, 2), (1, 16, 5), (65, 16, 2)):
        with pytest.raises(ns.NsError) as ei:
            ctx.model(*args)
        assert ei.value.status == ns.NS_EINVAL
    m = ctx.model(1, 16, 2)
    with pytest.raises(ns.NsError) as ei:
        m.set_weights(np.zeros(10, np.uint16))
    assert ei.value.status == ns.NS_EINVAL


def test_pool_too_small():
    """A pool below the fixed scratch is rejected at create; a pool that holds
    the scratch but not an SR arena fails the SR call with NS_ENOMEM before
    anything is launched -- including the whole path, whose selection would
    otherwise already have run."""
    with pytest.raises(ns.NsError) as ei:
        ns.Context(0, pool_bytes=64 << 20)
    assert ei.value.status == ns.NS_EINVAL
    small = ns.Context(0, pool_bytes=400 << 20)
    try:
        m = small.model(8, 32, 3)
        m.set_weights(synth.make_weights(9, 8, 32, 3))
        lr = torch.zeros((3, 720, 1280), dtype=torch.uint8, device=DEV)
        hr = torch.full((3, 2160, 3840), 5, dtype=torch.uint8, device=DEV)
        _expect(ns.NS_ENOMEM, small.sr_anchors, [(m, lr, hr)], msg="pool")
        assert bool((hr == 5).all())
        c = synth.make_chunk(11, 1280, 720, 3, 2, types=synth.default_types(2, None))
        dc = dev_chunk(ns, c, DEV, model=m, state=True)
        hrs = [torch.full((3, 2160, 3840), 5, dtype=torch.uint8, device=DEV) for _ in range(2)]
        ia = torch.full((1, 2), 7, dtype=torch.uint8, device=DEV)
        _expect(ns.NS_ENOMEM, small.enhance_streams, [dc], [hrs], is_anchor_out=ia, k=1, msg="pool")
        _untouched(hrs, ia, fill=5)
    finally:
        small.close()
