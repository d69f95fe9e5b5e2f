"""ns_enhance_streams_host (include/ns.h): the whole path with the decoder's
outputs in pinned host memory must give exactly the results of the device-input
path (ns_enhance_streams) -- HR frames, anchors, stats and the carried
hr_last / hr_golden state -- while moving only res/mv/type (+ the anchors' LR)
over PCIe, in several overlapped stream groups per call."""
import numpy as np
import pytest
import torch

import paper_conf_sigcomm_yeolkjyh22_b200 as ns
import synth
from helpers import alloc_hr

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


@pytest.fixture(scope="module")
def ctx():
    c = ns.Context(0, pool_bytes=6 << 30)
    yield c
    c.close()


def _streams(seed0, shapes, n, keys, interp=0):
    return [synth.make_chunk(seed0 + i, w, h, s, n, types=synth.default_types(n, keys), interp=interp)
            for i, (w, h, s) in enumerate(shapes)]


def _run_both(ctx, chunks, specs, n_calls=2, **kw):
    """Runs n_calls consecutive chunks of every stream through both paths (fresh
    state buffers per path) and returns the per-call outputs of each."""
    models = []
    for i, ((B, C), c) in enumerate(zip(specs, chunks[0])):
        m = ctx.model(B, C, c.scale)
        m.set_weights(synth.make_weights(700 + i, B, C, c.scale))
        models.append(m)
    outs = {}
    for path in ("device", "host"):
        state = [(torch.zeros((3, c.scale * c.h, c.scale * c.w), dtype=torch.uint8, device=DEV),
                  torch.zeros((3, c.scale * c.h, c.scale * c.w), dtype=torch.uint8, device=DEV)) for c in chunks[0]]
        res = []
        for call in range(n_calls):
            cs = chunks[call]
            n = cs[0].type.shape[0]
            hr = [alloc_hr(n, c, DEV, fill=7) for c in cs]
            ia = torch.zeros((len(cs), n), dtype=torch.uint8, device=DEV)
            st = torch.zeros((len(cs), 8), dtype=torch.float64, device=DEV)
            if path == "device":
                dc = [ns.DeviceChunk.from_numpy(c.lr, c.res, c.mv, c.type, c.w, c.h, c.scale, DEV, model=models[i],
                                                hr_last=state[i][0], hr_golden=state[i][1], interp=c.interp)
                      for i, c in enumerate(cs)]
                ctx.enhance_streams(dc, hr, is_anchor_out=ia, stats=st, **kw)
                moved = None
            else:
                hc = [ns.DeviceChunk.pinned_from_numpy(c.lr, c.res, c.mv, c.type, c.w, c.h, c.scale, model=models[i],
                                                       hr_last=state[i][0], hr_golden=state[i][1], interp=c.interp)
                      for i, c in enumerate(cs)]
                moved = ctx.enhance_streams_host(hc, hr, is_anchor_out=ia, stats=st, **kw)
            torch.cuda.synchronize()
            res.append(dict(hr=[np.stack([t.cpu().numpy() for t in row]) for row in hr], ia=ia.cpu().numpy(),
                            st=st.cpu().numpy(), state=[(a.cpu().numpy(), b.cpu().numpy()) for a, b in state],
                            moved=moved))
        outs[path] = res
    return outs


def _assert_same(outs):
    for d, h in zip(outs["device"], outs["host"]):
        assert np.array_equal(d["ia"], h["ia"])
        assert np.array_equal(d["st"], h["st"])
        for a, b in zip(d["hr"], h["hr"]):
            assert np.array_equal(a, b)
        for (a0, a1), (b0, b1) in zip(d["state"], h["state"]):
            assert np.array_equal(a0, b0) and np.array_equal(a1, b1)


def test_host_path_matches_device_path_topk():
    """5 mixed-shape streams (5 groups of 1 stream: the double-buffered upload
    pipeline wraps), two consecutive chunks (state carried across calls)."""
    c = ns.Context(0, pool_bytes=4 << 30)
    try:
        shapes = [(64, 32, 2), (64, 32, 2), (48, 24, 3), (64, 32, 2), (48, 24, 3)]
        specs = [(2, 16), (1, 16), (1, 32), (2, 16), (1, 32)]
        n, k = 10, 3
        chunks = [_streams(5100 + 10 * call, shapes, n, 4) for call in range(2)]
        outs = _run_both(c, chunks, specs, k=k)
        _assert_same(outs)
        for call in range(2):
            exp = sum(x.res.nbytes + x.mv.nbytes + x.type.nbytes + k * 3 * x.h * x.w for x in chunks[call])
            assert outs["host"][call]["moved"] == exp
    finally:
        c.close()


def test_host_path_8tap_matches_device_path(ctx):
    """8-tap streams (R13) through the host-input call equal the device path."""
    shapes = [(64, 32, 2), (48, 24, 3), (32, 16, 4)]
    chunks = [_streams(5500, shapes, 8, 3, interp=4)]
    outs = _run_both(ctx, chunks, [(1, 16)] * 3, n_calls=1, k=2)
    _assert_same(outs)


def test_host_path_matches_device_path_many_streams(ctx):
    """17 streams -> groups of 3 (6 groups, last one short)."""
    shapes = [(64, 32, 2)] * 17
    specs = [(1, 16)] * 17
    chunks = [_streams(5300, shapes, 6, 3)]
    outs = _run_both(ctx, chunks, specs, n_calls=1, k=2)
    _assert_same(outs)


def test_host_path_global_budget(ctx):
    shapes = [(64, 32, 2), (48, 24, 3), (64, 32, 2)]
    specs = [(1, 16), (1, 32), (1, 16)]
    chunks = [_streams(5400, shapes, 8, 4)]
    outs = _run_both(ctx, chunks, specs, n_calls=1, mode=ns.NS_GLOBAL_BUDGET, budget=9, cost=[1, 2, 1])
    _assert_same(outs)


def test_host_path_rejects_pageable_memory(ctx):
    c = synth.make_chunk(5500, 64, 32, 2, 4, types=synth.default_types(4, None))
    m = ctx.model(1, 16, 2)
    m.set_weights(synth.make_weights(1, 1, 16, 2))
    hc = ns.DeviceChunk.pinned_from_numpy(c.lr, c.res, c.mv, c.type, c.w, c.h, c.scale, model=m)
    hc.res = torch.from_numpy(np.ascontiguousarray(c.res))  # pageable
    hr = [alloc_hr(4, c, DEV)]
    with pytest.raises(ns.NsError) as ei:
        ctx.enhance_streams_host([hc], hr, k=1)
    assert ei.value.status == ns.NS_EINVAL and "page-locked" in str(ei.value)


def test_host_path_i420_matches_device_path(ctx):
    """4:2:0 streams (NS_FMT_I420) through the host-input path: the uploaded
    residual frames and the gathered anchor LR frames have the 4:2:0 sizes;
    results equal the device-input path byte for byte."""
    n, k = 10, 2
    cs = [synth.make_chunk_i420(7300 + i, w, h, s, n, types=synth.default_types(n, 4))
          for i, (w, h, s) in enumerate([(64, 32, 2), (48, 32, 3), (64, 32, 2)])]
    outs = {}
    for path in ("device", "host"):
        dcs, hrs = [], []
        for i, c in enumerate(cs):
            m = ctx.model(1, 16, c.scale)
            m.set_weights(synth.make_weights(7300 + i, 1, 16, c.scale))
            size = c.scale * c.h * c.scale * c.w * 3 // 2
            last = torch.zeros(size, dtype=torch.uint8, device=DEV)
            gold = torch.zeros(size, dtype=torch.uint8, device=DEV)
            mk = ns.DeviceChunk.from_numpy if path == "device" else ns.DeviceChunk.pinned_from_numpy
            kw = dict(device=DEV) if path == "device" else {}
            dcs.append(mk(c.lr, c.res, c.mv, c.type, c.w, c.h, c.scale, model=m, hr_last=last, hr_golden=gold,
                          format=ns.NS_FMT_I420, **kw))
            hrs.append([torch.full((size,), 7, dtype=torch.uint8, device=DEV) for _ in range(n)])
        ia = torch.zeros((len(cs), n), dtype=torch.uint8, device=DEV)
        if path == "device":
            ctx.enhance_streams(dcs, hrs, is_anchor_out=ia, k=k)
        else:
            ctx.enhance_streams_host(dcs, hrs, is_anchor_out=ia, k=k)
        torch.cuda.synchronize()
        outs[path] = (ia.cpu().numpy(), [np.stack([t.cpu().numpy() for t in r]) for r in hrs],
                      [d.hr_last.cpu().numpy() for d in dcs])
    d, h = outs["device"], outs["host"]
    assert np.array_equal(d[0], h[0])
    for a, b in zip(d[1], h[1]):
        assert np.array_equal(a, b)
    for a, b in zip(d[2], h[2]):
        assert np.array_equal(a, b)
