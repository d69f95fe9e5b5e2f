"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bars (BASELINE.json north_star): anchor choice (gain, rank, is_anchor) and the
reuse warp / upsample bit-exact given identical SR reference bytes; SR within
max-abs 2/255 per pixel and mean PSNR difference <= 0.05 dB.
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


@pytest.fixture(scope="module")
def ctx():
    c = ns.Context(0, pool_bytes=12 << 30)
    yield c
    c.close()


def _model(ctx, B, C, s, seed, gain=1.0):
    m = ctx.model(B, C, s)
    blob = synth.make_weights(seed, B, C, s, gain=gain)
    m.set_weights(blob)
    return m, blob


def _select_gpu(ctx, dcs, **kw):
    S, n = len(dcs), dcs[0].n
    gain = torch.zeros((S, n), dtype=torch.int64, device=DEV)
    rank = torch.zeros((S, n), dtype=torch.int32, device=DEV)
    ia = torch.zeros((S, n), dtype=torch.uint8, device=DEV)
    ctx.select_anchors(dcs, gain, rank, ia, **kw)
    torch.cuda.synchronize()
    return gain.cpu().numpy(), rank.cpu().numpy(), ia.cpu().numpy()


# ---------------------------------------------------------------- selection
@pytest.mark.parametrize("types,k,fresh,use_rs", [
    (None, 2, False, False),                           # c1
    ([0, 2, 2, 2, 1, 2, 2, 2], 2, False, False),       # c1-alt
    ([0, 2, 2, 1, 2, 2, 2, 2], 3, True, False),        # FRESH
    (None, 3, False, True),                            # encoded-size proxy
])
def test_select_c1(ctx, types, k, fresh, use_rs):
    t = synth.default_types(8, None) if types is None else np.array(types, np.uint8)
    c = synth.make_chunk(1001, 128, 72, 2, 8, types=t)
    dc = dev_chunk(ns, c, DEV, res_size=use_rs)
    g, r, a = _select_gpu(ctx, [dc], k=k, fresh=fresh, use_res_size=use_rs)
    sc = oracle.score(c.res, c.res_size if use_rs else None)
    eg, er, ea = oracle.select_topk(list(c.type), [int(v) for v in sc], k, oracle.FRESH if fresh else oracle.CARRY)
    assert list(g[0]) == eg
    assert list(r[0]) == er
    assert list(a[0]) == ea


def test_select_many_streams_and_lengths(ctx):
    rng = np.random.default_rng(5)
    for n in (1, 2, 33, 60, 256):
        dcs, cs = [], []
        for s in range(6):
            t = synth.default_types(n, int(rng.integers(2, 9)))
            c = synth.make_chunk(5000 + 17 * s + n, 16, 16, 2, n, types=t)
            cs.append(c)
            dcs.append(dev_chunk(ns, c, DEV))
        k = min(n, 5)
        g, r, a = _select_gpu(ctx, dcs, k=k)
        for s, c in enumerate(cs):
            sc = [int(v) for v in oracle.score(c.res)]
            eg, er, ea = oracle.select_topk(list(c.type), sc, k)
            assert list(g[s]) == eg and list(r[s]) == er and list(a[s]) == ea, (n, s)


def test_select_global_budget(ctx):
    cs, dcs = [], []
    for s in range(7):
        c = synth.make_chunk(7000 + s, 32, 24, 3, 20, types=synth.default_types(20, 6))
        cs.append(c)
        dcs.append(dev_chunk(ns, c, DEV))
    cost = [1 + (s % 3) for s in range(7)]
    for budget in (0, 5, 23, 60, 1000):
        g, r, a = _select_gpu(ctx, dcs, mode=ns.NS_GLOBAL_BUDGET, budget=budget, cost=cost)
        streams = [(list(c.type), [int(v) for v in oracle.score(c.res)]) for c in cs]
        eg, er, ea = oracle.select_global(streams, cost, budget)
        for s in range(7):
            assert list(g[s]) == eg[s] and list(r[s]) == er[s] and list(a[s]) == ea[s], (budget, s)


# ---------------------------------------------------------------- SR
@pytest.mark.parametrize("B,C,s,w,h", [
    (4, 16, 2, 128, 72),     # c1 model
    (1, 32, 3, 64, 40),      # c2/c3 layer shapes, ragged M tile (64 < 128)
    (2, 32, 2, 200, 24),     # ragged W (200 = 128 + 72), C32 x2
    (1, 32, 4, 48, 16),      # x4: two N=256 upsampler launches
    (1, 16, 3, 136, 16),     # C16 x3
    (1, 16, 4, 32, 8),       # C16 x4, 8-row frame
])
def test_sr_small_full_oracle(ctx, B, C, s, w, h):
    m, blob = _model(ctx, B, C, s, seed=11 + B + C + s)
    c = synth.make_chunk(100 + w + h, w, h, s, 2, with_gt=True)
    lr = torch.from_numpy(c.lr).to(DEV)
    hr = torch.zeros((2, 3, s * h, s * w), dtype=torch.uint8, device=DEV)
    ctx.sr_anchors([(m, lr[i], hr[i]) for i in range(2)])
    torch.cuda.synchronize()
    got = hr.cpu().numpy()
    for i in range(2):
        exp = oracle.sr_forward(c.lr[i], blob, B, C, s)
        d = np.abs(got[i].astype(int) - exp.astype(int))
        assert d.max() <= SR_MAX_ABS, (d.max(), np.argwhere(d > SR_MAX_ABS)[:5])
        assert abs(psnr(got[i], c.gt[i]) - psnr(exp, c.gt[i])) <= SR_PSNR_DB


def test_sr_stress_weights(ctx):
    """4x weights (SURVEY.md §8(d) stress variant): the activations grow 4x per
    layer pair, so bf16 storage error grows too.  The 2/255 bar applies to the
    nominal weights; here the max-abs is reported and bounded loosely (8), and
    the mean error must stay small."""
    B, C, s = 2, 32, 3
    m, blob = _model(ctx, B, C, s, seed=77, gain=4.0)
    c = synth.make_chunk(78, 64, 32, s, 1)
    lr = torch.from_numpy(c.lr).to(DEV)
    hr = torch.zeros((1, 3, s * 32, s * 64), dtype=torch.uint8, device=DEV)
    ctx.sr_anchors([(m, lr[0], hr[0])])
    torch.cuda.synchronize()
    exp = oracle.sr_forward(c.lr[0], blob, B, C, s)
    d = np.abs(hr.cpu().numpy()[0].astype(int) - exp.astype(int))
    print(f"stress x4 weights: max-abs {d.max()}, mean {d.mean():.4f}")
    assert d.max() <= 8 and d.mean() < 0.5


def test_sr_mixed_models_batch(ctx):
    """Jobs of different streams carry different content-aware weights
    and different shapes, batched in one call."""
    specs = [(2, 16, 2, 64, 32), (2, 16, 2, 64, 32), (1, 32, 3, 48, 24), (2, 16, 2, 64, 32)]
    models, jobs, exp = [], [], []
    for i, (B, C, s, w, h) in enumerate(specs):
        m, blob = _model(ctx, B, C, s, seed=300 + i)
        c = synth.make_chunk(400 + i, w, h, s, 1)
        lr = torch.from_numpy(c.lr[0]).to(DEV)
        hr = torch.zeros((3, s * h, s * w), dtype=torch.uint8, device=DEV)
        jobs.append((m, lr, hr))
        exp.append(oracle.sr_forward(c.lr[0], blob, B, C, s))
        models.append(m)
    ctx.sr_anchors(jobs)
    torch.cuda.synchronize()
    for (m, lr, hr), e in zip(jobs, exp):
        d = np.abs(hr.cpu().numpy().astype(int) - e.astype(int))
        assert d.max() <= SR_MAX_ABS


# ---------------------------------------------------------------- reconstruct
def _recon_case(ctx, c, ia, seed_anchor=0, state=False):
    n, s = c.n, c.scale
    rng = np.random.default_rng(seed_anchor)
    hr_anchor = np.zeros((n, 3, s * c.h, s * c.w), np.uint8)
    for f in range(n):
        if ia[f]:
            hr_anchor[f] = rng.integers(0, 256, hr_anchor[f].shape)
    last0 = rng.integers(0, 256, hr_anchor[0].shape).astype(np.uint8) if state else None
    gold0 = rng.integers(0, 256, hr_anchor[0].shape).astype(np.uint8) if state else None
    exp, elast, egold = oracle.reconstruct(c, ia, hr_anchor, last0, gold0)
    dc = dev_chunk(ns, c, DEV)
    if state:
        dc.hr_last = torch.from_numpy(last0).to(DEV)
        dc.hr_golden = torch.from_numpy(gold0).to(DEV)
    hr = [torch.from_numpy(hr_anchor[f]).to(DEV) for f in range(n)]
    ia_t = torch.from_numpy(np.array(ia, np.uint8)[None]).to(DEV)
    ctx.reconstruct_chunk([dc], ia_t, [hr])
    torch.cuda.synchronize()
    got = np.stack([t.cpu().numpy() for t in hr])
    for f in range(n):
        assert np.array_equal(got[f], exp[f]), (f, int(np.abs(got[f].astype(int) - exp[f]).max()))
    if state:
        assert np.array_equal(dc.hr_last.cpu().numpy(), elast)
        assert np.array_equal(dc.hr_golden.cpu().numpy(), egold)


@pytest.mark.parametrize("s", [2, 3, 4])
def test_reconstruct_bit_exact(ctx, s):
    c = synth.make_chunk(900 + s, 64, 40, s, 12, types=synth.default_types(12, 5))
    _recon_case(ctx, c, [1, 0, 0, 0, 0, 1, 0, 0, 0, 0, 0, 0])


def test_reconstruct_no_key_uses_state(ctx):
    t = np.array([2, 2, 1, 2, 2, 2], np.uint8)   # chunk without a leading KEY
    c = synth.make_chunk(950, 32, 24, 3, 6, types=t)
    c.mv["ref"][0][c.mv["ref"][0] == synth.NS_REF_INTRA] = synth.NS_REF_LAST
    c.mv["ref"][0][::2, ::2] = synth.NS_REF_GOLDEN
    _recon_case(ctx, c, [0, 0, 0, 1, 0, 0], state=True)


def test_reconstruct_zero_motion_identity(ctx):
    c = synth.make_chunk(960, 48, 32, 3, 5, types=synth.default_types(5, None))
    c.res[:] = 0
    c.mv["mvx"] = 0
    c.mv["mvy"] = 0
    c.mv["ref"][1:] = synth.NS_REF_LAST
    _recon_case(ctx, c, [1, 0, 0, 0, 0])


# ---------------------------------------------------------------- whole path
def _enhance_vs_oracle(ctx, cs, specs, k, **kw):
    dcs, blobs, hr = [], [], []
    for c, (B, C) in zip(cs, specs):
        m, blob = _model(ctx, B, C, c.scale, seed=c.w * 7 + c.h + B)
        blobs.append(blob)
        dcs.append(dev_chunk(ns, c, DEV, model=m, with_gt=c.gt is not None, state=True))
        hr.append(alloc_hr(c.n, c, DEV))
    S, n = len(cs), cs[0].n
    ia = torch.zeros((S, n), dtype=torch.uint8, device=DEV)
    stats = torch.zeros((S, 8), dtype=torch.float64, device=DEV)
    ctx.enhance_streams(dcs, hr, is_anchor_out=ia, stats=stats, k=k, **kw)
    torch.cuda.synchronize()
    ia = ia.cpu().numpy()
    st = stats.cpu().numpy()
    for si, c in enumerate(cs):
        B, C = specs[si]
        ref = oracle.enhance_chunk(c, blobs[si], B, C, k)
        assert list(ia[si]) == ref["is_anchor"]
        got = np.stack([t.cpu().numpy() for t in hr[si]])
        d = np.abs(got.astype(int) - ref["hr"].astype(int))
        assert d.max() <= SR_MAX_ABS, (si, d.max())
        assert st[si, 0] == n and st[si, 1] == sum(ref["is_anchor"])
        assert st[si, 3] == float(sum(int(v) for v in ref["score"]))
        if c.gt is not None:
            p_gpu = st[si, 5]
            assert abs(p_gpu - psnr(got, c.gt)) < 1e-6
            assert abs(p_gpu - psnr(ref["hr"], c.gt)) <= SR_PSNR_DB
        assert np.array_equal(dcs[si].hr_last.cpu().numpy(), got[-1])


def test_enhance_c1(ctx):
    c = synth.make_chunk(1001, 128, 72, 2, 8, types=synth.default_types(8, None), with_gt=True)
    _enhance_vs_oracle(ctx, [c], [(4, 16)], k=2)


def test_enhance_multistream_mixed(ctx):
    cs = [synth.make_chunk(2100 + i, w, h, s, 10, types=synth.default_types(10, 4), with_gt=True)
          for i, (w, h, s) in enumerate([(64, 32, 2), (64, 32, 2), (48, 24, 3), (64, 32, 2), (48, 24, 3)])]
    specs = [(2, 16), (2, 16), (1, 32), (2, 16), (1, 32)]
    _enhance_vs_oracle(ctx, cs, specs, k=3)


def test_enhance_two_sr_batches(ctx):
    """More anchors of one shape than one SR batch holds (24 > 16): the batches
    alternate between the caller's stream and the context's second SR stream,
    each with its own arena (ns_api.cu run_sr_group); the results are the
    oracle's as for one batch."""
    cs = [synth.make_chunk(2300 + i, 48, 24, 2, 8, types=synth.default_types(8, 4), with_gt=True) for i in range(6)]
    _enhance_vs_oracle(ctx, cs, [(1, 16)] * 6, k=4)


@pytest.mark.parametrize("k", [0, 8])
def test_enhance_k_extremes(ctx, k):
    """k = 0 (pure reuse from KEY up-sampling) and k = n (per-frame SR)."""
    c = synth.make_chunk(3100 + k, 64, 32, 2, 8, types=synth.default_types(8, None))
    _enhance_vs_oracle(ctx, [c], [(2, 16)], k=k)


# ---------------------------------------------------------------- c2 full size
@pytest.mark.slow
def test_c2_full_size(ctx):
    cfg = synth.CONFIGS[2]
    B, C, s, n, k = cfg["n_blocks"], cfg["n_ch"], cfg["scale"], cfg["n"], cfg["k"]
    c = synth.make_chunk(2001, cfg["w"], cfg["h"], s, n, types=synth.default_types(n, 16))
    m, blob = _model(ctx, B, C, s, seed=2001)
    dc = dev_chunk(ns, c, DEV, model=m, state=True)
    hr = alloc_hr(n, c, DEV)
    ia = torch.zeros((1, n), dtype=torch.uint8, device=DEV)
    ctx.enhance_streams([dc], [hr], is_anchor_out=ia, k=k)
    torch.cuda.synchronize()
    sc = [int(v) for v in oracle.score(c.res)]
    _, _, ea = oracle.select_topk(list(c.type), sc, k)
    assert list(ia.cpu().numpy()[0]) == ea
    got = np.stack([t.cpu().numpy() for t in hr])
    # SR: sampled windows (corners, edges, interior) of every anchor
    wins = [(0, 0, 24, 32), (0, cfg["w"] - 40, 24, 40), (cfg["h"] - 16, 0, 16, 48),
            (cfg["h"] - 24, cfg["w"] - 32, 24, 32), (170, 300, 20, 36)]
    for f in [f for f in range(n) if ea[f]]:
        for (Y0, X0, HH, WW), patch in oracle_sr_crops(c.lr[f], blob, B, C, s, wins):
            d = np.abs(got[f][:, Y0:Y0 + HH, X0:X0 + WW].astype(int) - patch.astype(int))
            assert d.max() <= SR_MAX_ABS, (f, (Y0, X0), d.max())
    # reuse: bit-exact against the oracle given the GPU's own SR anchor bytes
    exp, _, _ = oracle.reconstruct(c, ea, got, np.zeros_like(got[0]), np.zeros_like(got[0]))
    assert np.array_equal(got, exp)


# ---------------------------------------------------------------- c3 / c4 full size (bench config)
@pytest.mark.slow
def test_c3_full_size_batched(ctx):
    """BASELINE configs[2]/[3] at full size through the bench's call
    (ns_enhance_streams, several streams with distinct content-aware models,
    SR jobs batched across streams): selection bit-exact for every stream; SR
    on sampled windows incl. the four frame corners (exercises the exact
    frame-border fix-up of the composed upsampler+tail); reconstruction of a
    whole 60-frame 4K chunk bit-exact given the GPU's SR anchor bytes."""
    cfg = synth.CONFIGS[3]
    B, C, s, n, k = cfg["n_blocks"], cfg["n_ch"], cfg["scale"], cfg["n"], cfg["k"]
    w, h = cfg["w"], cfg["h"]
    S = 3
    cs = [synth.make_chunk(3001 + i, w, h, s, n, types=synth.default_types(n, 16)) for i in range(S)]
    blobs, dcs, hrs = [], [], []
    for i, c in enumerate(cs):
        m, blob = _model(ctx, B, C, s, seed=3001 + i)
        blobs.append(blob)
        dcs.append(dev_chunk(ns, c, DEV, model=m, state=True))
        hrs.append(alloc_hr(n, c, DEV))
    ia = torch.zeros((S, n), dtype=torch.uint8, device=DEV)
    ctx.enhance_streams(dcs, hrs, is_anchor_out=ia, k=k)
    torch.cuda.synchronize()
    ia = ia.cpu().numpy()
    for i, c in enumerate(cs):
        sc = [int(v) for v in oracle.score(c.res)]
        _, _, ea = oracle.select_topk(list(c.type), sc, k)
        assert list(ia[i]) == ea, i
    c, blob = cs[0], blobs[0]
    got = np.stack([t.cpu().numpy() for t in hrs[0]])
    wins = [(0, 0, 16, 24), (0, w - 24, 16, 24), (h - 16, 0, 16, 24), (h - 16, w - 24, 16, 24), (352, 640, 16, 24)]
    anchors = [f for f in range(n) if ia[0, f]]
    worst = 0
    for f in anchors[:3]:
        for (Y0, X0, HH, WW), patch in oracle_sr_crops(c.lr[f], blob, B, C, s, wins):
            d = np.abs(got[f][:, Y0:Y0 + HH, X0:X0 + WW].astype(int) - patch.astype(int))
            worst = max(worst, int(d.max()))
    assert worst <= SR_MAX_ABS, worst
    exp, _, _ = oracle.reconstruct(c, list(ia[0]), got, np.zeros_like(got[0]), np.zeros_like(got[0]))
    assert np.array_equal(got, exp)


# ---------------------------------------------------------------- SR is a pure function
@pytest.mark.parametrize("C,s", [(16, 2), (32, 3)])
def test_sr_deterministic_across_batches(ctx, C, s):
    """SR(weights, LR) must not depend on what ran before or on the batch it is
    in: tensor-memory accumulators start at zero in every CTA (TMEM keeps what
    an earlier CTA on the SM left unretired).  256 LR rows span three res-block
    strips (y0 = 0, 120, 240) and several uptail / head strips."""
    m, _ = _model(ctx, 2, C, s, seed=91)
    w, h = 136, 256
    lrs = [torch.from_numpy(synth.make_chunk(9100 + i, w, h, s, 1).lr[0]).to(DEV) for i in range(5)]
    outs = []
    for order in ([0, 1, 2, 3, 4], [4, 3, 2, 1, 0], [2], [0, 2, 4]):
        hr = {i: torch.zeros((3, s * h, s * w), dtype=torch.uint8, device=DEV) for i in order}
        # unrelated work in between leaves different TMEM contents behind
        other, _ = _model(ctx, 1, C, s, seed=92 + len(outs))
        junk = torch.zeros((3, s * 64, s * 64), dtype=torch.uint8, device=DEV)
        ctx.sr_anchors([(other, torch.randint(0, 256, (3, 64, 64), dtype=torch.uint8, device=DEV), junk)])
        ctx.sr_anchors([(m, lrs[i], hr[i]) for i in order])
        torch.cuda.synchronize()
        outs.append({i: t.cpu().numpy() for i, t in hr.items()})
    for o in outs[1:]:
        for i, a in o.items():
            assert np.array_equal(a, outs[0][i]), i
