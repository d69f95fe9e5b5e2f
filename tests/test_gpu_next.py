"""GPU parity of the SURVEY §8(f) NEXT rows built this round, through the C ABI:

  NEXT-4  the real-time baseline selectors of §3: Key SR and
          Key+Uniform SR (ns_select_params.selector), bit-exact against
          oracle/select.py, and through the whole path;
  NEXT-1  global anchor selection across GPUs (§5.2): per-GPU
          gains -> gathered rows -> ns_select_merge, emulated here with the
          streams split into shards on one device (the gather is a
          concatenation); bit-exact against oracle merge_gathered and equal to
          the single-call global mode; the whole path in NS_GIVEN_ANCHORS mode
          per shard gives byte-identical frames to one global call.
"""
import numpy as np
import pytest

import oracle
import synth
from helpers import alloc_hr, dev_chunk
from oracle import select as OS

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ns = pytest.importorskip("paper_conf_sigcomm_yeolkjyh22_b200")

DEV = "cuda:0"


@pytest.fixture(scope="module")
def ctx():
    c = ns.Context(0, pool_bytes=6 << 30)
    yield c
    c.close()


def _select_gpu(ctx, dcs, **kw):
    S, n = len(dcs), dcs[0].n
    gain = torch.zeros((S, n), dtype=torch.int64, device=DEV)
    rank = torch.zeros((S, n), dtype=torch.int32, device=DEV)
    ia = torch.zeros((S, n), dtype=torch.uint8, device=DEV)
    ctx.select_anchors(dcs, gain, rank, ia, **kw)
    torch.cuda.synchronize()
    return gain, rank, ia


# ---------------------------------------------------------------- NEXT-4
@pytest.mark.parametrize("selector,name", [(ns.NS_SEL_KEY, "key"), (ns.NS_SEL_KEY_UNIFORM, "key_uniform")])
def test_baseline_selectors_bit_exact(ctx, selector, name):
    rng = np.random.default_rng(21)
    for n in (1, 7, 8, 60, 61, 256):
        cs = [synth.make_chunk(9000 + 31 * s + n, 16, 16, 2, n, types=synth.default_types(n, int(rng.integers(2, 9))))
              for s in range(5)]
        # a chunk without a leading key frame, and one with extra key frames
        t = synth.default_types(n, None).copy()
        t[0] = synth.NS_NORMAL
        cs.append(synth.make_chunk(9500 + n, 16, 16, 2, n, types=t))
        t2 = synth.default_types(n, 4).copy()
        t2[n // 2] = 0
        cs.append(synth.make_chunk(9600 + n, 16, 16, 2, n, types=t2))
        dcs = [dev_chunk(ns, c, DEV) for c in cs]
        for k in sorted({0, 1, min(n, 5), n}):
            g, r, a = (x.cpu().numpy() for x in _select_gpu(ctx, dcs, k=k, selector=selector))
            for s, c in enumerate(cs):
                fn = OS.select_key if name == "key" else OS.select_key_uniform
                eg, er, ea = fn([int(v) for v in c.type], k)
                assert list(g[s]) == eg and list(r[s]) == er and list(a[s]) == ea, (n, k, s)


def test_baseline_selector_rejected_in_global_mode(ctx):
    c = synth.make_chunk(9700, 16, 16, 2, 8)
    with pytest.raises(ns.NsError):
        _select_gpu(ctx, [dev_chunk(ns, c, DEV)], mode=ns.NS_GLOBAL_BUDGET, budget=3, cost=[1],
                    selector=ns.NS_SEL_KEY_UNIFORM)


@pytest.mark.parametrize("selector,name", [(ns.NS_SEL_KEY, "key"), (ns.NS_SEL_KEY_UNIFORM, "key_uniform")])
def test_baseline_selector_whole_path(ctx, selector, name):
    c = synth.make_chunk(9800, 64, 32, 2, 12, types=synth.default_types(12, 6))
    m = ctx.model(2, 16, 2)
    blob = synth.make_weights(77, 2, 16, 2)
    m.set_weights(blob)
    dc = dev_chunk(ns, c, DEV, model=m, state=True)
    hr = [alloc_hr(c.n, c, DEV)]
    ia = torch.zeros((1, c.n), dtype=torch.uint8, device=DEV)
    ctx.enhance_streams([dc], hr, is_anchor_out=ia, k=4, selector=selector)
    torch.cuda.synchronize()
    ref = oracle.enhance_chunk(c, blob, 2, 16, 4, selector=name)
    assert list(ia.cpu().numpy()[0]) == ref["is_anchor"]
    got = np.stack([t.cpu().numpy() for t in hr[0]])
    assert np.abs(got.astype(int) - ref["hr"].astype(int)).max() <= 2


# ---------------------------------------------------------------- NEXT-1
def _shards(S):
    """Two unequal, interleaved shards of S streams (rank 0: sid % 3 == 0)."""
    a = [i for i in range(S) if i % 3 == 0]
    b = [i for i in range(S) if i % 3 != 0]
    return [a, b]


def test_select_merge_bit_exact(ctx):
    S, n = 9, 24
    cs = [synth.make_chunk(9900 + s, 32, 24, 3, n, types=synth.default_types(n, 8)) for s in range(S)]
    dcs = [dev_chunk(ns, c, DEV) for c in cs]
    cost = [1 + (s % 3) for s in range(S)]
    streams = [(list(c.type), [int(v) for v in oracle.score(c.res)]) for c in cs]
    for budget in (0, 7, 30, 75, 10_000):
        rows = {"g": [], "r": [], "t": [], "sid": [], "cost": []}
        for shard in _shards(S):
            g, r, _ = _select_gpu(ctx, [dcs[i] for i in shard], k=0)
            rows["g"].append(g)
            rows["r"].append(r)
            rows["t"].append(torch.stack([dcs[i].type for i in shard]))
            rows["sid"] += shard
            rows["cost"] += [cost[i] for i in shard]
        g_all, r_all, t_all = (torch.cat(rows[k]) for k in ("g", "r", "t"))
        sid = torch.tensor(rows["sid"], dtype=torch.int32, device=DEV)
        co = torch.tensor(rows["cost"], dtype=torch.int64, device=DEV)
        rank = torch.empty_like(r_all)
        anc = torch.empty_like(t_all)
        ctx.select_merge(g_all, r_all, t_all, sid, co, budget, rank, anc)
        torch.cuda.synchronize()
        er, ea = OS.merge_gathered(t_all.cpu().tolist(), g_all.cpu().tolist(), rows["sid"], rows["cost"], budget)
        assert rank.cpu().tolist() == er and anc.cpu().tolist() == ea, budget
        # equals the single-call global mode over all streams (sid order)
        gg, gr, ga = (x.cpu().numpy() for x in _select_gpu(ctx, dcs, mode=ns.NS_GLOBAL_BUDGET, budget=budget,
                                                            cost=cost))
        _, _, oa = oracle.select_global(streams, cost, budget)
        for j, s in enumerate(rows["sid"]):
            assert list(ga[s]) == anc[j].cpu().tolist() == oa[s]
            assert list(gr[s]) == rank[j].cpu().tolist()


def test_select_merge_does_not_trust_rank_in(ctx):
    """ns_select_merge rebuilds each stream's priority order from (type, gain
    desc, frame asc) (ns.h): a rank array from a baseline selector, a garbage
    one (values >= n, negative) or NULL give the same merge as the true ranks."""
    S, n = 5, 16
    cs = [synth.make_chunk(9800 + s, 32, 24, 3, n, types=synth.default_types(n, 5)) for s in range(S)]
    dcs = [dev_chunk(ns, c, DEV) for c in cs]
    g, r, _ = _select_gpu(ctx, dcs, k=0)
    t_all = torch.stack([d.type for d in dcs])
    sid = torch.arange(S, dtype=torch.int32, device=DEV)
    co = torch.tensor([1, 2, 1, 3, 1], dtype=torch.int64, device=DEV)
    _, rk, _ = _select_gpu(ctx, dcs, k=3, selector=ns.NS_SEL_KEY_UNIFORM)
    bad = torch.randint(-1000, 1000, r.shape, dtype=torch.int32, device=DEV)
    outs = []
    for rin in (r, rk, bad, None):
        rank = torch.empty_like(r)
        anc = torch.empty_like(t_all)
        ctx.select_merge(g, rin, t_all, sid, co, 17, rank, anc)
        torch.cuda.synchronize()
        outs.append((rank.cpu().tolist(), anc.cpu().tolist()))
    er, ea = OS.merge_gathered(t_all.cpu().tolist(), g.cpu().tolist(), list(range(S)), [1, 2, 1, 3, 1], 17)
    for o in outs:
        assert o == (er, ea)


def test_enhance_given_anchors_equals_global(ctx):
    """Per-shard whole path on the merged anchor map == one global call."""
    S, n = 6, 10
    cs = [synth.make_chunk(9950 + s, 48, 24, 2, n, types=synth.default_types(n, 4)) for s in range(S)]
    cost = [1 + (s % 2) for s in range(S)]
    budget = 11
    m = ctx.model(1, 16, 2)
    m.set_weights(synth.make_weights(78, 1, 16, 2))

    def run(groups, given):
        out = {}
        for shard in groups:
            dcs = [dev_chunk(ns, cs[i], DEV, model=m, state=True) for i in shard]
            hr = [alloc_hr(n, cs[i], DEV, fill=3) for i in shard]
            ia = torch.zeros((len(shard), n), dtype=torch.uint8, device=DEV)
            kw = dict(cost=[cost[i] for i in shard], budget=budget)
            if given is None:
                ctx.enhance_streams(dcs, hr, is_anchor_out=ia, mode=ns.NS_GLOBAL_BUDGET, **kw)
            else:
                anc_in = given[shard[0]]
                ctx.enhance_streams(dcs, hr, is_anchor_out=ia, mode=ns.NS_GIVEN_ANCHORS, anchor_in=anc_in, **kw)
            torch.cuda.synchronize()
            for j, i in enumerate(shard):
                out[i] = (ia[j].cpu().numpy(), np.stack([t.cpu().numpy() for t in hr[j]]),
                          dcs[j].hr_last.cpu().numpy(), dcs[j].hr_golden.cpu().numpy())
        return out

    ref = run([list(range(S))], None)
    # merged selection across two shards
    given = {}
    shards = _shards(S)
    rows = []
    for shard in shards:
        g, r, _ = _select_gpu(ctx, [dev_chunk(ns, cs[i], DEV) for i in shard], k=0)
        rows.append((g, r, torch.stack([torch.from_numpy(cs[i].type).to(DEV) for i in shard])))
    g_all, r_all, t_all = (torch.cat([x[j] for x in rows]) for j in range(3))
    sid_l = shards[0] + shards[1]
    rank = torch.empty_like(r_all)
    anc = torch.empty_like(t_all)
    ctx.select_merge(g_all, r_all, t_all, torch.tensor(sid_l, dtype=torch.int32, device=DEV),
                     torch.tensor([cost[i] for i in sid_l], dtype=torch.int64, device=DEV), budget, rank, anc)
    off = 0
    for shard in shards:
        given[shard[0]] = anc[off:off + len(shard)].contiguous()
        off += len(shard)
    got = run(shards, given)
    assert sum(int(ref[i][0].sum()) for i in range(S)) > 0
    for i in range(S):
        for a, b in zip(ref[i], got[i]):
            assert np.array_equal(a, b), i


@pytest.mark.parametrize("kw", [dict(k=10, selector=ns.NS_SEL_KEY), dict(k=3, selector=ns.NS_SEL_KEY_UNIFORM),
                                "given"])
def test_host_path_new_modes_match_device_path(ctx, kw):
    """ns_enhance_streams_host == ns_enhance_streams for the baseline selectors
    (Key SR has fewer anchors than k: claimed job slots) and a given map."""
    S, n = 5, 10
    cs = [synth.make_chunk(9970 + i, 48, 24, 2, n, types=synth.default_types(n, 4)) for i in range(S)]
    cs[2].type[5] = synth.NS_KEY                                  # two key frames in one stream
    m = ctx.model(1, 16, 2)
    m.set_weights(synth.make_weights(79, 1, 16, 2))
    if kw == "given":
        anc = torch.zeros((S, n), dtype=torch.uint8, device=DEV)
        anc[:, 0] = 1
        anc[1, 4] = anc[3, 7] = anc[4, 2] = 1
        kw = dict(mode=ns.NS_GIVEN_ANCHORS, anchor_in=anc, cost=[1] * S, budget=8)
    outs = []
    for path in ("device", "host"):
        state = [torch.zeros((3, 2 * c.h, 2 * c.w), dtype=torch.uint8, device=DEV) for c in cs]
        gold = [torch.zeros_like(t) for t in state]
        hr = [alloc_hr(n, c, DEV, fill=9) for c in cs]
        ia = torch.zeros((S, n), dtype=torch.uint8, device=DEV)
        if path == "device":
            dc = [ns.DeviceChunk.from_numpy(c.lr, c.res, c.mv, c.type, c.w, c.h, 2, DEV, model=m, hr_last=state[i],
                                            hr_golden=gold[i]) for i, c in enumerate(cs)]
            ctx.enhance_streams(dc, hr, is_anchor_out=ia, **kw)
        else:
            hc = [ns.DeviceChunk.pinned_from_numpy(c.lr, c.res, c.mv, c.type, c.w, c.h, 2, model=m, hr_last=state[i],
                                                   hr_golden=gold[i]) for i, c in enumerate(cs)]
            ctx.enhance_streams_host(hc, hr, is_anchor_out=ia, **kw)
        torch.cuda.synchronize()
        outs.append((ia.cpu().numpy(), [np.stack([t.cpu().numpy() for t in row]) for row in hr],
                     [t.cpu().numpy() for t in state + gold]))
    (ia0, hr0, st0), (ia1, hr1, st1) = outs
    assert np.array_equal(ia0, ia1)
    if kw.get("selector") == ns.NS_SEL_KEY:
        assert ia0.sum() == S + 1                                 # every key frame, fewer than k
    for a, b in zip(hr0 + st0, hr1 + st1):
        assert np.array_equal(a, b)


def test_select_merge_full_size_c5_rows(ctx):
    """ns_select_merge at the scale of c5 (512 streams x 60 frames, rows from 8
    GPUs in LPT-like interleaved order, ~8% budget): bit-exact against the oracle
    merge.  Gains come from ns_select_anchors on small frames (the merge only
    sees gain / rank / type rows, whatever the resolution)."""
    S, n = 512, 60
    rng = np.random.default_rng(77)
    cs = [synth.make_chunk(20000 + s, 16, 16, 2, n, types=synth.default_types(n, int(rng.integers(8, 20))))
          for s in range(S)]
    dcs = [dev_chunk(ns, c, DEV) for c in cs]
    g, r, _ = _select_gpu(ctx, dcs, k=0)
    # gathered order: 8 ranks, rank j owns streams with s % 8 == j
    perm = [s for j in range(8) for s in range(S) if s % 8 == j]
    pt = torch.tensor(perm, device=DEV)
    g_all, r_all = g[pt].contiguous(), r[pt].contiguous()
    t_all = torch.stack([dcs[s].type for s in perm])
    cost = [1 + (s % 2) * 3 for s in perm]                  # 720p streams cost ~4x a 360p stream
    budget = int(0.08 * n * sum(cost) / 2.5)
    rank = torch.empty_like(r_all)
    anc = torch.empty_like(t_all)
    ctx.select_merge(g_all, r_all, t_all, torch.tensor(perm, dtype=torch.int32, device=DEV),
                     torch.tensor(cost, dtype=torch.int64, device=DEV), budget, rank, anc)
    torch.cuda.synchronize()
    er, ea = OS.merge_gathered(t_all.cpu().tolist(), g_all.cpu().tolist(), perm, cost, budget)
    assert anc.cpu().tolist() == ea
    assert rank.cpu().tolist() == er
    chosen = sum(c for c, row in zip(cost, ea) for v in row if v)
    assert 0 < chosen <= budget


def test_balanced_path_single_gpu_equals_given(ctx):
    """shard.balanced_sr_and_reconstruct (ns_sr_anchors + ns_reconstruct_chunk on
    the balanced anchor set) on one GPU -- no moves -- gives the frames of the
    one-call NS_GIVEN_ANCHORS path byte for byte."""
    from paper_conf_sigcomm_yeolkjyh22_b200 import shard
    S, n = 4, 10
    cs = [synth.make_chunk(9990 + s, 48, 24, 2, n, types=synth.default_types(n, 4)) for s in range(S)]
    m = ctx.model(1, 16, 2)
    m.set_weights(synth.make_weights(81, 1, 16, 2))
    anc = torch.zeros((S, n), dtype=torch.uint8, device=DEV)
    anc[:, 0] = 1
    anc[0, 4] = anc[2, 7] = anc[3, 3] = 1
    outs = []
    for path in ("given", "balanced"):
        dcs = [dev_chunk(ns, c, DEV, model=m, state=True) for c in cs]
        hr = [alloc_hr(n, c, DEV, fill=5) for c in cs]
        if path == "given":
            ctx.enhance_streams(dcs, hr, mode=ns.NS_GIVEN_ANCHORS, anchor_in=anc, cost=[1] * S, budget=S * n)
        else:
            anchors_all = [[f for f in range(n) if anc[s, f]] for s in range(S)]
            moves = shard.balanced_sr_and_reconstruct(ctx, dcs, {s: m for s in range(S)}, list(range(S)), anc, hr,
                                                      anchors_all, [0] * S, list(range(S)), [1] * S)
            assert moves == []
        torch.cuda.synchronize()
        outs.append([np.stack([t.cpu().numpy() for t in row]) for row in hr] +
                    [d.hr_last.cpu().numpy() for d in dcs] + [d.hr_golden.cpu().numpy() for d in dcs])
    for a, b in zip(*outs):
        assert np.array_equal(a, b)


def test_select_h26x_groups(ctx):
    """Codec neutrality (§9): H.26x chunks carry G_I / G_P / G_B frame
    groups in place of G_key / G_altref / G_normal -- an IBBPBBP... decode-order
    GOP with a second I frame; the selection equals the oracle's over the same
    three tiers, I frames first, then P by gain, then B by gain."""
    n = 30
    t = np.full(n, ns.NS_B, np.uint8)
    t[0::3] = ns.NS_P
    t[0] = t[15] = ns.NS_I
    dcs, cs = [], []
    for s in range(4):
        c = synth.make_chunk(9700 + s, 32, 16, 2, n, types=t)
        cs.append(c)
        dcs.append(dev_chunk(ns, c, DEV))
    for k in (1, 2, 5, 12, 30):
        g, r, a = (x.cpu().numpy() for x in _select_gpu(ctx, dcs, k=k))
        for s, c in enumerate(cs):
            eg, er, ea = oracle.select_topk(list(c.type), [int(v) for v in oracle.score(c.res)], k)
            assert list(g[s]) == eg and list(r[s]) == er and list(a[s]) == ea, (k, s)
            if k >= 2:
                assert a[s][0] and a[s][15]          # both I frames before any P or B


def test_invisible_altrefs(ctx):
    """NS_INVISIBLE ALTREFs (reading R12): selected and reconstructed as
    references exactly like visible ones (the oracle on the same flagged chunk),
    but the stats count and score only the displayed frames."""
    n, k = 20, 3
    m = ctx.model(1, 16, 2)
    blob = synth.make_weights(31, 1, 16, 2)
    m.set_weights(blob)
    c = synth.make_chunk(3131, 48, 24, 2, n, types=synth.default_types(n, 5), with_gt=True)
    c.type = np.where(c.type == synth.NS_ALTREF, c.type | ns.NS_INVISIBLE, c.type).astype(np.uint8)
    shown = [f for f in range(n) if not c.type[f] & ns.NS_INVISIBLE]
    assert len(shown) < n
    dc = dev_chunk(ns, c, DEV, model=m, with_gt=True, state=True)
    hr = alloc_hr(n, c, DEV)
    ia = torch.zeros((1, n), dtype=torch.uint8, device=DEV)
    st = torch.zeros((1, 8), dtype=torch.float64, device=DEV)
    ctx.enhance_streams([dc], [hr], is_anchor_out=ia, stats=st, k=k)
    torch.cuda.synchronize()
    ref = oracle.enhance_chunk(c, blob, 1, 16, k)
    assert list(ia.cpu().numpy()[0]) == ref["is_anchor"]
    got = np.stack([t.cpu().numpy() for t in hr])
    assert np.abs(got.astype(int) - ref["hr"].astype(int)).max() <= 2
    exp, _, _ = oracle.reconstruct(c, ref["is_anchor"], got, np.zeros_like(got[0]), np.zeros_like(got[0]))
    assert np.array_equal(got, exp)
    s = st.cpu().numpy()[0]
    assert s[0] == len(shown)
    d = got[shown].astype(np.float64) - c.gt[shown].astype(np.float64)
    mse = float((d * d).mean())
    assert abs(s[5] - min(100.0, 10 * np.log10(255.0 ** 2 / mse))) < 1e-6
