"""HR rings and given-anchor-map bounds (include/ns.h ns_enhance_streams;
SURVEY.md §8(b): "Rings of >= 3 entries are allowed").

A ring stream's hr_out row repeats entries (hr_out[s][f] = ring[f % R]); its
anchors are SR'd into the context's anchor cache and copied into their slot at
their own frame step, and GOLDEN is kept in hr_golden (the client
"caches [SR anchors] in memory").  After the call each slot must hold exactly
the frame a full (one buffer per frame) run writes last into it, byte for
byte, and the chunk-end state must be identical -- the reuse chain cannot tell
the difference.  The full run itself is checked against the oracle here too.
"""
import numpy as np
import pytest

import oracle
import synth
from helpers import dev_chunk

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ns = pytest.importorskip("paper_conf_sigcomm_yeolkjyh22_b200")

DEV = "cuda:0"


@pytest.fixture(scope="module")
def ctx():
    c = ns.Context(0, pool_bytes=8 << 30)
    yield c
    c.close()


def _streams(ctx, specs, n, seed0, altref=4, interp=0):
    out = []
    for i, (B, C, s, w, h) in enumerate(specs):
        types = synth.default_types(n, altref)
        if i % 2 == 1 and n > 6:
            types[n // 2] = synth.NS_KEY          # a KEY frame inside the chunk
        c = synth.make_chunk(seed0 + i, w, h, s, n, types=types, interp=interp if i % 2 == 0 else 0)
        m = ctx.model(B, C, s)
        blob = synth.make_weights(seed0 + i, B, C, s)
        m.set_weights(blob)
        out.append((c, m, blob, (B, C)))
    return out


def _state(c, rng):
    shp = (3, c.scale * c.h, c.scale * c.w)
    return (torch.from_numpy(rng.integers(0, 256, shp, dtype=np.uint8)).to(DEV),
            torch.from_numpy(rng.integers(0, 256, shp, dtype=np.uint8)).to(DEV))


def _run(ctx, streams, ring, **kw):
    """ring = 0: one HR buffer per frame; else a ring of `ring` slots per stream."""
    rng = np.random.default_rng(17)
    dcs, rows, slots = [], [], []
    for c, m, _, _ in streams:
        last, gold = _state(c, rng)
        dc = dev_chunk(ns, c, DEV, model=m)
        dc.hr_last, dc.hr_golden = last, gold
        dcs.append(dc)
        R = ring or c.n
        buf = [torch.full((3, c.scale * c.h, c.scale * c.w), 3, dtype=torch.uint8, device=DEV) for _ in range(R)]
        slots.append(buf)
        rows.append([buf[f % R] for f in range(c.n)])
    S, n = len(streams), streams[0][0].n
    ia = torch.zeros((S, n), dtype=torch.uint8, device=DEV)
    ctx.enhance_streams(dcs, rows, is_anchor_out=ia, **kw)
    torch.cuda.synchronize()
    return ([[t.cpu().numpy() for t in b] for b in slots], ia.cpu().numpy(),
            [(d.hr_last.cpu().numpy(), d.hr_golden.cpu().numpy()) for d in dcs])


@pytest.mark.parametrize("R", [2, 3, 5])
def test_ring_equals_full_table(ctx, R):
    specs = [(2, 16, 2, 64, 32), (1, 32, 3, 48, 24), (2, 16, 2, 64, 32), (1, 16, 4, 32, 16)]
    n = 13
    streams = _streams(ctx, specs, n, 8100)
    full, ia_f, st_f = _run(ctx, streams, 0, k=4)
    ring, ia_r, st_r = _run(ctx, streams, R, k=4)
    assert np.array_equal(ia_f, ia_r)
    for si in range(len(specs)):
        for r in range(R):
            f_last = max(f for f in range(n) if f % R == r)
            assert np.array_equal(ring[si][r], full[si][f_last]), (si, r, f_last)
        assert np.array_equal(st_r[si][0], st_f[si][0]), si     # hr_last
        assert np.array_equal(st_r[si][1], st_f[si][1]), si     # hr_golden


def test_ring_equals_full_table_8tap(ctx):
    """Rings with 8-tap streams (R13; k_recon8 reads the GOLDEN copies and the
    anchor-cache copies the bilinear kernel makes) next to bilinear ones."""
    specs = [(2, 16, 2, 64, 32), (1, 32, 3, 48, 24), (1, 16, 3, 48, 24), (1, 16, 4, 32, 16)]
    n, R = 13, 3
    streams = _streams(ctx, specs, n, 8300, interp=4)
    full, ia_f, st_f = _run(ctx, streams, 0, k=4)
    ring, ia_r, st_r = _run(ctx, streams, R, k=4)
    assert np.array_equal(ia_f, ia_r)
    for si, (c, m, blob, (B, C)) in enumerate(streams):
        for r in range(R):
            f_last = max(f for f in range(n) if f % R == r)
            assert np.array_equal(ring[si][r], full[si][f_last]), (si, r, f_last)
        assert np.array_equal(st_r[si][0], st_f[si][0]) and np.array_equal(st_r[si][1], st_f[si][1]), si
    # and the full run is the oracle's reconstruction from its own anchors (non-anchor frames exact)
    rng = np.random.default_rng(17)
    for si, (c, m, blob, _) in enumerate(streams):
        last, gold = (x.cpu().numpy() for x in _state(c, rng))
        got = np.stack(full[si])
        exp, _, _ = oracle.reconstruct(c, list(ia_f[si]), got, last, gold)
        assert np.array_equal(got, exp), si


def test_ring_full_table_matches_oracle(ctx):
    """The full-table run the ring is compared with is itself the oracle's
    (incoming LAST/GOLDEN state, a KEY inside the chunk, ALTREFs)."""
    specs = [(2, 16, 2, 64, 32), (1, 32, 3, 48, 24)]
    n = 13
    streams = _streams(ctx, specs, n, 8100)
    full, ia_f, st_f = _run(ctx, streams, 0, k=4)
    rng = np.random.default_rng(17)
    for si, (c, m, blob, (B, C)) in enumerate(streams):
        last, gold = _state(c, rng)
        ref = oracle.enhance_chunk(c, blob, B, C, 4, hr_last=last.cpu().numpy(), hr_golden=gold.cpu().numpy())
        assert list(ia_f[si]) == ref["is_anchor"]
        got = np.stack(full[si])
        assert np.abs(got.astype(int) - ref["hr"].astype(int)).max() <= 2
        # reuse bit-exact given the GPU's anchors and the same incoming state
        exp, elast, egold = oracle.reconstruct(c, ref["is_anchor"], got, last.cpu().numpy(), gold.cpu().numpy())
        assert np.array_equal(got, exp)
        assert np.array_equal(st_f[si][0], elast) and np.array_equal(st_f[si][1], egold)


def test_ring_global_and_given_modes(ctx):
    specs = [(1, 16, 2, 48, 24)] * 3 + [(1, 32, 3, 40, 16)] * 2
    n = 9
    streams = _streams(ctx, specs, n, 8300, altref=3)
    kw = dict(mode=ns.NS_GLOBAL_BUDGET, budget=9, cost=[1, 2, 1, 3, 1])
    full, ia_f, st_f = _run(ctx, streams, 0, **kw)
    ring, ia_r, st_r = _run(ctx, streams, 3, **kw)
    assert np.array_equal(ia_f, ia_r) and int(ia_f.sum()) > 0
    for si in range(len(specs)):
        for r in range(3):
            f_last = max(f for f in range(n) if f % 3 == r)
            assert np.array_equal(ring[si][r], full[si][f_last]), (si, r)
        assert np.array_equal(st_r[si][1], st_f[si][1])


def test_ring_rejections(ctx):
    c = synth.make_chunk(8400, 32, 16, 2, 6, types=synth.default_types(6, None))
    m = ctx.model(1, 16, 2)
    m.set_weights(synth.make_weights(1, 1, 16, 2))
    dc = dev_chunk(ns, c, DEV, model=m, state=True)
    ring = [torch.zeros((3, 32, 64), dtype=torch.uint8, device=DEV) for _ in range(3)]
    row = [ring[f % 3] for f in range(6)]
    ia = torch.zeros((1, 6), dtype=torch.uint8, device=DEV)
    # no hr_golden to keep GOLDEN in
    d2 = ns.DeviceChunk(**{**vars(dc), "hr_golden": None})
    with pytest.raises(ns.NsError, match="hr_golden") as ei:
        ctx.enhance_streams([d2], [row], is_anchor_out=ia, k=2)
    assert ei.value.status == ns.NS_EINVAL
    # quality stats need every frame after the call
    d3 = dev_chunk(ns, synth.make_chunk(8401, 32, 16, 2, 6, types=synth.default_types(6, None), with_gt=True), DEV,
                   model=m, state=True, with_gt=True)
    with pytest.raises(ns.NsError, match="gt"):
        ctx.enhance_streams([d3], [row], is_anchor_out=ia, k=2)
    # ns_reconstruct_chunk needs every anchor's SR bytes in place: no rings
    with pytest.raises(ns.NsError, match="ring"):
        ctx.reconstruct_chunk([dc], ia, [row])


def test_given_map_over_budget_is_demoted(ctx):
    """NS_GIVEN_ANCHORS with a map that breaks its budget: per SR shape group
    the anchors take job slots stream by stream, frame by frame; the ones past
    min(streams * n, budget / min cost) are demoted (is_anchor_out cleared) and
    reconstructed -- deterministically, and the output is the oracle's for the
    demoted map."""
    specs = [(1, 16, 2, 48, 24)] * 3
    n = 8
    streams = _streams(ctx, specs, n, 8500, altref=None)
    amap = np.zeros((3, n), np.uint8)
    amap[:, 0] = 1
    amap[0, [2, 5]] = 1
    amap[1, [1, 3, 6]] = 1
    amap[2, [4]] = 1                          # 9 anchors, budget 6 with unit cost -> 6 slots
    results = []
    for _ in range(2):
        rng = np.random.default_rng(5)
        dcs, rows = [], []
        for c, m, _, _ in streams:
            dc = dev_chunk(ns, c, DEV, model=m, state=True)
            dcs.append(dc)
            rows.append([torch.zeros((3, 2 * c.h, 2 * c.w), dtype=torch.uint8, device=DEV) for _ in range(n)])
        ia = torch.zeros((3, n), dtype=torch.uint8, device=DEV)
        ctx.enhance_streams(dcs, rows, is_anchor_out=ia, mode=ns.NS_GIVEN_ANCHORS,
                            anchor_in=torch.from_numpy(amap).to(DEV), cost=[1, 1, 1], budget=6)
        torch.cuda.synchronize()
        results.append((ia.cpu().numpy(), [np.stack([t.cpu().numpy() for t in r]) for r in rows]))
        del rng
    ia0, hr0 = results[0]
    exp = amap.copy()
    # stream order, frame order: stream 0 keeps 0, 2, 5; stream 1 keeps 0, 1, 3; the rest is demoted
    exp[1, 6] = 0
    exp[2, :] = 0
    assert np.array_equal(ia0, exp), ia0
    assert np.array_equal(results[1][0], ia0)
    for si, (c, m, blob, (B, C)) in enumerate(streams):
        assert np.array_equal(results[1][1][si], hr0[si])
        ref = oracle.enhance_chunk(c, blob, B, C, 0, is_anchor=list(exp[si]),
                                   hr_last=np.zeros((3, 2 * c.h, 2 * c.w), np.uint8),
                                   hr_golden=np.zeros((3, 2 * c.h, 2 * c.w), np.uint8))
        assert np.abs(hr0[si].astype(int) - ref["hr"].astype(int)).max() <= 2
