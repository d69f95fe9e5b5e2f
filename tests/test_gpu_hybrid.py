"""Hybrid encoding of the SR anchors (§6.1; SURVEY §8(f)
NEXT-3) through ns_encode_anchors: every frame gets a header (frame type; the
JPEG of the super-resolved frame for an anchor), anchors are coded at
Table 2's quality for the chunk's anchor fraction.  The decoded
anchors are checked against the HR frames they encode and against an
independent JPEG encoder (PIL/libjpeg) at the same quality."""
import io

import numpy as np
import pytest

import synth
from helpers import alloc_hr, dev_chunk, psnr

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ns = pytest.importorskip("paper_conf_sigcomm_yeolkjyh22_b200")
Image = pytest.importorskip("PIL.Image")

DEV = "cuda:0"


@pytest.fixture(scope="module")
def ctx():
    c = ns.Context(0, pool_bytes=4 << 30)
    yield c
    c.close()


def _decode(jpeg: bytes) -> np.ndarray:
    im = Image.open(io.BytesIO(jpeg))
    assert im.format == "JPEG" and im.mode == "RGB"
    return np.asarray(im).transpose(2, 0, 1).copy()      # [3][H][W], the planes in order


def _pil_jpeg(planes: np.ndarray, q: int) -> bytes:
    b = io.BytesIO()
    Image.fromarray(planes.transpose(1, 2, 0)).save(b, format="JPEG", quality=q, subsampling=0)
    return b.getvalue()


def test_hybrid_package_and_quality(ctx):
    n, k = 20, 2                                            # 10% anchors -> Table 2 quality 80
    specs = [(64, 48, 2), (48, 32, 3)]
    dcs, hrs, models = [], [], []
    for i, (w, h, s) in enumerate(specs):
        c = synth.make_chunk(7700 + i, w, h, s, n, types=synth.default_types(n, 8))
        m = ctx.model(1, 16, s)
        m.set_weights(synth.make_weights(7700 + i, 1, 16, s))
        models.append(m)
        dcs.append(dev_chunk(ns, c, DEV, model=m, state=True))
        hrs.append(alloc_hr(n, c, DEV))
    ia = torch.zeros((len(specs), n), dtype=torch.uint8, device=DEV)
    ctx.enhance_streams(dcs, hrs, is_anchor_out=ia, k=k)
    torch.cuda.synchronize()
    ia_h = ia.cpu().numpy()
    pk = ctx.encode_anchors(dcs, ia_h, hrs)
    q = ns.hybrid_quality(k, n)
    assert q == 80
    for si, pkg in enumerate(pk):
        frames = ns.parse_hybrid(pkg)
        assert [h.frame for h, _ in frames] == list(range(n))
        assert all(h.stream == si for h, _ in frames)
        for (h, payload), a in zip(frames, ia_h[si]):
            assert h.anchor == a
            if not a:
                assert h.bytes == 0 and h.quality == 0
                continue
            assert h.quality == q and h.bytes == len(payload) > 0
            hr = hrs[si][h.frame].cpu().numpy()
            dec = _decode(payload)
            assert dec.shape == hr.shape
            p_nv = psnr(dec, hr)
            ref = _pil_jpeg(hr, q)
            p_ref = psnr(_decode(ref), hr)
            print(f"stream {si} frame {h.frame}: nvjpeg {len(payload)} B {p_nv:.2f} dB, libjpeg {len(ref)} B "
                  f"{p_ref:.2f} dB")
            assert p_nv >= 30.0
            assert abs(p_nv - p_ref) <= 2.0
            assert 0.5 <= len(payload) / len(ref) <= 2.0


def test_hybrid_rejections(ctx):
    n = 10
    c = synth.make_chunk(7800, 32, 16, 2, n, types=synth.default_types(n, None))
    m = ctx.model(1, 16, 2)
    m.set_weights(synth.make_weights(1, 1, 16, 2))
    dc = dev_chunk(ns, c, DEV, model=m, state=True)
    hr = alloc_hr(n, c, DEV)
    ia = np.zeros((1, n), np.uint8)
    ia[0, :3] = 1                                           # 30% anchors: above Table 2's JPEG range
    with pytest.raises(ns.NsError) as ei:
        ctx.encode_anchors([dc], ia, [hr])
    assert ei.value.status == ns.NS_EUNSUPPORTED
    pk = ctx.encode_anchors([dc], ia, [hr], quality=70)     # an explicit quality is accepted
    assert sum(h.anchor for h, _ in ns.parse_hybrid(pk[0])) == 3
    with pytest.raises(ns.NsError) as ei:
        ctx.encode_anchors([dc], ia, [hr], quality=70, out_cap=64)
    assert ei.value.status == ns.NS_ENOMEM
