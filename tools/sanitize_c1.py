"""Config-1 workload for compute-sanitizer (racecheck / synccheck /
memcheck on c1): the whole path (ns_enhance_streams) plus ns_sr_anchors at a
multi-strip size and ns_reconstruct_chunk at s = 2, 3, 4, all through the C
ABI.  Checks the results against the oracle so a sanitizer run also proves the
instrumented kernels still compute the right thing.

  compute-sanitizer --tool racecheck python tools/sanitize_c1.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_sigcomm_yeolkjyh22_b200 as ns  # noqa: E402
import synth  # noqa: E402


def main():
    dev = "cuda:0"
    cfg = synth.CONFIGS[1]
    B, C, s, n, k = cfg["n_blocks"], cfg["n_ch"], cfg["scale"], cfg["n"], cfg["k"]
    ctx = ns.Context(0, pool_bytes=3 << 30)
    # whole path, c1
    c = synth.make_chunk(1001, cfg["w"], cfg["h"], s, n, types=synth.default_types(n, None))
    blob = synth.make_weights(1001, B, C, s)
    m = ctx.model(B, C, s)
    m.set_weights(blob)
    dc = ns.DeviceChunk.from_numpy(c.lr, c.res, c.mv, c.type, c.w, c.h, s, dev, model=m)
    hr = [torch.zeros((3, s * c.h, s * c.w), dtype=torch.uint8, device=dev) for _ in range(n)]
    ia = torch.zeros((1, n), dtype=torch.uint8, device=dev)
    ctx.enhance_streams([dc], [hr], is_anchor_out=ia, k=k)
    torch.cuda.synchronize()
    ref = oracle.enhance_chunk(c, blob, B, C, k)
    got = np.stack([t.cpu().numpy() for t in hr])
    d = int(np.abs(got.astype(int) - ref["hr"].astype(int)).max())
    assert list(ia.cpu().numpy()[0]) == ref["is_anchor"] and d <= 2, d
    print("c1 whole path ok, max-abs", d, flush=True)
    # 4:2:0 whole path at c1's scale (chroma up_2 in k_prep_lr, k_pack420, chroma reconstruction)
    c4 = synth.make_chunk_i420(1002, 128, 64, s, n, types=synth.default_types(n, None))
    d4 = ns.DeviceChunk.from_numpy(c4.lr, c4.res, c4.mv, c4.type, 128, 64, s, dev, model=m, format=ns.NS_FMT_I420)
    hr4 = [torch.zeros((s * 64 * s * 128 * 3 // 2,), dtype=torch.uint8, device=dev) for _ in range(n)]
    ia4 = torch.zeros((1, n), dtype=torch.uint8, device=dev)
    ctx.enhance_streams([d4], [hr4], is_anchor_out=ia4, k=k)
    torch.cuda.synchronize()
    got4 = np.stack([t.cpu().numpy() for t in hr4])
    anc4 = list(ia4.cpu().numpy()[0])
    grey = np.zeros_like(got4[0])
    assert np.array_equal(got4, oracle.reconstruct_i420(c4, anc4, got4, grey, grey)[0])
    print("c1-scale 4:2:0 whole path ok", flush=True)
    # C32 x3 SR: several res-block / rotated-conv strips and two x-tiles per CTA
    m3 = ctx.model(1, 32, 3)
    blob3 = synth.make_weights(7, 1, 32, 3)
    m3.set_weights(blob3)
    c3 = synth.make_chunk(77, 264, 256, 3, 1)
    lr = torch.from_numpy(c3.lr[0]).to(dev)
    out = torch.zeros((3, 3 * 256, 3 * 264), dtype=torch.uint8, device=dev)
    ctx.sr_anchors([(m3, lr, out)])
    torch.cuda.synchronize()
    e3 = oracle.sr_forward(c3.lr[0], blob3, 1, 32, 3)
    d3 = int(np.abs(out.cpu().numpy().astype(int) - e3.astype(int)).max())
    assert d3 <= 2, d3
    print("C32 x3 SR 264x256 ok, max-abs", d3, flush=True)
    # reconstruction at every scale
    for sc in (2, 3, 4):
        cc = synth.make_chunk(900 + sc, 64, 40, sc, 6, types=synth.default_types(6, 3))
        iav = [1, 0, 0, 0, 0, 0]
        rng = np.random.default_rng(sc)
        hra = np.zeros((6, 3, sc * 40, sc * 64), np.uint8)
        hra[0] = rng.integers(0, 256, hra[0].shape)
        exp, _, _ = oracle.reconstruct(cc, iav, hra)
        dcc = ns.DeviceChunk.from_numpy(cc.lr, cc.res, cc.mv, cc.type, cc.w, cc.h, sc, dev)
        hrt = [torch.from_numpy(hra[f]).to(dev) for f in range(6)]
        ctx.reconstruct_chunk([dcc], torch.tensor([iav], dtype=torch.uint8, device=dev), [hrt])
        torch.cuda.synchronize()
        assert all(np.array_equal(hrt[f].cpu().numpy(), exp[f]) for f in range(6)), sc
        print(f"reconstruct s={sc} ok (bit-exact)", flush=True)
    # 8-tap MC (k_recon8, per-block kernels) at every scale, 4:4:4 and 4:2:0 (chroma kernels)
    for sc in (2, 3, 4):
        for i420 in (False, True):
            mk = synth.make_chunk_i420 if i420 else synth.make_chunk
            cc = mk(950 + sc, 64, 32, sc, 5, types=synth.default_types(5, 3), interp=4 if sc != 3 else 1)
            iav = [1, 0, 0, 0, 0]
            rng = np.random.default_rng(sc)
            shape = (sc * 32 * sc * 64 * 3 // 2,) if i420 else (3, sc * 32, sc * 64)
            hra = np.zeros((5,) + shape, np.uint8)
            hra[0] = rng.integers(0, 256, shape)
            exp = (oracle.reconstruct_i420 if i420 else oracle.reconstruct)(cc, iav, hra)[0]
            dcc = ns.DeviceChunk.from_numpy(cc.lr, cc.res, cc.mv, cc.type, cc.w, cc.h, sc, dev, interp=cc.interp,
                                            format=ns.NS_FMT_I420 if i420 else ns.NS_FMT_444)
            hrt = [torch.from_numpy(hra[f]).to(dev) for f in range(5)]
            ctx.reconstruct_chunk([dcc], torch.tensor([iav], dtype=torch.uint8, device=dev), [hrt])
            torch.cuda.synchronize()
            assert all(np.array_equal(hrt[f].cpu().numpy(), exp[f]) for f in range(5)), (sc, i420)
            # the same chunk with bilinear MC (4:2:0: the chroma k_recon_step)
            if i420:
                cc.interp = 0
                exp = oracle.reconstruct_i420(cc, iav, hra)[0]
                dcc.interp = 0
                hrt = [torch.from_numpy(hra[f]).to(dev) for f in range(5)]
                ctx.reconstruct_chunk([dcc], torch.tensor([iav], dtype=torch.uint8, device=dev), [hrt])
                torch.cuda.synchronize()
                assert all(np.array_equal(hrt[f].cpu().numpy(), exp[f]) for f in range(5)), (sc, "i420 bilinear")
            print(f"8-tap reconstruct s={sc} {'i420' if i420 else '444'} ok (bit-exact)", flush=True)
    ctx.close()
    print("sanitize_c1 done")


if __name__ == "__main__":
    main()
