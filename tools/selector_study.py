"""Selector quality study (the shape of PAPER.md Fig. 5,
P:108, and Fig. 19): PSNR of the enhanced chunk against per-frame SR (every
frame through the DNN, the paper's quality reference for reuse)
as a function of the anchor fraction, for NeuroScaler's selector (Alg. 1),
Key+Uniform and Key-only, on synthetic c2-type streams (640x360 -> x3, B8/C32,
60-frame chunks, six content profiles, random-init weights).

Everything runs through the C ABI on cuda:0 (ns_enhance_streams with
selector / k, stats against gt = the per-frame SR frames).  Synthetic content
and random weights: the absolute dB are not the paper's; the ordering of the
selectors at equal anchor fractions is what this reproduces.

  python tools/selector_study.py [--streams 6] [--out profiles/r01_selector_study.json]
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sigcomm_yeolkjyh22_b200 as ns  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--streams", type=int, default=6)
    ap.add_argument("--w", type=int, default=640)
    ap.add_argument("--h", type=int, default=360)
    ap.add_argument("--n", type=int, default=60)
    ap.add_argument("--out", default="profiles/r01_selector_study.json")
    a = ap.parse_args()
    dev = "cuda:0"
    S, n, s = a.streams, a.n, 3
    ctx = ns.Context(0, pool_bytes=24 << 30)
    chunks = [synth.make_chunk(2000 + i, a.w, a.h, s, n, profile=i % 6) for i in range(S)]
    models = []
    for i in range(S):
        m = ctx.model(8, 32, s)
        m.set_weights(synth.make_weights(3000 + i, 8, 32, s))
        models.append(m)

    def run(k, selector, gt=None):
        dcs = []
        hr = []
        for i, c in enumerate(chunks):
            st0 = torch.zeros((3, s * c.h, s * c.w), dtype=torch.uint8, device=dev)
            dc = ns.DeviceChunk.from_numpy(c.lr, c.res, c.mv, c.type, c.w, c.h, s, dev, model=models[i],
                                           hr_last=st0, hr_golden=st0.clone())
            if gt is not None:
                dc.gt = gt[i]
            dcs.append(dc)
            hr.append(torch.zeros((n, 3, s * c.h, s * c.w), dtype=torch.uint8, device=dev))
        stats = torch.zeros((S, 8), dtype=torch.float64, device=dev)
        ia = torch.zeros((S, n), dtype=torch.uint8, device=dev)
        ctx.enhance_streams(dcs, [list(h.unbind(0)) for h in hr], is_anchor_out=ia, stats=stats, k=k,
                            selector=selector)
        torch.cuda.synchronize()
        return hr, stats.cpu().numpy(), ia.cpu().numpy()

    ref, _, _ = run(n, ns.NS_SEL_NEUROSCALER)          # per-frame SR: every frame an anchor
    rows = []
    sels = [("neuroscaler", ns.NS_SEL_NEUROSCALER), ("key_uniform", ns.NS_SEL_KEY_UNIFORM)]
    for k in (1, 2, 3, 4, 5, 6, 8, 10, 12, 15):
        for name, sel in sels:
            _, st, ia = run(k, sel, gt=ref)
            rows.append(dict(selector=name, k=k, anchor_frac=float(ia.mean()), psnr_vs_per_frame=st[:, 5].tolist(),
                             mean_psnr=float(np.mean(st[:, 5]))))
    _, st, ia = run(n, ns.NS_SEL_KEY, gt=ref)
    rows.append(dict(selector="key", k=n, anchor_frac=float(ia.mean()), psnr_vs_per_frame=st[:, 5].tolist(),
                     mean_psnr=float(np.mean(st[:, 5]))))
    out = dict(workload=f"{S} streams {a.w}x{a.h} -> x{s}, B8/C32 random-init, n={n}, profiles 0..5",
               reference="per-frame SR (k = n) frames of the same streams", rows=rows)
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(out, f, indent=1)
    for r in rows:
        print(f"{r['selector']:12s} k={r['k']:3d} frac={r['anchor_frac']:.3f} psnr={r['mean_psnr']:.2f}")


if __name__ == "__main__":
    main()
