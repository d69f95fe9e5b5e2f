"""Shared helpers for the GPU parity tests: moving synth chunks to the device,
allocating HR outputs, and crop-based oracle SR sampling for full-size frames."""
from __future__ import annotations

import numpy as np

import oracle
import synth


def dev_chunk(ns, c: "synth.Chunk", device, model=None, with_gt=False, res_size=False, state=False):
    import torch
    hr_last = hr_golden = None
    if state:
        hr_last = torch.zeros((3, c.scale * c.h, c.scale * c.w), dtype=torch.uint8, device=device)
        hr_golden = torch.zeros_like(hr_last)
    return ns.DeviceChunk.from_numpy(c.lr, c.res, c.mv, c.type, c.w, c.h, c.scale, device,
                                     res_size=c.res_size if res_size else None,
                                     gt=c.gt if with_gt else None, model=model,
                                     hr_last=hr_last, hr_golden=hr_golden, interp=getattr(c, "interp", 0))


def alloc_hr(n, c, device, fill=0):
    import torch
    return [torch.full((3, c.scale * c.h, c.scale * c.w), fill, dtype=torch.uint8, device=device) for _ in range(n)]


def sr_receptive_radius(B: int) -> int:
    """LR pixels of context an SR output needs: head + 2B body + end + up convs
    (radius 1 each), the HR tail (1 HR px -> 1 LR px) and the bilinear skip."""
    return 2 * B + 3 + 2


def oracle_sr_crops(lr: np.ndarray, blob, B, C, s, windows):
    """Oracle SR evaluated on LR crops with enough halo that the window interior
    is exact.  windows: list of (y0, x0, hh, ww) in LR pixels.  Returns a list of
    ((Y0, X0, HH, WW), hr_patch) in HR pixels."""
    _, h, w = lr.shape
    R = sr_receptive_radius(B)
    out = []
    for (y0, x0, hh, ww) in windows:
        cy0, cx0 = max(0, y0 - R), max(0, x0 - R)
        cy1, cx1 = min(h, y0 + hh + R), min(w, x0 + ww + R)
        # crop dims must stay multiples of 8 only for the GPU; the oracle takes any size
        crop = np.ascontiguousarray(lr[:, cy0:cy1, cx0:cx1])
        hr = oracle.sr_forward(crop, blob, B, C, s)
        oy, ox = (y0 - cy0) * s, (x0 - cx0) * s
        out.append(((y0 * s, x0 * s, hh * s, ww * s), hr[:, oy:oy + hh * s, ox:ox + ww * s]))
    return out


def psnr(a: np.ndarray, b: np.ndarray) -> float:
    d = a.astype(np.float64) - b.astype(np.float64)
    mse = float((d * d).mean())
    return 100.0 if mse == 0 else min(100.0, 10 * np.log10(255.0 ** 2 / mse))
