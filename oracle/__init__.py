"""CPU oracle for the NeuroScaler hot path -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
``--impl reference`` legs may import this package.  The product package
(paper_conf_sigcomm_yeolkjyh22_b200) never imports it, and it imports nothing
from the product package: the two share no code.  The only shared module is
synth/ (seeded inputs, none of the method's arithmetic).

  oracle/ns_oracle.c  score (O2), upsample (O6), warp (O7), reconstruct (O8),
                      conv3x3 / pixel shuffle / SR net in fp64 (O5)
  oracle/select.py    Alg. 1 + selection (O3, O4), pure Python

Parity status per function is listed in DESIGN.md "Oracle pins".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from . import select  # noqa: F401  (re-export)
from .select import (ALTREF, CARRY, FRESH, KEY, KEY_GAIN, NORMAL,  # noqa: F401
                     select_global, select_topk, stream_gains, stream_order)

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ns_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle/ns_oracle.c -> oracle/liboracle.so (gcc, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-o", _LIB, _SRC, "-lm"])
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        i = ctypes.c_int
        L.or_score.argtypes = [P, i, i, i, P, P]
        L.or_upsample.argtypes = [P, i, i, i, P]
        L.or_warp_plane.argtypes = [P, i, i, i, P, i, P]
        L.or_reconstruct.argtypes = [i, i, i, i, P, P, P, P, P, P, P, P, i]
        L.or_reconstruct.restype = i
        L.or_reconstruct_i420.argtypes = [i, i, i, i, P, P, P, P, P, P, P, P, i]
        L.or_filter8.argtypes = [i, i, i]
        L.or_reconstruct_i420.restype = i
        L.or_conv3x3.argtypes = [P, i, i, i, P, P, i, P]
        L.or_pixel_shuffle.argtypes = [P, i, i, i, i, P]
        L.or_blob_len.argtypes = [i, i, i]
        L.or_blob_len.restype = ctypes.c_size_t
        L.or_sr_forward.argtypes = [P, i, i, i, i, i, P, P, P]
        L.or_sr_forward.restype = i
        L.or_psnr.argtypes = [P, P, ctypes.c_size_t]
        L.or_psnr.restype = ctypes.c_double
        _lib = L
    return _lib


def _p(a: np.ndarray | None):
    if a is None:
        return None
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


def score(res: np.ndarray, res_size: np.ndarray | None = None) -> np.ndarray:
    """O2: res i16 [n][3][h][w] -> int64 [n]."""
    res = np.ascontiguousarray(res, np.int16)
    n, _, h, w = res.shape
    out = np.zeros(n, np.int64)
    rs = None if res_size is None else np.ascontiguousarray(res_size, np.uint32)
    lib().or_score(_p(res), n, h, w, _p(rs), _p(out))
    return out


def upsample(plane: np.ndarray, s: int) -> np.ndarray:
    """O6 on one plane (any integer dtype) -> int32 [s*h][s*w]."""
    a = np.ascontiguousarray(plane, np.int32)
    h, w = a.shape
    out = np.zeros((s * h, s * w), np.int32)
    lib().or_upsample(_p(a), h, w, s, _p(out))
    return out


def warp_plane(ref: np.ndarray, mv: np.ndarray, s: int) -> np.ndarray:
    """O7 on one HR plane u8 [H][W] with mv (MV_DTYPE [h/8][w/8])."""
    ref = np.ascontiguousarray(ref, np.uint8)
    mv = np.ascontiguousarray(mv)
    assert mv.dtype.itemsize == 8
    H, W = ref.shape
    out = np.zeros_like(ref)
    lib().or_warp_plane(_p(ref), H, W, s, _p(mv), mv.shape[1], _p(out))
    return out


def reconstruct(chunk, is_anchor, hr_anchor, hr_last=None, hr_golden=None, s=None):
    """O8 over one chunk.  hr_anchor: u8 [n][3][sH][sW] holding the SR output
    of the anchors (other frames ignored).  Returns (hr, hr_last, hr_golden)."""
    s = chunk.scale if s is None else s
    n, h, w = chunk.n, chunk.h, chunk.w
    hr = np.array(hr_anchor, np.uint8, copy=True, order="C")
    assert hr.shape == (n, 3, s * h, s * w)
    ia = np.ascontiguousarray(is_anchor, np.uint8)
    last = None if hr_last is None else np.array(hr_last, np.uint8, copy=True, order="C")
    gold = None if hr_golden is None else np.array(hr_golden, np.uint8, copy=True, order="C")
    rc = lib().or_reconstruct(w, h, s, n, _p(np.ascontiguousarray(chunk.lr)),
                              _p(np.ascontiguousarray(chunk.res)), _p(np.ascontiguousarray(chunk.mv)),
                              _p(np.ascontiguousarray(chunk.type)), _p(ia), _p(hr), _p(last), _p(gold),
                              int(getattr(chunk, "interp", 0)))
    if rc != 0:
        raise RuntimeError(f"or_reconstruct failed: {rc}")
    return hr, last, gold


def reconstruct_i420(chunk, is_anchor, hr_anchor, hr_last=None, hr_golden=None, s=None):
    """O8 on a YUV 4:2:0 chunk (NEXT-2, reading R9).  hr_anchor: u8 [n][s*h*s*w*3/2]
    holding the anchors' SR frames.  Returns (hr, hr_last, hr_golden)."""
    s = chunk.scale if s is None else s
    n, h, w = chunk.n, chunk.h, chunk.w
    hr = np.array(hr_anchor, np.uint8, copy=True, order="C")
    assert hr.shape == (n, s * h * s * w * 3 // 2)
    ia = np.ascontiguousarray(is_anchor, np.uint8)
    last = None if hr_last is None else np.array(hr_last, np.uint8, copy=True, order="C")
    gold = None if hr_golden is None else np.array(hr_golden, np.uint8, copy=True, order="C")
    rc = lib().or_reconstruct_i420(w, h, s, n, _p(np.ascontiguousarray(chunk.lr)),
                                   _p(np.ascontiguousarray(chunk.res)), _p(np.ascontiguousarray(chunk.mv)),
                                   _p(np.ascontiguousarray(chunk.type)), _p(ia), _p(hr), _p(last), _p(gold),
                                   int(getattr(chunk, "interp", 0)))
    if rc != 0:
        raise RuntimeError(f"or_reconstruct_i420 failed: {rc}")
    return hr, last, gold


def filter8(kernel: int) -> np.ndarray:
    """The oracle's 8-tap table of one kernel (0 regular, 1 smooth, 2 sharp): int [16][8]."""
    return np.array([[lib().or_filter8(kernel, p, t) for t in range(8)] for p in range(16)], np.int64)


def i420_planes(flat: np.ndarray, h: int, w: int):
    """Flat 4:2:0 frame -> (Y [h][w], U [h/2][w/2], V [h/2][w/2]) views."""
    P = h * w
    return flat[:P].reshape(h, w), flat[P:P + P // 4].reshape(h // 2, w // 2), flat[P + P // 4:].reshape(h // 2, w // 2)


def sr_forward_i420(lr_flat: np.ndarray, blob, B: int, C: int, s: int, h: int, w: int) -> np.ndarray:
    """SR of a 4:2:0 anchor (reading R10): the 4:4:4 net (O5) on (Y, up_2(U),
    up_2(V)) -- chroma brought to luma resolution with the O6 upsample -- then
    the HR chroma planes back to 4:2:0 by the rounded 2x2 average
    floor((a + b + c + d + 2) / 4).  Returns the flat HR 4:2:0 frame."""
    y, u, v = i420_planes(np.asarray(lr_flat), h, w)
    full = np.stack([y, upsample(u, 2), upsample(v, 2)]).astype(np.uint8)
    hr = sr_forward(full, blob, B, C, s).astype(np.int64)
    cs = (hr[1:, 0::2, 0::2] + hr[1:, 1::2, 0::2] + hr[1:, 0::2, 1::2] + hr[1:, 1::2, 1::2] + 2) >> 2
    return np.concatenate([hr[0].ravel(), cs.reshape(-1)]).astype(np.uint8)


def conv3x3(x: np.ndarray, wt: np.ndarray, bias: np.ndarray | None) -> np.ndarray:
    """fp64 conv, x [Cin][h][w], wt [Cout][Cin][3][3]."""
    x = np.ascontiguousarray(x, np.float64)
    wt = np.ascontiguousarray(wt, np.float64)
    cin, h, w = x.shape
    cout = wt.shape[0]
    out = np.zeros((cout, h, w), np.float64)
    b = None if bias is None else np.ascontiguousarray(bias, np.float64)
    lib().or_conv3x3(_p(x), cin, h, w, _p(wt), _p(b), cout, _p(out))
    return out


def pixel_shuffle(x: np.ndarray, s: int) -> np.ndarray:
    x = np.ascontiguousarray(x, np.float64)
    c, h, w = x.shape
    out = np.zeros((c // (s * s), s * h, s * w), np.float64)
    lib().or_pixel_shuffle(_p(x), c // (s * s), h, w, s, _p(out))
    return out


def blob_len(B: int, C: int, s: int) -> int:
    return int(lib().or_blob_len(B, C, s))


def sr_forward(lr: np.ndarray, blob: np.ndarray, B: int, C: int, s: int, want_t: bool = False):
    """O5 on one LR frame u8 [3][h][w] -> u8 [3][s*h][s*w] (and t if want_t)."""
    lr = np.ascontiguousarray(lr, np.uint8)
    blob = np.ascontiguousarray(blob, np.uint16)
    assert blob.size == blob_len(B, C, s), (blob.size, blob_len(B, C, s))
    _, h, w = lr.shape
    out = np.zeros((3, s * h, s * w), np.uint8)
    t = np.zeros((3, s * h, s * w), np.float64) if want_t else None
    rc = lib().or_sr_forward(_p(lr), h, w, B, C, s, _p(blob), _p(out), _p(t))
    if rc != 0:
        raise RuntimeError(f"or_sr_forward failed: {rc}")
    return (out, t) if want_t else out


def psnr(a: np.ndarray, b: np.ndarray) -> float:
    a = np.ascontiguousarray(a, np.uint8)
    b = np.ascontiguousarray(b, np.uint8)
    assert a.shape == b.shape
    return float(lib().or_psnr(_p(a), _p(b), a.size))


def enhance_chunk(chunk, blob, B, C, k, mode=CARRY, hr_last=None, hr_golden=None, use_res_size=False,
                  selector="neuroscaler", is_anchor=None):
    """The whole hot path for one stream-chunk: score -> gain/select (top-k;
    selector "neuroscaler" = Alg. 1, "key" / "key_uniform" = the §3 baselines
    of P:108; or a given anchor map) -> SR on anchors -> reconstruct.  Returns
    dict(gain, rank, is_anchor, hr, hr_last, hr_golden)."""
    sc = score(chunk.res, chunk.res_size if use_res_size else None)
    if is_anchor is not None:
        gain, rank, is_anchor = None, None, [int(v) for v in is_anchor]
    elif selector == "key":
        gain, rank, is_anchor = select.select_key(list(chunk.type), k)
    elif selector == "key_uniform":
        gain, rank, is_anchor = select.select_key_uniform(list(chunk.type), k)
    else:
        gain, rank, is_anchor = select_topk(list(chunk.type), [int(v) for v in sc], k, mode)
    s = chunk.scale
    hr = np.zeros((chunk.n, 3, s * chunk.h, s * chunk.w), np.uint8)
    for f in range(chunk.n):
        if is_anchor[f]:
            hr[f] = sr_forward(chunk.lr[f], blob, B, C, s)
    hr, last, gold = reconstruct(chunk, is_anchor, hr, hr_last, hr_golden)
    return dict(score=sc, gain=gain, rank=rank, is_anchor=is_anchor, hr=hr, hr_last=last, hr_golden=gold)
