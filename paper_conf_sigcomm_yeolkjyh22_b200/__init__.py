"""NeuroScaler data-parallel enhancement hot path on B200 (sm_100a).

Thin ctypes binding of libneuroscaler.so (C ABI: include/ns.h).  This module
only marshals arguments: every step of the path -- scoring, anchor selection,
SR on anchors, reuse reconstruction, stats -- runs in the library's CUDA
kernels.  PyTorch provides device memory and streams only.  There is no CPU
fallback: if the extension is missing the import of `lib()` raises.
"""
from __future__ import annotations

import ctypes
import dataclasses
import os
from typing import Optional, Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# NS_LIB: an alternative in-tree build of the same library (A/B timing of variants)
LIB_PATH = os.environ.get("NS_LIB") or os.path.join(_HERE, "libneuroscaler.so")

NS_OK, NS_EINVAL, NS_ECUDA, NS_ENOMEM, NS_EUNSUPPORTED = 0, -1, -2, -3, -4
NS_KEY, NS_ALTREF, NS_NORMAL = 0, 1, 2
NS_I, NS_P, NS_B = NS_KEY, NS_ALTREF, NS_NORMAL      # H.26x groups G_I, G_P, G_B
NS_INVISIBLE, NS_TYPE_MASK = 0x80, 0x7F               # invisible frames, reading R12
NS_REF_LAST, NS_REF_GOLDEN, NS_REF_INTRA = 0, 1, 2
NS_TOPK_PER_STREAM, NS_GLOBAL_BUDGET, NS_GIVEN_ANCHORS = 0, 1, 2
NS_CARRY, NS_FRESH = 0, 1
NS_SEL_NEUROSCALER, NS_SEL_KEY, NS_SEL_KEY_UNIFORM = 0, 1, 2
NS_FMT_444, NS_FMT_I420 = 0, 1
# sub-pel motion compensation (ns_chunk.interp; reading R13)
NS_INTERP_BILINEAR, NS_INTERP_EIGHTTAP, NS_INTERP_EIGHTTAP_SMOOTH, NS_INTERP_EIGHTTAP_SHARP, NS_INTERP_SWITCHABLE = \
    0, 1, 2, 3, 4

P = ctypes.c_void_p


class NsChunk(ctypes.Structure):
    _fields_ = [("w", ctypes.c_int32), ("h", ctypes.c_int32), ("scale", ctypes.c_int32), ("n_frames", ctypes.c_int32),
                ("lr", P), ("res", P), ("mv", P), ("type", P), ("res_size", P), ("model", P),
                ("hr_last", P), ("hr_golden", P), ("gt", P), ("format", ctypes.c_int32),
                ("interp", ctypes.c_int32)]


class NsSelectParams(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int32), ("k", ctypes.c_int32), ("budget", ctypes.c_int64), ("cost", P),
                ("group_residual", ctypes.c_int32), ("use_res_size", ctypes.c_int32),
                ("selector", ctypes.c_int32), ("reserved", ctypes.c_int32), ("anchor_in", P)]


class NsProfEntry(ctypes.Structure):
    _fields_ = [("name", ctypes.c_char * 24), ("launches", ctypes.c_uint64), ("scopes", ctypes.c_uint64),
                ("total_ms", ctypes.c_double)]


class NsSrJob(ctypes.Structure):
    _fields_ = [("model", P), ("lr", P), ("w", ctypes.c_int32), ("h", ctypes.c_int32), ("hr_out", P),
                ("format", ctypes.c_int32)]


EXPORTS = ["ns_ctx_create", "ns_ctx_destroy", "ns_model_create", "ns_model_set_weights", "ns_model_blob_len",
           "ns_model_destroy", "ns_select_anchors", "ns_select_merge", "ns_sr_anchors", "ns_reconstruct_chunk", "ns_enhance_streams",
           "ns_enhance_streams_host", "ns_launch_count", "ns_last_error", "ns_profile_enable", "ns_profile_read",
           "ns_hybrid_quality", "ns_encode_anchors"]

NS_HYBRID_MAGIC = 0x4648534E


class NsHybridHeader(ctypes.Structure):
    """ns_hybrid_header (include/ns.h): per-frame header of the hybrid package."""
    _fields_ = [("magic", ctypes.c_uint32), ("stream", ctypes.c_uint32), ("frame", ctypes.c_uint16),
                ("anchor", ctypes.c_uint8), ("quality", ctypes.c_uint8), ("bytes", ctypes.c_uint32)]

_lib = None


class NsError(RuntimeError):
    def __init__(self, status: int, where: str, msg: str):
        super().__init__(f"{where} -> {status}: {msg}")
        self.status = status


def lib() -> ctypes.CDLL:
    """Loads libneuroscaler.so (raises if it has not been built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run `python -m paper_conf_sigcomm_yeolkjyh22_b200.build`")
        L = ctypes.CDLL(LIB_PATH)
        i32 = ctypes.c_int
        L.ns_ctx_create.argtypes = [i32, ctypes.c_size_t, ctypes.POINTER(P)]
        L.ns_ctx_destroy.argtypes = [P]
        L.ns_model_create.argtypes = [P, i32, i32, i32, ctypes.POINTER(P)]
        L.ns_model_set_weights.argtypes = [P, P, ctypes.c_size_t, P]
        L.ns_model_blob_len.argtypes = [i32, i32, i32]
        L.ns_model_blob_len.restype = ctypes.c_size_t
        L.ns_model_destroy.argtypes = [P]
        L.ns_select_anchors.argtypes = [P, P, i32, ctypes.POINTER(NsSelectParams), P, P, P, P]
        L.ns_select_merge.argtypes = [P, i32, i32, P, P, P, P, P, ctypes.c_int64, P, P, P]
        L.ns_sr_anchors.argtypes = [P, P, i32, P]
        L.ns_reconstruct_chunk.argtypes = [P, P, i32, P, P, P]
        L.ns_enhance_streams.argtypes = [P, P, i32, ctypes.POINTER(NsSelectParams), P, P, P, P]
        L.ns_enhance_streams_host.argtypes = [P, P, i32, ctypes.POINTER(NsSelectParams), P, P, P,
                                              ctypes.POINTER(ctypes.c_uint64), P]
        L.ns_launch_count.argtypes = [i32]
        L.ns_launch_count.restype = ctypes.c_uint64
        L.ns_last_error.restype = ctypes.c_char_p
        L.ns_profile_enable.argtypes = [i32]
        L.ns_profile_enable.restype = i32
        L.ns_profile_read.argtypes = [P, i32]
        L.ns_profile_read.restype = i32
        L.ns_hybrid_quality.argtypes = [i32, i32]
        L.ns_hybrid_quality.restype = i32
        L.ns_encode_anchors.argtypes = [P, P, i32, P, P, i32, P, ctypes.c_size_t, P, P]
        for f in ("ns_ctx_create", "ns_ctx_destroy", "ns_model_create", "ns_model_set_weights", "ns_model_destroy",
                  "ns_select_anchors", "ns_select_merge", "ns_sr_anchors", "ns_reconstruct_chunk", "ns_enhance_streams",
                  "ns_enhance_streams_host", "ns_encode_anchors"):
            getattr(L, f).restype = i32
        _lib = L
    return _lib


def _check(rc: int, where: str):
    if rc != NS_OK:
        raise NsError(rc, where, lib().ns_last_error().decode())


def hybrid_quality(n_anchors: int, n_frames: int) -> int:
    """Table 2's JPEG quality for a chunk's anchor fraction (-1: above 10%)."""
    return int(lib().ns_hybrid_quality(n_anchors, n_frames))


def parse_hybrid(pkg: bytes):
    """Splits one stream's hybrid package into [(header, payload bytes)]."""
    out, pos, hs = [], 0, ctypes.sizeof(NsHybridHeader)
    while pos < len(pkg):
        h = NsHybridHeader.from_buffer_copy(pkg[pos:pos + hs])
        if h.magic != NS_HYBRID_MAGIC:
            raise ValueError(f"bad hybrid header magic at byte {pos}")
        out.append((h, pkg[pos + hs:pos + hs + h.bytes]))
        pos += hs + h.bytes
    return out


def last_error() -> str:
    return lib().ns_last_error().decode()


def launch_count(reset: bool = False) -> int:
    return int(lib().ns_launch_count(1 if reset else 0))


def profile_enable(on: bool = True):
    """Starts (clearing) / stops per-kernel-family event timing in the library."""
    lib().ns_profile_enable(1 if on else 0)


def profile_read() -> dict:
    """{family: (launches, groups, total_ms)} over the recorded launches (syncs)."""
    arr = (NsProfEntry * 32)()
    n = lib().ns_profile_read(arr, 32)
    if n < 0:
        raise NsError(n, "ns_profile_read", last_error())
    return {arr[i].name.decode(): (int(arr[i].launches), int(arr[i].scopes), float(arr[i].total_ms))
            for i in range(n)}


def _ptr(t) -> Optional[int]:
    if t is None:
        return None
    return int(t.data_ptr())


def _stream(stream) -> Optional[int]:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return int(stream.cuda_stream) or None


@dataclasses.dataclass
class DeviceChunk:
    """One stream's chunk in device memory (torch tensors), see ns_chunk."""
    w: int
    h: int
    scale: int
    lr: "object"              # uint8 [n,3,h,w]
    res: "object"             # int16 [n,3,h,w]
    mv: "object"              # uint8 [n,h/8,w/8,8] (ns_block_mv bytes)
    type: "object"            # uint8 [n]
    model: Optional["Model"] = None
    res_size: "object" = None  # int32/uint32 [n]
    hr_last: "object" = None   # uint8 [3,sH,sW]
    hr_golden: "object" = None
    gt: "object" = None        # uint8 [n,3,sH,sW]
    format: int = NS_FMT_444   # NS_FMT_I420: lr/res [n, h*w*3/2], HR frames s*h*s*w*3/2 bytes
    interp: int = NS_INTERP_BILINEAR  # the codec's sub-pel filter (NS_INTERP_*)

    @property
    def n(self) -> int:
        return int(self.type.shape[0])

    def to_c(self) -> NsChunk:
        return NsChunk(self.w, self.h, self.scale, self.n, _ptr(self.lr), _ptr(self.res), _ptr(self.mv),
                       _ptr(self.type), _ptr(self.res_size), self.model.handle if self.model else None,
                       _ptr(self.hr_last), _ptr(self.hr_golden), _ptr(self.gt), int(self.format), int(self.interp))

    @staticmethod
    def from_numpy(lr, res, mv, types, w, h, scale, device, res_size=None, gt=None, model=None,
                   hr_last=None, hr_golden=None, format=NS_FMT_444, interp=NS_INTERP_BILINEAR) -> "DeviceChunk":
        """Copies host arrays (mv as a structured or raw 8-byte array) to `device`."""
        import torch
        mvb = np.ascontiguousarray(mv).view(np.uint8).reshape(mv.shape[0], h // 8, w // 8, 8)
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).to(device)
        rs = None if res_size is None else t(np.asarray(res_size).astype(np.int32))
        return DeviceChunk(w=w, h=h, scale=scale, lr=t(lr), res=t(res), mv=t(mvb), type=t(np.asarray(types, np.uint8)),
                           model=model, res_size=rs, gt=None if gt is None else t(gt),
                           hr_last=hr_last, hr_golden=hr_golden, format=format, interp=interp)


    @staticmethod
    def pinned_from_numpy(lr, res, mv, types, w, h, scale, res_size=None, model=None,
                          hr_last=None, hr_golden=None, format=NS_FMT_444, interp=NS_INTERP_BILINEAR) -> "DeviceChunk":
        """Host chunk for ns_enhance_streams_host: inputs in page-locked host
        memory (torch pinned tensors); hr_last / hr_golden stay on the device."""
        import torch
        mvb = np.ascontiguousarray(mv).view(np.uint8).reshape(mv.shape[0], h // 8, w // 8, 8)
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory()
        rs = None if res_size is None else t(np.asarray(res_size).astype(np.int32))
        return DeviceChunk(w=w, h=h, scale=scale, lr=t(lr), res=t(res), mv=t(mvb), type=t(np.asarray(types, np.uint8)),
                           model=model, res_size=rs, hr_last=hr_last, hr_golden=hr_golden, format=format,
                           interp=interp)


class Model:
    """A model slot (ns_model): shape-specialised kernels, runtime weights."""

    def __init__(self, ctx: "Context", n_blocks: int, n_ch: int, scale: int):
        h = P()
        _check(lib().ns_model_create(ctx.handle, n_blocks, n_ch, scale, ctypes.byref(h)), "ns_model_create")
        self.ctx, self.handle = ctx, h.value
        self.n_blocks, self.n_ch, self.scale = n_blocks, n_ch, scale

    @staticmethod
    def blob_len(n_blocks: int, n_ch: int, scale: int) -> int:
        return int(lib().ns_model_blob_len(n_blocks, n_ch, scale))

    def set_weights(self, blob, stream=None):
        """blob: uint16 bf16 bit patterns, numpy (host) or torch tensor (host/device)."""
        if isinstance(blob, np.ndarray):
            blob = np.ascontiguousarray(blob, np.uint16)
            _check(lib().ns_model_set_weights(self.handle, blob.ctypes.data, blob.size, _stream(stream)),
                   "ns_model_set_weights")
        else:
            _check(lib().ns_model_set_weights(self.handle, _ptr(blob), blob.numel(), _stream(stream)),
                   "ns_model_set_weights")


def _params(mode=NS_TOPK_PER_STREAM, k=0, budget=0, cost=None, fresh=False, use_res_size=False,
            selector=NS_SEL_NEUROSCALER, anchor_in=None):
    p = NsSelectParams()
    p.mode, p.k, p.budget = mode, k, budget
    p.selector = selector
    p.anchor_in = _ptr(anchor_in)
    keep = None
    if cost is not None:
        keep = np.ascontiguousarray(cost, np.int64)
        p.cost = keep.ctypes.data
    p.group_residual = NS_FRESH if fresh else NS_CARRY
    p.use_res_size = 1 if use_res_size else 0
    return p, keep


class Context:
    """ns_ctx: one device, one pre-allocated pool."""

    def __init__(self, device: int = 0, pool_bytes: int = 8 << 30):
        h = P()
        _check(lib().ns_ctx_create(device, pool_bytes, ctypes.byref(h)), "ns_ctx_create")
        self.handle, self.device = h.value, device

    def close(self):
        if self.handle:
            _check(lib().ns_ctx_destroy(self.handle), "ns_ctx_destroy")
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def model(self, n_blocks: int, n_ch: int, scale: int) -> Model:
        return Model(self, n_blocks, n_ch, scale)

    @staticmethod
    def _chunks(chunks: Sequence[DeviceChunk]):
        arr = (NsChunk * len(chunks))(*[c.to_c() for c in chunks])
        return arr

    def select_anchors(self, chunks, gain, rank, is_anchor, stream=None, **kw):
        arr = self._chunks(chunks)
        p, keep = _params(**kw)
        _check(lib().ns_select_anchors(self.handle, arr, len(chunks), ctypes.byref(p), _ptr(gain), _ptr(rank),
                                       _ptr(is_anchor), _stream(stream)), "ns_select_anchors")
        del keep

    def select_merge(self, gain, rank_in, type_, sid, cost, budget, rank, is_anchor, stream=None):
        """ns_select_merge: global selection over streams gathered from every
        GPU (device tensors: gain i64 / rank_in i32 / type u8 [S, n], sid i32
        [S], cost i64 [S]; outputs rank i32 / is_anchor u8 [S, n])."""
        S, n = int(gain.shape[0]), int(gain.shape[1])
        _check(lib().ns_select_merge(self.handle, S, n, _ptr(gain), _ptr(rank_in), _ptr(type_), _ptr(sid), _ptr(cost),
                                     int(budget), _ptr(rank), _ptr(is_anchor), _stream(stream)), "ns_select_merge")

    def sr_anchors(self, jobs, stream=None):
        """jobs: list of (model, lr [3,h,w] u8 tensor, hr_out [3,sh,sw] u8 tensor), or
        (model, lr, hr_out, w, h, format) for a 4:2:0 frame (flat tensors)."""
        arr = (NsSrJob * len(jobs))()
        for i, job in enumerate(jobs):
            if len(job) == 3:
                m, lr, hr = job
                w, h, fmt = int(lr.shape[-1]), int(lr.shape[-2]), NS_FMT_444
            else:
                m, lr, hr, w, h, fmt = job
            arr[i] = NsSrJob(m.handle, _ptr(lr), int(w), int(h), _ptr(hr), int(fmt))
        _check(lib().ns_sr_anchors(self.handle, arr, len(jobs), _stream(stream)), "ns_sr_anchors")

    @staticmethod
    def _hr_table(hr_out):
        flat = [_ptr(t) for row in hr_out for t in row]
        return (ctypes.c_void_p * len(flat))(*flat)

    def reconstruct_chunk(self, chunks, is_anchor, hr_out, stream=None):
        arr = self._chunks(chunks)
        tab = self._hr_table(hr_out)
        _check(lib().ns_reconstruct_chunk(self.handle, arr, len(chunks), _ptr(is_anchor), tab, _stream(stream)),
               "ns_reconstruct_chunk")

    def enhance_streams(self, chunks, hr_out, is_anchor_out=None, stats=None, stream=None, **kw):
        arr = self._chunks(chunks)
        tab = self._hr_table(hr_out)
        p, keep = _params(**kw)
        _check(lib().ns_enhance_streams(self.handle, arr, len(chunks), ctypes.byref(p), tab, _ptr(is_anchor_out),
                                        _ptr(stats), _stream(stream)), "ns_enhance_streams")
        del keep

    def enhance_streams_host(self, chunks, hr_out, is_anchor_out=None, stats=None, stream=None, **kw) -> int:
        """ns_enhance_streams_host: chunks' inputs in pinned host memory
        (DeviceChunk.pinned_from_numpy); returns the host->device bytes moved."""
        arr = self._chunks(chunks)
        tab = self._hr_table(hr_out)
        p, keep = _params(**kw)
        moved = ctypes.c_uint64(0)
        _check(lib().ns_enhance_streams_host(self.handle, arr, len(chunks), ctypes.byref(p), tab,
                                             _ptr(is_anchor_out), _ptr(stats), ctypes.byref(moved), _stream(stream)),
               "ns_enhance_streams_host")
        del keep
        return int(moved.value)

    def encode_anchors(self, chunks, is_anchor, hr_out, quality=0, out_cap=None, stream=None):
        """ns_encode_anchors (§6.1 hybrid encoding): JPEG of every anchor +
        per-frame headers.  is_anchor: [S, n] array-like (host copy is made);
        hr_out as for enhance_streams.  Returns a list of S `bytes` packages.
        The host buffer starts at a quarter of the anchors' raw size and is
        grown to the size the library reports if that is too small."""
        arr = self._chunks(chunks)
        tab = self._hr_table(hr_out)
        ia = np.ascontiguousarray(np.asarray(is_anchor, dtype=np.uint8))
        S = len(chunks)
        hdr = ctypes.sizeof(NsHybridHeader)
        grow = out_cap is None
        if out_cap is None:
            raw = sum(int(ia[i].sum()) * (3 if c.format == NS_FMT_444 else 1.5) * (c.scale * c.h) * (c.scale * c.w)
                      for i, c in enumerate(chunks))
            out_cap = int(raw // 4) + hdr * S * int(ia.shape[1]) + (1 << 16)
        lens = (ctypes.c_size_t * S)()
        for attempt in range(2):
            buf = np.empty(max(out_cap, 1), np.uint8)
            rc = lib().ns_encode_anchors(self.handle, arr, S, ia.ctypes.data, tab, int(quality), buf.ctypes.data,
                                         out_cap, lens, _stream(stream))
            if rc == NS_ENOMEM and grow and attempt == 0 and sum(lens) > out_cap:
                out_cap = int(sum(lens)) + (1 << 16)
                continue
            _check(rc, "ns_encode_anchors")
            break
        out, pos = [], 0
        for s in range(S):
            out.append(buf[pos:pos + lens[s]].tobytes())
            pos += lens[s]
        return out

    @staticmethod
    def host_pool_bytes(w: int, h: int, n: int, k: int, streams: int) -> int:
        """Pool bytes ns_enhance_streams_host carves on first use (two input
        staging buffers of one ~S/8-stream group + the anchors' LR staging)."""
        a = lambda v: (v + 255) // 256 * 256
        g = int(os.environ.get("NS_HOST_GROUPS", "0")) or 8
        gs = max(1, (streams + g - 1) // g)
        px = h * w
        per = a(n * 3 * px * 2) + a(n * (px // 64) * 8) + a(n) + a(n * 4)
        return 2 * gs * per + gs * k * a(3 * px) + (1 << 20)
