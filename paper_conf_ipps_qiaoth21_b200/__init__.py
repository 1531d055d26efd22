"""B200-native image border handling via iteration space partitioning (ISP).

Thin Python binding over the C ABI in ``include/isp.h`` (``libisp.so``, hand-written
sm_100a kernels).  Argument marshalling only: every step of the hot path runs in the
library's CUDA kernels.  PyTorch provides device memory and streams.  There is no
CPU fallback: if ``libisp.so`` is missing the import fails loudly.

Paper: Qiao, Teich, Hannig, "An Efficient Approach for Image Border Handling on GPUs
via Iteration Space Partitioning", IPDPS 2021.

Image convention: a 2-D contiguous tensor of shape (h, pitch) holds an image of width
``w`` (default ``pitch``) with row pitch ``pitch`` elements.  Outputs are allocated as
(h, w) contiguous tensors unless ``out`` is given.
"""
from __future__ import annotations

import ctypes
import os

import torch

__all__ = [
    "CLAMP", "MIRROR", "REPEAT", "CONSTANT", "AUTO", "BLOCK", "WARP", "NAIVE", "TMA", "SPLIT", "TEX", "MODES",
    "VARIANTS",
    "lib", "IspError", "PlanInfo", "ModelParams",
    "isp_filter", "isp_filter_naive", "isp_filter_ex", "isp_filter_sep_f32", "isp_filter_u8",
    "isp_sobel_u8", "isp_laplace5_u8", "isp_harris_u8", "isp_pipeline_cfg3_u8", "isp_bilateral_f32", "isp_atrous_f32",
    "isp_night_f32", "isp_plan", "isp_model_defaults", "isp_mask_reach", "isp_plan_reach", "isp_last_plan", "isp_recent_plans", "isp_clear_plans",
    "isp_set_launch_override",
    "isp_shard_unique_id", "isp_shard_init", "isp_shard_rows", "isp_shard_schedule",
    "isp_shard_filter_f32", "isp_shard_filter_u8", "isp_shard_filter_local_f32", "isp_shard_filter_local_u8",
    "isp_shard_exchange", "isp_shard_destroy", "isp_shard_peer_open", "isp_shard_peer_filter_f32",
    "isp_shard_peer_close", "isp_shard_filter_peer_local_f32", "isp_shard_filter_peer_local_u8",
    "isp_shard_peer_handle", "isp_shard_peer_attach",
]

CLAMP, MIRROR, REPEAT, CONSTANT = 0, 1, 2, 3
MODES = {"clamp": CLAMP, "mirror": MIRROR, "repeat": REPEAT, "constant": CONSTANT}
AUTO, BLOCK, WARP, NAIVE, TMA, SPLIT, TEX = 0, 1, 2, 3, 4, 5, 6
VARIANTS = {"auto": AUTO, "block": BLOCK, "warp": WARP, "naive": NAIVE, "tma": TMA, "split": SPLIT, "tex": TEX}

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libisp.so")


class IspError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(msg)
        self.status = status


class PlanInfo(ctypes.Structure):
    _fields_ = [("bh_l", ctypes.c_int), ("bh_r", ctypes.c_int), ("bh_t", ctypes.c_int), ("bh_b", ctypes.c_int),
                ("nx", ctypes.c_int), ("ny", ctypes.c_int), ("w_l", ctypes.c_int), ("w_r", ctypes.c_int),
                ("degenerate", ctypes.c_int), ("n_block", ctypes.c_longlong * 9),
                ("n_naive", ctypes.c_double), ("n_isp", ctypes.c_double), ("r_reduced", ctypes.c_double),
                ("o_naive", ctypes.c_double), ("o_isp", ctypes.c_double), ("g", ctypes.c_double),
                ("choice", ctypes.c_int), ("tile_w", ctypes.c_int), ("tile_h", ctypes.c_int),
                ("warp_w", ctypes.c_int)]

    def as_dict(self):
        d = {k: getattr(self, k) for k, _ in self._fields_}
        d["n_block"] = list(self.n_block)
        return d


class ModelParams(ctypes.Structure):
    _fields_ = [("n_check", ctypes.c_double), ("n_kernel", ctypes.c_double), ("ipc_switch", ctypes.c_double),
                ("o_naive", ctypes.c_double), ("o_isp", ctypes.c_double), ("form", ctypes.c_int)]


class ShardOp(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int), ("peer", ctypes.c_int), ("row", ctypes.c_int), ("nrows", ctypes.c_int)]


class ShardLaunch(ctypes.Structure):
    _fields_ = [("oy0", ctypes.c_int), ("nrows", ctypes.c_int), ("ylim", ctypes.c_int), ("t_real", ctypes.c_int),
                ("b_real", ctypes.c_int), ("after_halo", ctypes.c_int)]


class ShardSched(ctypes.Structure):
    _fields_ = [("y0", ctypes.c_int), ("strip_h", ctypes.c_int), ("prev", ctypes.c_int), ("next", ctypes.c_int),
                ("n_ops", ctypes.c_int), ("n_launch", ctypes.c_int), ("ops", ShardOp * 4),
                ("launch", ShardLaunch * 3)]

    def as_dict(self):
        return dict(y0=self.y0, strip_h=self.strip_h, prev=self.prev, next=self.next,
                    ops=[(o.kind, o.peer, o.row, o.nrows) for o in self.ops[:self.n_ops]],
                    launch=[(l.oy0, l.nrows, l.ylim, l.t_real, l.b_real, l.after_halo)
                            for l in self.launch[:self.n_launch]])


_I, _P, _F, _D = ctypes.c_int, ctypes.c_void_p, ctypes.c_float, ctypes.c_double
_SIGS = {
    "isp_filter": [_P, _I, _I, _I, _P, _I, _I, _I, _F, _P],
    "isp_filter_naive": [_P, _I, _I, _I, _P, _I, _I, _I, _F, _P],
    "isp_filter_ex": [_P, _I, _I, _I, _P, _I, _I, _I, _F, _P, _I, _I, _P],
    "isp_filter_sep_f32": [_P, _I, _I, _I, _P, _I, _P, _I, _I, _F, _P, _I, _I, _P],
    "isp_filter_u8": [_P, _I, _I, _I, _P, _I, _I, ctypes.c_int32, _I, _I, _P, _I, _I, _P],
    "isp_sobel_u8": [_P, _I, _I, _I, _I, _I, _P, _P, _P, _I, _I, _P],
    "isp_laplace5_u8": [_P, _I, _I, _I, _I, _I, _P, _I, _I, _P],
    "isp_harris_u8": [_P, _P, _I, _I, _I, _I, _I, ctypes.c_int64, _P, _I, _I, _P],
    "isp_pipeline_cfg3_u8": [_P, _I, _I, _I, _I, _I, _I, ctypes.c_int64, _P, _P, _P, _P, _P, _I, _I, _P],
    "isp_bilateral_f32": [_P, _I, _I, _I, _I, _F, _F, _I, _F, _P, _I, _I, _P],
    "isp_atrous_f32": [_P, _I, _I, _I, _I, _I, _F, _I, _P, _I, _I, _P],
    "isp_night_f32": [_P, _I, _I, _I, _I, _F, _P, _P, _P, _I, _I, _P],
    "isp_plan": [_I, _I, _I, _I, _I, _I, _I, _I, _I, _P, _P],
    "isp_model_defaults": [_I, _I, _I, _I, _P],
    "isp_last_plan": [_P],
    "isp_set_launch_override": [_I, _I],
    "isp_shard_unique_id": [_P],
    "isp_shard_init": [_P, _P, _I, _I, _I],
    "isp_shard_rows": [_I, _I, _I, _P, _P],
    "isp_shard_schedule": [_I, _I, _I, _I, _I, _I, _P],
    "isp_shard_filter_f32": [_P, _P, _I, _I, _I, _I, _P, _I, _I, _I, _F, _P, _I, _I, _P, _P],
    "isp_shard_filter_u8": [_P, _P, _I, _I, _I, _I, _P, _I, _I, ctypes.c_int32, _I, _I, _P, _I, _I, _P, _P],
    "isp_shard_destroy": [_P],
    "isp_shard_filter_local_f32": [_P, _I, _I, _I, _I, _I, _I, _P, _I, _I, _I, _F, _P, _I, _I, _P],
    "isp_shard_filter_local_u8": [_P, _I, _I, _I, _I, _I, _I, _P, _I, _I, ctypes.c_int32, _I, _I, _P, _I, _I, _P],
    "isp_recent_plans": [_P, _I],
    "isp_shard_exchange": [_P, _P, _I, _I, _I, _I, _I, _I, _P],
    "isp_mask_reach": [_P, _I, _I, _I, _P],
    "isp_shard_peer_open": [_P, _P, _I, _P],
    "isp_shard_peer_filter_f32": [_P, _I, _I, _I, _P, _I, _I, _I, _F, _P, _I, _I, _P],
    "isp_shard_peer_close": [_P],
    "isp_shard_peer_handle": [_P, _P],
    "isp_shard_peer_attach": [_I, _I, _I, _P, _P, _I, _P],
    "isp_shard_filter_peer_local_f32": [_P, _P, _P, _I, _I, _I, _I, _I, _P, _I, _I, _I, _F, _P, _I, _I, _P],
    "isp_shard_filter_peer_local_u8": [_P, _P, _P, _I, _I, _I, _I, _I, _P, _I, _I, ctypes.c_int32, _I, _I, _P, _I,
                                       _I, _P],
    "isp_plan_reach": [_I, _I, _P, _I, _I, _I, _P],
}

_lib = None


def lib():
    """Load libisp.so (the CUDA path).  Raises ImportError if it is not built."""
    global _lib
    if _lib is None:
        path = os.environ.get("ISP_LIB_PATH") or LIB_PATH  # experiment builds (tools/exp_lib.py)
        if not os.path.exists(path):
            raise ImportError(f"{path} missing: run `python -m paper_conf_ipps_qiaoth21_b200.build` "
                              "(there is no CPU fallback)")
        L = ctypes.CDLL(path)
        for name, args in _SIGS.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        L.isp_last_error.restype = ctypes.c_char_p
        L.isp_status_string.restype = ctypes.c_char_p
        L.isp_status_string.argtypes = [ctypes.c_int]
        L.isp_version.restype = ctypes.c_int
        L.isp_clear_plans.restype = None
        L.isp_clear_plans.argtypes = []
        _lib = L
    return _lib


def _check(status):
    if status != 0:
        L = lib()
        raise IspError(status, f"{L.isp_status_string(status).decode()}: {L.isp_last_error().decode()}")


def _mode(m):
    return MODES[m] if isinstance(m, str) else int(m)


def _variant(v):
    return VARIANTS[v] if isinstance(v, str) else int(v)


def _img(t, dtype, name="img"):
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor")
    if t.dtype != dtype:
        raise ValueError(f"{name} must be {dtype}, got {t.dtype}")
    if t.dim() != 2 or not t.is_contiguous():
        raise ValueError(f"{name} must be a contiguous 2-D (h, pitch) tensor")
    return t


def _geom(img, w):
    h, pitch = img.shape
    w = pitch if w is None else int(w)
    if w > pitch:
        raise ValueError(f"width {w} exceeds the buffer's row pitch {pitch}")
    return w, h, pitch


def _out(out, img, w, dtype, rows=None, name="out"):
    """Caller-supplied output: right dtype, contiguous 2-D, on img's device, at least
    `rows` (default: img's) rows and w columns -- checked here because the C ABI takes
    raw pointers and cannot see the allocation."""
    rows = img.shape[0] if rows is None else rows
    if out is None:
        return torch.empty((rows, w), dtype=dtype, device=img.device)
    _img(out, dtype, name)
    if out.device != img.device:
        raise ValueError(f"{name} is on {out.device}, input on {img.device}")
    if out.shape[0] < rows or out.shape[1] < w:
        raise ValueError(f"{name} has shape {tuple(out.shape)}, needs at least ({rows}, {w})")
    return out


def _in_geom(t, w, h, name):
    if t.shape[0] < h or t.shape[1] < w:
        raise ValueError(f"{name} has shape {tuple(t.shape)}, needs at least ({h}, {w})")


def _stream(t, stream=None):
    s = stream if stream is not None else torch.cuda.current_stream(t.device)
    return ctypes.c_void_p(s.cuda_stream)


def _host(arr, ctype):
    import numpy as np
    a = np.ascontiguousarray(np.asarray(arr, dtype={ctypes.c_float: np.float32, ctypes.c_int32: np.int32}[ctype]))
    return a, a.ctypes.data_as(ctypes.c_void_p)


# ------------------------------------------------------------------------------------------
def isp_filter_ex(img, mask, border_mode, const_val=0.0, out=None, variant=AUTO, w=None, stream=None):
    """Generic f32 local operator (mask: 2-D array-like, host); see isp.h."""
    _img(img, torch.float32)
    w, h, pitch = _geom(img, w)
    out = _out(out, img, w, torch.float32)
    m, mp = _host(mask, ctypes.c_float)
    mh, mw = m.shape
    _check(lib().isp_filter_ex(img.data_ptr(), w, h, pitch, mp, mw, mh, _mode(border_mode), float(const_val),
                               out.data_ptr(), out.shape[1], _variant(variant), _stream(img, stream)))
    return out


def isp_filter(img, mask, border_mode, const_val=0.0, out=None, w=None, stream=None):
    """North-star call (variant AUTO = "isp+m")."""
    return isp_filter_ex(img, mask, border_mode, const_val, out, AUTO, w, stream)


def isp_filter_naive(img, mask, border_mode, const_val=0.0, out=None, w=None, stream=None):
    return isp_filter_ex(img, mask, border_mode, const_val, out, NAIVE, w, stream)


def isp_filter_sep_f32(img, row, col, border_mode, const_val=0.0, out=None, variant=AUTO, w=None, stream=None):
    _img(img, torch.float32)
    w, h, pitch = _geom(img, w)
    out = _out(out, img, w, torch.float32)
    r, rp = _host(row, ctypes.c_float)
    c, cp = _host(col, ctypes.c_float)
    _check(lib().isp_filter_sep_f32(img.data_ptr(), w, h, pitch, rp, r.size, cp, c.size, _mode(border_mode),
                                    float(const_val), out.data_ptr(), out.shape[1], _variant(variant),
                                    _stream(img, stream)))
    return out


def isp_filter_u8(img, mask, divisor, border_mode, const_val=0, out=None, variant=AUTO, w=None, stream=None):
    _img(img, torch.uint8)
    w, h, pitch = _geom(img, w)
    out = _out(out, img, w, torch.uint8)
    m, mp = _host(mask, ctypes.c_int32)
    mh, mw = m.shape
    _check(lib().isp_filter_u8(img.data_ptr(), w, h, pitch, mp, mw, mh, int(divisor), _mode(border_mode),
                               int(const_val), out.data_ptr(), out.shape[1], _variant(variant), _stream(img, stream)))
    return out


def isp_sobel_u8(img, border_mode, const_val=0, dx=None, dy=None, mag=None, variant=AUTO, w=None, stream=None,
                 want=("dx", "dy", "mag")):
    _img(img, torch.uint8)
    w, h, pitch = _geom(img, w)
    if dx is None and "dx" in want:
        dx = torch.empty((h, w), dtype=torch.int16, device=img.device)
    if dy is None and "dy" in want:
        dy = torch.empty((h, w), dtype=torch.int16, device=img.device)
    if mag is None and "mag" in want:
        mag = torch.empty((h, w), dtype=torch.uint8, device=img.device)
    op = next(t for t in (dx, dy, mag) if t is not None).shape[1]
    for t, dt, nm in ((dx, torch.int16, "dx"), (dy, torch.int16, "dy"), (mag, torch.uint8, "mag")):
        if t is not None:
            _out(t, img, w, dt, name=nm)
            if t.shape[1] != op:
                raise ValueError("dx, dy and mag must share out_pitch")
    ptr = lambda t: t.data_ptr() if t is not None else None  # noqa: E731
    _check(lib().isp_sobel_u8(img.data_ptr(), w, h, pitch, _mode(border_mode), int(const_val), ptr(dx), ptr(dy),
                              ptr(mag), op, _variant(variant), _stream(img, stream)))
    return dx, dy, mag


def isp_laplace5_u8(img, border_mode, const_val=0, out=None, variant=AUTO, w=None, stream=None):
    _img(img, torch.uint8)
    w, h, pitch = _geom(img, w)
    out = _out(out, img, w, torch.uint8)
    _check(lib().isp_laplace5_u8(img.data_ptr(), w, h, pitch, _mode(border_mode), int(const_val), out.data_ptr(),
                                 out.shape[1], _variant(variant), _stream(img, stream)))
    return out


def isp_harris_u8(dx, dy, border_mode, const_val=0, thr=0, out=None, variant=AUTO, w=None, stream=None):
    _img(dx, torch.int16, "dx")
    _img(dy, torch.int16, "dy")
    if dx.shape != dy.shape:
        raise ValueError("dx and dy must have the same shape")
    w, h, pitch = _geom(dx, w)
    out = _out(out, dx, w, torch.uint8)
    _check(lib().isp_harris_u8(dx.data_ptr(), dy.data_ptr(), w, h, pitch, _mode(border_mode), int(const_val),
                               int(thr), out.data_ptr(), out.shape[1], _variant(variant), _stream(dx, stream)))
    return out


def isp_pipeline_cfg3_u8(img, border_mode, const_val=0, harris_const=0, thr=0, mag=None, lap=None, harris=None,
                         dx=None, dy=None, variant=AUTO, w=None, stream=None):
    """Sobel + Laplace 5x5 + Harris in one launch (include/isp.h); dx/dy written only if given.
    Returns (mag, lap, harris)."""
    _img(img, torch.uint8)
    w, h, pitch = _geom(img, w)
    mag = _out(mag, img, w, torch.uint8)
    lap = _out(lap, img, w, torch.uint8)
    harris = _out(harris, img, w, torch.uint8)
    op = mag.shape[1]
    for t, dt in ((lap, torch.uint8), (harris, torch.uint8), (dx, torch.int16), (dy, torch.int16)):
        if t is not None:
            _out(t, img, w, dt)
            if t.shape[1] != op:
                raise ValueError("all outputs must share out_pitch")
    ptr = lambda t: t.data_ptr() if t is not None else None  # noqa: E731
    _check(lib().isp_pipeline_cfg3_u8(img.data_ptr(), w, h, pitch, _mode(border_mode), int(const_val),
                                      int(harris_const), int(thr), ptr(dx), ptr(dy), mag.data_ptr(), lap.data_ptr(),
                                      harris.data_ptr(), op, _variant(variant), _stream(img, stream)))
    return mag, lap, harris


def isp_bilateral_f32(img, win, sigma_d, sigma_r, border_mode, const_val=0.0, out=None, variant=AUTO, w=None,
                      stream=None):
    _img(img, torch.float32)
    w, h, pitch = _geom(img, w)
    out = _out(out, img, w, torch.float32)
    _check(lib().isp_bilateral_f32(img.data_ptr(), w, h, pitch, int(win), float(sigma_d), float(sigma_r),
                                   _mode(border_mode), float(const_val), out.data_ptr(), out.shape[1],
                                   _variant(variant), _stream(img, stream)))
    return out


def isp_atrous_f32(img, dilation, border_mode, const_val=0.0, tonemap=False, out=None, variant=AUTO, w=None,
                   stream=None):
    _img(img, torch.float32)
    w, h, pitch = _geom(img, w)
    out = _out(out, img, w, torch.float32)
    _check(lib().isp_atrous_f32(img.data_ptr(), w, h, pitch, int(dilation), _mode(border_mode), float(const_val),
                                int(bool(tonemap)), out.data_ptr(), out.shape[1], _variant(variant),
                                _stream(img, stream)))
    return out


def isp_night_f32(img, border_mode, const_val=0.0, out=None, variant=AUTO, w=None, stream=None):
    _img(img, torch.float32)
    w, h, pitch = _geom(img, w)
    out = _out(out, img, w, torch.float32)
    t0 = torch.empty_like(out)
    t1 = torch.empty_like(out)
    _check(lib().isp_night_f32(img.data_ptr(), w, h, pitch, _mode(border_mode), float(const_val), t0.data_ptr(),
                               t1.data_ptr(), out.data_ptr(), out.shape[1], _variant(variant), _stream(img, stream)))
    return out


# ------------------------------------------------------------------------------------------
def isp_model_defaults(filter_id, border_mode, mw=3, mh=3):
    mp = ModelParams()
    _check(lib().isp_model_defaults(int(filter_id), _mode(border_mode), int(mw), int(mh), ctypes.byref(mp)))
    return mp


def isp_plan(w, h, mw, mh, tile_w=0, tile_h=0, warp_w=0, border_mode=CLAMP, filter_id=0, params=None):
    """Pure-host planner + model (no GPU needed); returns a dict (see isp_plan_info)."""
    info = PlanInfo()
    pp = ctypes.byref(params) if params is not None else None
    _check(lib().isp_plan(int(w), int(h), int(mw), int(mh), int(tile_w), int(tile_h), int(warp_w),
                          _mode(border_mode), int(filter_id), pp, ctypes.byref(info)))
    return info.as_dict()


def isp_mask_reach(mask):
    """(left, right, top, bottom) reach of the mask's non-zero taps (reading A31)."""
    import numpy as np
    m = np.asarray(mask)
    is_int = np.issubdtype(m.dtype, np.integer)
    a, ap = _host(m, ctypes.c_int32 if is_int else ctypes.c_float)
    r = (ctypes.c_int * 4)()
    _check(lib().isp_mask_reach(ap, 2 if is_int else 3, a.shape[1], a.shape[0], r))
    return tuple(r)


def isp_plan_reach(w, h, reach, tile_w, tile_h, warp_w=0):
    r = (ctypes.c_int * 4)(*[int(x) for x in reach])
    info = PlanInfo()
    _check(lib().isp_plan_reach(int(w), int(h), r, int(tile_w), int(tile_h), int(warp_w), ctypes.byref(info)))
    return info.as_dict()


def isp_last_plan():
    info = PlanInfo()
    _check(lib().isp_last_plan(ctypes.byref(info)))
    return info.as_dict()


def isp_recent_plans(n=16):
    """The last min(n, 16) launch plans of this thread, oldest first."""
    arr = (PlanInfo * 16)()
    k = lib().isp_recent_plans(arr, min(int(n), 16))
    return [arr[i].as_dict() for i in range(k)]


def isp_clear_plans():
    lib().isp_clear_plans()


def isp_set_launch_override(warps_x=0, tile_h=0):
    _check(lib().isp_set_launch_override(int(warps_x), int(tile_h)))


# ------------------------------------------------------------------------------------------
def isp_shard_unique_id() -> bytes:
    buf = (ctypes.c_ubyte * 128)()
    _check(lib().isp_shard_unique_id(buf))
    return bytes(buf)


def isp_shard_init(uid: bytes, rank, nranks, device):
    ctx = ctypes.c_void_p()
    buf = (ctypes.c_ubyte * 128).from_buffer_copy(uid)
    _check(lib().isp_shard_init(ctypes.byref(ctx), buf, int(rank), int(nranks), int(device)))
    _CTX_RANKS[ctx.value] = (int(rank), int(nranks))
    return ctx


def isp_shard_rows(H, rank, nranks):
    y0, sh = ctypes.c_int(), ctypes.c_int()
    _check(lib().isp_shard_rows(int(H), int(rank), int(nranks), ctypes.byref(y0), ctypes.byref(sh)))
    return y0.value, sh.value


def isp_shard_schedule(H, rank, nranks, halo, hy, border_mode):
    sc = ShardSched()
    _check(lib().isp_shard_schedule(int(H), int(rank), int(nranks), int(halo), int(hy), _mode(border_mode),
                                    ctypes.byref(sc)))
    return sc.as_dict()


def _strip_rows(strip, H, halo, rank, nranks, hy):
    """Check the strip buffer holds strip_h + 2*halo rows (include/isp.h) before the C ABI
    writes halo rows into it; returns strip_h."""
    if halo < hy:
        raise ValueError(f"halo {halo} < window half-height {hy}")
    _, sh = isp_shard_rows(H, rank, nranks)
    if strip.shape[0] != sh + 2 * halo:
        raise ValueError(f"strip has {strip.shape[0]} rows, rank {rank}/{nranks} of H={H} needs "
                         f"strip_h + 2*halo = {sh + 2 * halo}")
    return sh


_CTX_RANKS = {}


def _ctx_ranks(ctx, rank, nranks):
    if rank is None or nranks is None:
        rank, nranks = _CTX_RANKS[ctx.value]
    return int(rank), int(nranks)


def isp_shard_filter_f32(ctx, strip, H, halo, mask, border_mode, const_val=0.0, out=None, variant=AUTO, w=None,
                         stream=None, comm_stream=None, rank=None, nranks=None):
    _img(strip, torch.float32, "strip")
    w, _, pitch = _geom(strip, w)
    m, mp = _host(mask, ctypes.c_float)
    mh, mw = m.shape
    rank, nranks = _ctx_ranks(ctx, rank, nranks)
    sh = _strip_rows(strip, H, halo, rank, nranks, mh // 2)
    out = _out(out, strip, w, torch.float32, rows=sh)
    cs = comm_stream if comm_stream is not None else torch.cuda.current_stream(strip.device)
    _check(lib().isp_shard_filter_f32(ctx, strip.data_ptr(), w, int(H), pitch, int(halo), mp, mw, mh,
                                      _mode(border_mode), float(const_val), out.data_ptr(), out.shape[1],
                                      _variant(variant), _stream(strip, stream), ctypes.c_void_p(cs.cuda_stream)))
    return out


def isp_shard_filter_u8(ctx, strip, H, halo, mask, divisor, border_mode, const_val=0, out=None, variant=AUTO, w=None,
                        stream=None, comm_stream=None, rank=None, nranks=None):
    _img(strip, torch.uint8, "strip")
    w, _, pitch = _geom(strip, w)
    m, mp = _host(mask, ctypes.c_int32)
    mh, mw = m.shape
    rank, nranks = _ctx_ranks(ctx, rank, nranks)
    sh = _strip_rows(strip, H, halo, rank, nranks, mh // 2)
    out = _out(out, strip, w, torch.uint8, rows=sh)
    cs = comm_stream if comm_stream is not None else torch.cuda.current_stream(strip.device)
    _check(lib().isp_shard_filter_u8(ctx, strip.data_ptr(), w, int(H), pitch, int(halo), mp, mw, mh, int(divisor),
                                     _mode(border_mode), int(const_val), out.data_ptr(), out.shape[1],
                                     _variant(variant), _stream(strip, stream), ctypes.c_void_p(cs.cuda_stream)))
    return out


def isp_shard_filter_local_f32(strip, H, halo, rank, nranks, mask, border_mode, const_val=0.0, out=None,
                               variant=AUTO, w=None, stream=None):
    """Strip launches of one rank without communication (halo rows already filled)."""
    _img(strip, torch.float32, "strip")
    w, _, pitch = _geom(strip, w)
    m, mp = _host(mask, ctypes.c_float)
    mh, mw = m.shape
    sh = _strip_rows(strip, H, halo, rank, nranks, mh // 2)
    out = _out(out, strip, w, torch.float32, rows=sh)
    _check(lib().isp_shard_filter_local_f32(strip.data_ptr(), w, int(H), pitch, int(halo), int(rank), int(nranks), mp,
                                            mw, mh, _mode(border_mode), float(const_val), out.data_ptr(),
                                            out.shape[1], _variant(variant), _stream(strip, stream)))
    return out


def isp_shard_filter_local_u8(strip, H, halo, rank, nranks, mask, divisor, border_mode, const_val=0, out=None,
                              variant=AUTO, w=None, stream=None):
    """u8 strip launches of one rank without communication (halo rows already filled)."""
    _img(strip, torch.uint8, "strip")
    w, _, pitch = _geom(strip, w)
    m, mp = _host(mask, ctypes.c_int32)
    mh, mw = m.shape
    sh = _strip_rows(strip, H, halo, rank, nranks, mh // 2)
    out = _out(out, strip, w, torch.uint8, rows=sh)
    _check(lib().isp_shard_filter_local_u8(strip.data_ptr(), w, int(H), pitch, int(halo), int(rank), int(nranks), mp,
                                           mw, mh, int(divisor), _mode(border_mode), int(const_val), out.data_ptr(),
                                           out.shape[1], _variant(variant), _stream(strip, stream)))
    return out


def isp_shard_exchange(ctx, strip, H, halo, hy, border_mode, comm_stream=None, rank=None, nranks=None):
    """Only the NCCL halo exchange of a strip buffer (include/isp.h)."""
    if not isinstance(strip, torch.Tensor) or not strip.is_cuda or strip.dim() != 2 or not strip.is_contiguous():
        raise ValueError("strip must be a contiguous 2-D CUDA tensor")
    rank, nranks = _ctx_ranks(ctx, rank, nranks)
    _strip_rows(strip, H, halo, rank, nranks, hy)
    cs = comm_stream if comm_stream is not None else torch.cuda.current_stream(strip.device)
    _check(lib().isp_shard_exchange(ctx, strip.data_ptr(), strip.element_size(), int(H), strip.shape[1], int(halo),
                                    int(hy), _mode(border_mode), ctypes.c_void_p(cs.cuda_stream)))


def _own_strip(strip, dtype, H, rank, nranks, name="strip"):
    _img(strip, dtype, name)
    _, sh = isp_shard_rows(H, rank, nranks)
    if strip.shape[0] != sh:
        raise ValueError(f"peer {name} has {strip.shape[0]} rows, rank {rank}/{nranks} of H={H} owns {sh}")
    return sh


def isp_shard_filter_peer_local_f32(own, prev, nxt, H, rank, nranks, mask, border_mode, const_val=0.0, out=None,
                                    variant=AUTO, w=None, stream=None):
    """Peer-direct strip launch (no halo rows): neighbour rows read from prev / nxt strips."""
    sh = _own_strip(own, torch.float32, H, rank, nranks)
    w, _, pitch = _geom(own, w)
    m, mp = _host(mask, ctypes.c_float)
    mh, mw = m.shape
    out = _out(out, own, w, torch.float32, rows=sh)
    ptr = lambda t: t.data_ptr() if t is not None else None  # noqa: E731
    _check(lib().isp_shard_filter_peer_local_f32(own.data_ptr(), ptr(prev), ptr(nxt), w, int(H), pitch, int(rank),
                                                 int(nranks), mp, mw, mh, _mode(border_mode), float(const_val),
                                                 out.data_ptr(), out.shape[1], _variant(variant), _stream(own, stream)))
    return out


def isp_shard_filter_peer_local_u8(own, prev, nxt, H, rank, nranks, mask, divisor, border_mode, const_val=0, out=None,
                                   variant=AUTO, w=None, stream=None):
    sh = _own_strip(own, torch.uint8, H, rank, nranks)
    w, _, pitch = _geom(own, w)
    m, mp = _host(mask, ctypes.c_int32)
    mh, mw = m.shape
    out = _out(out, own, w, torch.uint8, rows=sh)
    ptr = lambda t: t.data_ptr() if t is not None else None  # noqa: E731
    _check(lib().isp_shard_filter_peer_local_u8(own.data_ptr(), ptr(prev), ptr(nxt), w, int(H), pitch, int(rank),
                                                int(nranks), mp, mw, mh, int(divisor), _mode(border_mode),
                                                int(const_val), out.data_ptr(), out.shape[1], _variant(variant),
                                                _stream(own, stream)))
    return out


def isp_shard_peer_open(ctx, strip, ring=True):
    """Collective: map the neighbour ranks' strips (CUDA IPC); strip = own rows only."""
    pp = ctypes.c_void_p()
    _check(lib().isp_shard_peer_open(ctx, strip.data_ptr(), int(bool(ring)), ctypes.byref(pp)))
    _PEER_CTX[pp.value] = (ctx, strip)
    return pp


_PEER_CTX = {}


def isp_shard_peer_handle(strip) -> bytes:
    """72-byte CUDA IPC handle (+ offset) of a strip's allocation, for isp_shard_peer_attach."""
    buf = (ctypes.c_ubyte * 72)()
    _check(lib().isp_shard_peer_handle(strip.data_ptr(), buf))
    return bytes(buf)


def isp_shard_peer_attach(rank, nranks, strip, handles, ring=True, device=None):
    """Map the neighbour strips from every rank's handle (list of 72-byte blobs, rank order)."""
    dev_i = strip.device.index if device is None else int(device)
    blob = b"".join(handles)
    if len(blob) != 72 * int(nranks):
        raise ValueError("need one 72-byte handle per rank")
    buf = (ctypes.c_ubyte * len(blob)).from_buffer_copy(blob)
    pp = ctypes.c_void_p()
    _check(lib().isp_shard_peer_attach(int(rank), int(nranks), dev_i, strip.data_ptr(), buf, int(bool(ring)),
                                       ctypes.byref(pp)))
    _PEER_CTX[pp.value] = ((int(rank), int(nranks)), strip)
    return pp


def isp_shard_peer_filter_f32(pp, H, mask, border_mode, const_val=0.0, out=None, variant=AUTO, w=None, stream=None):
    ctx, strip = _PEER_CTX[pp.value]
    rank, nranks = ctx if isinstance(ctx, tuple) else _ctx_ranks(ctx, None, None)
    sh = _own_strip(strip, torch.float32, H, rank, nranks)
    w, _, pitch = _geom(strip, w)
    m, mp = _host(mask, ctypes.c_float)
    mh, mw = m.shape
    out = _out(out, strip, w, torch.float32, rows=sh)
    _check(lib().isp_shard_peer_filter_f32(pp, w, int(H), pitch, mp, mw, mh, _mode(border_mode), float(const_val),
                                           out.data_ptr(), out.shape[1], _variant(variant), _stream(strip, stream)))
    return out


def isp_shard_peer_close(pp):
    _PEER_CTX.pop(pp.value, None)
    _check(lib().isp_shard_peer_close(pp))


def isp_shard_destroy(ctx):
    _check(lib().isp_shard_destroy(ctx))
