"""CPU oracle for the ISP hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  It shares no code with the
CUDA path (``paper_conf_ipps_qiaoth21_b200``) and never imports it.

* ``isp_oracle.c`` -- the plain definition of every filter with a per-read border
  index function, double / exact-integer arithmetic.  Loaded through
  ctypes from ``liboracle.so`` (built by ``build_oracle()`` with gcc; also run by
  ``__graft_entry__.build()``).
* ``planner.py`` -- the paper's block-index bounds and analytic model
  (Eqs. 2-10, Listings 3 and 5), followed step by step.

Parity status of each function is listed in DESIGN.md "Oracle pins"; the ones
without an independent pin say "parity unpinned" there and in their docstring.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from concurrent.futures import ThreadPoolExecutor

import numpy as np

from . import planner  # noqa: F401  (re-export)

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "isp_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

CLAMP, MIRROR, REPEAT, CONSTANT = 0, 1, 2, 3
MODES = {"clamp": CLAMP, "mirror": MIRROR, "repeat": REPEAT, "constant": CONSTANT}


def build_oracle(force: bool = False) -> str:
    """Compile isp_oracle.c -> liboracle.so (plain gcc, -O2, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build_oracle())
        P, I, L64, D = ctypes.c_void_p, ctypes.c_int, ctypes.c_long, ctypes.c_double
        L.orc_border_index.restype = L64
        L.orc_border_index.argtypes = [I, L64, L64]
        L.orc_filter_f64.argtypes = [P, I, I, L64, P, I, I, I, D, I, I, P, P]
        L.orc_filter_u8.argtypes = [P, I, I, L64, P, I, I, ctypes.c_int32, I, I, I, I, P]
        L.orc_correlate_u8_i32.argtypes = [P, I, I, L64, P, I, I, I, I, I, I, P]
        L.orc_sobel_mag.argtypes = [P, P, L64, P]
        L.orc_harris.argtypes = [P, P, I, I, L64, I, I, ctypes.c_int64, I, I, P]
        L.orc_bilateral.argtypes = [P, I, I, L64, I, D, D, I, D, I, I, P]
        L.orc_atrous.argtypes = [P, I, I, L64, I, I, D, I, I, P]
        L.orc_tonemap.argtypes = [P, L64, P]
        for f in ("orc_filter_f64", "orc_filter_u8", "orc_correlate_u8_i32", "orc_sobel_mag",
                  "orc_harris", "orc_bilateral", "orc_atrous", "orc_tonemap"):
            getattr(L, f).restype = I
        _lib = L
    return _lib


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def _mode(m) -> int:
    return MODES[m] if isinstance(m, str) else int(m)


def _geom(img: np.ndarray, w):
    """(h, pitch) buffer -> (w, h, pitch). ``w`` defaults to the buffer width."""
    assert img.ndim == 2 and img.flags["C_CONTIGUOUS"]
    h, pitch = img.shape
    return (pitch if w is None else int(w)), h, pitch


def _rows(h, rows):
    if rows is None:
        return [(0, h)]
    if isinstance(rows, tuple):
        return [rows]
    return [(int(r), int(r) + 1) for r in rows]


def _run_rows(fn, w, h, rows, out_dtype, threads=1, n_out=1):
    """Evaluate fn(y0, y1, *outs) over a list of row ranges, optionally split over threads
    (ctypes releases the GIL, so row ranges run concurrently on separate cores)."""
    ranges = _rows(h, rows)
    tasks = []
    for (a, b) in ranges:
        if threads > 1 and b - a > threads:
            step = (b - a + threads - 1) // threads
            tasks += [(s, min(b, s + step)) for s in range(a, b, step)]
        else:
            tasks.append((a, b))
    outs = [[np.empty((b - a, w), dtype=out_dtype) for (a, b) in tasks] for _ in range(n_out)]

    def job(k):
        a, b = tasks[k]
        rc = fn(a, b, *[o[k] for o in outs])
        if rc != 0:
            raise ValueError(f"oracle rejected arguments (rc={rc})")

    if threads > 1 and len(tasks) > 1:
        with ThreadPoolExecutor(threads) as ex:
            list(ex.map(job, range(len(tasks))))
    else:
        for k in range(len(tasks)):
            job(k)
    res = [np.concatenate(o, axis=0) if len(o) > 1 else o[0] for o in outs]
    return res if n_out > 1 else res[0]


# ----------------------------------------------------------------------------------------
# Border index map
# ----------------------------------------------------------------------------------------
def border_index(mode, i: int, n: int) -> int:
    """B_mode(i, N): in-range index, or -1 meaning "the constant" (Constant pattern)."""
    return int(lib().orc_border_index(_mode(mode), int(i), int(n)))


# ----------------------------------------------------------------------------------------
# Filters (each: plain definition, per-read border map; rows = None | (y0, y1) | [rows])
# ----------------------------------------------------------------------------------------
def filter_f64(img, mask, mode, const=0.0, w=None, rows=None, threads=1, with_scale=False):
    """Generic local operator, f32 image, float mask, double accumulation (a6/a7)."""
    img = np.ascontiguousarray(img, dtype=np.float32)
    mask = np.ascontiguousarray(mask, dtype=np.float64)
    mh, mw = mask.shape
    w, h, pitch = _geom(img, w)
    L = lib()

    def fn(a, b, out, sc):
        return L.orc_filter_f64(_ptr(img), w, h, pitch, _ptr(mask), mw, mh, _mode(mode),
                                float(const), a, b, _ptr(out), _ptr(sc))

    out, sc = _run_rows(fn, w, h, rows, np.float64, threads, n_out=2)
    return (out, sc) if with_scale else out


def filter_u8(img, mask, divisor, mode, const=0, w=None, rows=None, threads=1):
    """u8 image, integer mask, sat_u8(round_half_up(acc/divisor)) (A12)."""
    img = np.ascontiguousarray(img, dtype=np.uint8)
    mask = np.ascontiguousarray(mask, dtype=np.int32)
    mh, mw = mask.shape
    w, h, pitch = _geom(img, w)
    L = lib()

    def fn(a, b, out):
        return L.orc_filter_u8(_ptr(img), w, h, pitch, _ptr(mask), mw, mh, int(divisor),
                               _mode(mode), int(const), a, b, _ptr(out))

    return _run_rows(fn, w, h, rows, np.uint8, threads)


def correlate_u8_i32(img, mask, mode, const=0, w=None, rows=None, threads=1):
    """u8 image, integer mask, raw int32 sums (Sobel derivatives, a9)."""
    img = np.ascontiguousarray(img, dtype=np.uint8)
    mask = np.ascontiguousarray(mask, dtype=np.int32)
    mh, mw = mask.shape
    w, h, pitch = _geom(img, w)
    L = lib()

    def fn(a, b, out):
        return L.orc_correlate_u8_i32(_ptr(img), w, h, pitch, _ptr(mask), mw, mh, _mode(mode),
                                      int(const), a, b, _ptr(out))

    return _run_rows(fn, w, h, rows, np.int32, threads)


SOBEL_KX = np.array([[-1, 0, 1], [-2, 0, 2], [-1, 0, 1]], dtype=np.int32)   # a9
SOBEL_KY = SOBEL_KX.T.copy()
LAPLACE5 = np.ones((5, 5), dtype=np.int32)                                     # a8
LAPLACE5[2, 2] = -24


def sobel_mag(dx, dy):
    dx = np.ascontiguousarray(dx, dtype=np.int32)
    dy = np.ascontiguousarray(dy, dtype=np.int32)
    out = np.empty(dx.shape, dtype=np.uint8)
    lib().orc_sobel_mag(_ptr(dx), _ptr(dy), dx.size, _ptr(out))
    return out


def sobel(img, mode, const=0, w=None, rows=None, threads=1):
    """Sobel application: dx, dy (int16 range) and magnitude (u8)."""
    dx = correlate_u8_i32(img, SOBEL_KX, mode, const, w, rows, threads)
    dy = correlate_u8_i32(img, SOBEL_KY, mode, const, w, rows, threads)
    return dx.astype(np.int16), dy.astype(np.int16), sobel_mag(dx, dy)


def laplace5_u8(img, mode, const=0, w=None, rows=None, threads=1):
    """Laplace 5x5 (a8): all-ones mask, centre -24, out = clamp(acc, 0, 255)."""
    return filter_u8(img, LAPLACE5, 1, mode, const, w, rows, threads)


def harris(dx, dy, mode, const=0, thr=0, w=None, rows=None, threads=1):
    """Harris response over (dx, dy) int16 (a10; not in the paper -- BASELINE configs[2])."""
    dx = np.ascontiguousarray(dx, dtype=np.int16)
    dy = np.ascontiguousarray(dy, dtype=np.int16)
    w, h, pitch = _geom(dx, w)
    L = lib()

    def fn(a, b, out):
        return L.orc_harris(_ptr(dx), _ptr(dy), w, h, pitch, _mode(mode), int(const), int(thr),
                            a, b, _ptr(out))

    return _run_rows(fn, w, h, rows, np.uint8, threads)


def bilateral(img, win, sigma_d, sigma_r, mode, const=0.0, w=None, rows=None, threads=1):
    """Bilateral filter (a11), double precision."""
    img = np.ascontiguousarray(img, dtype=np.float32)
    w, h, pitch = _geom(img, w)
    L = lib()

    def fn(a, b, out):
        return L.orc_bilateral(_ptr(img), w, h, pitch, int(win), float(sigma_d), float(sigma_r),
                               _mode(mode), float(const), a, b, _ptr(out))

    return _run_rows(fn, w, h, rows, np.float64, threads)


def atrous(img, d, mode, const=0.0, w=None, rows=None, threads=1):
    """One Atrous pass with dilation d (ref 28; a12, A26 -- coefficients ours)."""
    img = np.ascontiguousarray(img, dtype=np.float32)
    w, h, pitch = _geom(img, w)
    L = lib()

    def fn(a, b, out):
        return L.orc_atrous(_ptr(img), w, h, pitch, int(d), _mode(mode), float(const), a, b, _ptr(out))

    return _run_rows(fn, w, h, rows, np.float64, threads)


def tonemap(v):
    """Night tone map t(v) = v/(1+v) (A26; parity unpinned against the paper)."""
    v = np.ascontiguousarray(v, dtype=np.float64)
    out = np.empty_like(v)
    lib().orc_tonemap(_ptr(v), v.size, _ptr(out))
    return out


def night(img, mode, const=0.0, threads=1):
    """Night filter: Atrous with d = 1, 2, 4, 8 (windows 3, 5, 9, 17), then tone
    mapping.  Every kernel border-handles its own input; the intermediate images are f32
    images (the pipeline's pixel type), so each pass's output is rounded to f32."""
    cur = np.ascontiguousarray(img, dtype=np.float32)
    for d in (1, 2, 4, 8):
        cur = atrous(cur, d, mode, const, threads=threads).astype(np.float32)
    return tonemap(cur)


def gaussian_u8_mask(m: int):
    """Binomial u8 Gaussian (a7): integer mask b (x) b and divisor S = (sum b)^2."""
    b = np.array([1], dtype=np.int64)
    for _ in range(m - 1):
        b = np.convolve(b, [1, 1])
    return np.outer(b, b).astype(np.int32), int(b.sum() ** 2)
