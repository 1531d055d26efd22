"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the method (no border maps, no filtering, no
planner): only random images, pitched embedding and the filter *coefficients that
callers pass in as inputs*.  Both sides (``oracle/`` and the CUDA path) receive
these arrays as arguments; neither imports the other.

Input recipe:
  * uniform noise: u8 U{0..255}, f32 U[0,1)  -- throughput runs (timing is
    value-independent for every filter here);
  * "structured" natural-like images: smooth gradient + axis-aligned and
    diagonal step edges + rectangles + 5 % noise -- correctness runs for the
    edge/corner filters (Sobel, Harris, Bilateral);
  * seeds are fixed per config (numpy PCG64 ``default_rng(seed)``).
The paper's image sizes are 512^2 .. 4096^2 (§VI); BASELINE.json
configs fix 64^2, 2048^2, 4096^2 and 16384^2.
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "uniform_u8", "uniform_f32", "structured_f32", "structured_u8",
    "random_i16", "pitched", "binomial_row", "CONFIG_SEEDS",
]

# BASELINE.json configs[0..4] -> seeds 1..5; structured images use 7.
CONFIG_SEEDS = {"cfg1": 1, "cfg2": 2, "cfg3": 3, "cfg4": 4, "cfg5": 5, "structured": 7}


def uniform_u8(h: int, w: int, seed: int) -> np.ndarray:
    return np.random.default_rng(seed).integers(0, 256, size=(h, w), dtype=np.uint8)


def uniform_f32(h: int, w: int, seed: int) -> np.ndarray:
    return np.random.default_rng(seed).random((h, w), dtype=np.float32)


def random_i16(h: int, w: int, seed: int, lo: int = -1020, hi: int = 1020) -> np.ndarray:
    """Random int16 in [lo, hi] -- the value range of 3x3 Sobel derivatives of u8."""
    return np.random.default_rng(seed).integers(lo, hi + 1, size=(h, w), dtype=np.int16)


def structured_f32(h: int, w: int, seed: int = 7) -> np.ndarray:
    """Natural-like f32 image in [0, 1]: gradient, step edges, rectangles, 5 % noise."""
    rng = np.random.default_rng(seed)
    y, x = np.mgrid[0:h, 0:w].astype(np.float64)
    img = 0.25 * (x / max(w - 1, 1)) + 0.15 * (y / max(h - 1, 1))
    img += 0.20 * (x > 0.37 * w)                      # vertical step edge
    img += 0.15 * (y > 0.61 * h)                      # horizontal step edge
    img += 0.10 * ((x - 0.5 * w) * 0.7 + (y - 0.5 * h) > 0)   # diagonal edge
    for _ in range(max(2, (h * w) // 65536)):          # rectangles
        x0, y0 = rng.integers(0, max(w, 1)), rng.integers(0, max(h, 1))
        rw, rh = rng.integers(1, max(2, w // 6)), rng.integers(1, max(2, h // 6))
        img[y0:y0 + rh, x0:x0 + rw] += rng.uniform(-0.25, 0.25)
    img += 0.05 * rng.standard_normal((h, w))
    return np.clip(img, 0.0, 1.0).astype(np.float32)


def structured_u8(h: int, w: int, seed: int = 7) -> np.ndarray:
    return np.rint(structured_f32(h, w, seed) * 255.0).astype(np.uint8)


def pitched(img: np.ndarray, pitch: int, fill=0) -> np.ndarray:
    """Embed an (h, w) image in an (h, pitch) buffer (row stride ``pitch`` elements)."""
    h, w = img.shape
    assert pitch >= w
    buf = np.full((h, pitch), fill, dtype=img.dtype)
    buf[:, :w] = img
    return buf


def binomial_row(m: int) -> np.ndarray:
    """Row m of Pascal's triangle minus one: [1,2,1], [1,4,6,4,1], ... (integer coefficients)."""
    row = np.array([1], dtype=np.int64)
    for _ in range(m - 1):
        row = np.convolve(row, [1, 1])
    return row
