"""CPU pin of the f32 Harris decision argument (reading A33).

The kernels decide R25 > thr in f32 and fall back to f64 only for "undecided" pixels; this
test replays their arithmetic in numpy float32 (products of f32 values are exact in f64,
so each f32 operation is emulated as one f64 operation rounded to f32; an FMA's sum may
round twice, at most one extra f32 ulp, which the 5x margin of the bound absorbs) on
windows of Sobel-range derivatives, and checks against the exact integer definition
(Python / int64, independent of the oracle and of the CUDA path):

* every pixel the bound decides (|d| >= b) gets sign(d) == sign(R25 - thr), exactly;
* flat windows (all sums 0) at thr = 0 are decided (b = 0, d = 0, output 0 = [0 > 0]);
* near ties (thr = R25 - 2 .. R25 + 2) are left to the exact path unless the bound proves
  them.
Both bounds are covered: the band kernels' 1.5 * 2^-17 * t^2 (harris2p) and the tile
kernels' 2^-17 * (p + q + t^2) (harris2), each inflated by (1 + 2^-10).
"""
import numpy as np
import pytest

F32 = np.float32
C_BAND = F32(3 * 2.0 ** -18 * (1 + 2.0 ** -10))      # 1.14552676677703857421875e-05
C_TILE = F32(2.0 ** -17 * (1 + 2.0 ** -10))          # 7.6368451118469238281e-06
C_THR = F32(2.0 ** -23 * (1 + 2.0 ** -10))           # thr_bound()
W3 = np.outer([1, 2, 1], [1, 2, 1]).astype(np.int64)


def r32(x):
    return np.asarray(x, dtype=np.float64).astype(np.float32)


def mul(a, b):
    return r32(a.astype(np.float64) * b.astype(np.float64))


def add(a, b):
    return r32(a.astype(np.float64) + b.astype(np.float64))


def fma(a, b, c):
    return r32(a.astype(np.float64) * b.astype(np.float64) + c.astype(np.float64))


def windows(n, rng):
    """n 3x3 windows of (dx, dy) in the Sobel range with the structure real images give:
    random, flat, 1-D edges (dy = 0), aligned gradients (dy = +-dx, det = 0), small
    textures (R25 near 0) and extremes (+-1020)."""
    dx = rng.integers(-1020, 1021, (n, 3, 3))
    dy = rng.integers(-1020, 1021, (n, 3, 3))
    k = n // 8
    dx[:k] = 0
    dy[:k] = 0                                      # flat
    dy[k:2 * k] = 0                                 # 1-D edge
    dy[2 * k:3 * k] = dx[2 * k:3 * k]               # aligned gradient
    dy[3 * k:4 * k] = -dx[3 * k:4 * k]
    dx[4 * k:5 * k] = rng.integers(-3, 4, (k, 3, 3))
    dy[4 * k:5 * k] = rng.integers(-3, 4, (k, 3, 3))
    dx[5 * k:6 * k] = rng.choice([-1020, 1020], (k, 3, 3))
    dy[5 * k:6 * k] = rng.choice([-1020, 1020], (k, 3, 3))
    sxx = np.einsum("nij,ij->n", dx * dx, W3)
    syy = np.einsum("nij,ij->n", dy * dy, W3)
    sxy = np.einsum("nij,ij->n", dx * dy, W3)
    return sxx, syy, sxy


def r25_exact(sxx, syy, sxy):
    # int64 is exact here: |Sxx Syy| < 2^48, 25 * that < 2^53, (Sxx + Syy)^2 < 2^50
    return 25 * (sxx * syy - sxy * sxy) - (sxx + syy) ** 2


def decide(sxx, syy, sxy, thr, form):
    """The kernels' f32 sequence: returns (decided, output of the decided pixels)."""
    x, y, z = sxx.astype(F32), syy.astype(F32), sxy.astype(F32)
    assert np.all(x.astype(np.int64) == sxx) and np.all(z.astype(np.int64) == sxy)   # sums < 2^24
    thr_f = np.asarray(thr, dtype=np.float64).astype(F32)
    thr_e = mul(np.abs(thr_f), np.full_like(thr_f, C_THR))
    pp = mul(x, y)
    det = fma(-z, z, pp)
    t = add(x, y)
    tt = mul(t, t)
    R = fma(np.full_like(det, F32(25)), det, -tt)
    if form == "band":
        b = fma(tt, np.full_like(tt, C_BAND), thr_e)
    else:
        bnd = add(add(pp, mul(z, z)), tt)
        b = fma(bnd, np.full_like(bnd, C_TILE), thr_e)
    d = add(R, -thr_f)
    decided = np.abs(d) >= b
    return decided, d > 0


@pytest.mark.parametrize("form", ["band", "tile"])
def test_decided_pixels_are_exact(form):
    rng = np.random.default_rng(2024)
    sxx, syy, sxy = windows(200_000, rng)
    R = r25_exact(sxx, syy, sxy)
    n = len(R)
    cases = {
        "zero": np.zeros(n, dtype=np.int64),
        "near": R + rng.integers(-2, 3, n),
        "rel": R + (R // 1000),
        "far": rng.integers(-(10 ** 15), 10 ** 15, n),
        "pm1": rng.choice([-1, 1], n),
    }
    for name, thr in cases.items():
        decided, out = decide(sxx, syy, sxy, thr, form)
        want = R > thr
        bad = decided & (out != want)
        assert not bad.any(), (form, name, np.flatnonzero(bad)[:5])
        if name == "far":
            assert decided.mean() > 0.999, (form, decided.mean())


@pytest.mark.parametrize("form", ["band", "tile"])
def test_flat_windows_decide_in_f32(form):
    z = np.zeros(1000, dtype=np.int64)
    for thr, want in ((0, False), (-1, True), (1, False), (-(10 ** 12), True), (10 ** 12, False)):
        decided, out = decide(z, z, z, np.full(1000, thr, dtype=np.int64), form)
        assert decided.all(), (form, thr)
        assert (out == want).all(), (form, thr)


@pytest.mark.parametrize("form", ["band", "tile"])
def test_near_ties_go_to_the_exact_path(form):
    """thr within 2 of R25 with a large t^2: the f32 rounding cannot resolve them, so they
    must come out undecided (never guessed)."""
    rng = np.random.default_rng(7)
    sxx, syy, sxy = windows(50_000, rng)
    R = r25_exact(sxx, syy, sxy)
    big = (sxx + syy) ** 2 > 2 ** 40
    for off in (-1, 0, 1):
        decided, out = decide(sxx[big], syy[big], sxy[big], R[big] + off, form)
        assert not decided.any(), (form, off)
