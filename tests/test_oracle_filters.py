"""Pins for the oracle's filters (oracle/isp_oracle.c) against things other than itself.

Every check here uses an independent path: numpy.pad + explicit shifted-slice window
sums, scipy.ndimage.correlate, exact closed forms, invariants from the paper (Eq. 1's
body region), and special cases reducing to textbook filters.
"Oracle pins" for the list and the passage each follows.
"""
import math

import numpy as np
import pytest
import scipy.ndimage as ndi

import synth

NP_MODE = {"clamp": "edge", "mirror": "symmetric", "repeat": "wrap", "constant": "constant"}
NDI_MODE = {"clamp": "nearest", "mirror": "reflect", "repeat": "grid-wrap", "constant": "constant"}
MODES = ["clamp", "mirror", "repeat", "constant"]


def pad_correlate(img, mask, mode, C):
    """Independent path: pad the image with np.pad (the padding approach), then an
    explicit sum of shifted slices (correlation, A9) in float64 / int64."""
    n, m = mask.shape
    hy, hx = n // 2, m // 2
    kw = {"constant_values": C} if mode == "constant" else {}
    acc_t = np.int64 if np.issubdtype(mask.dtype, np.integer) else np.float64
    P = np.pad(img.astype(acc_t), ((hy, hy), (hx, hx)), mode=NP_MODE[mode], **kw)
    h, w = img.shape
    out = np.zeros((h, w), dtype=acc_t)
    for j in range(n):
        for i in range(m):
            out += mask[j, i].astype(acc_t) * P[j:j + h, i:i + w]
    return out


# ---------------------------------------------------------------- generic f32 local operator
@pytest.mark.parametrize("mode", MODES)
def test_filter_f64_tiny_bruteforce(orc, mode):
    rng = np.random.default_rng(11)
    for (h, w) in [(1, 1), (1, 5), (4, 1), (3, 7), (7, 3), (6, 9)]:
        for (n, m) in [(1, 1), (3, 3), (1, 5), (5, 3), (9, 9)]:   # windows larger than the image too
            img = rng.random((h, w), dtype=np.float32)
            mask = rng.standard_normal((n, m))
            got = orc.filter_f64(img, mask, mode, 0.375)
            ref = pad_correlate(img, mask, mode, 0.375)
            np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("mode", MODES)
def test_filter_f64_vs_scipy(orc, mode):
    img = synth.uniform_f32(37, 53, 3)
    mask = np.random.default_rng(5).standard_normal((7, 5))
    got = orc.filter_f64(img, mask, mode, -0.25)
    ref = ndi.correlate(img.astype(np.float64), mask, mode=NDI_MODE[mode], cval=-0.25)
    np.testing.assert_allclose(got, ref, rtol=1e-12, atol=1e-12)


def test_filter_f64_pitch_and_rows(orc):
    img = synth.uniform_f32(20, 31, 4)
    buf = synth.pitched(img, 40, fill=np.float32(np.nan))    # padding must never be read
    mask = np.random.default_rng(1).random((5, 5))
    full = orc.filter_f64(img, mask, "mirror")
    got = orc.filter_f64(buf, mask, "mirror", w=31)
    np.testing.assert_array_equal(got, full)
    np.testing.assert_array_equal(orc.filter_f64(buf, mask, "mirror", w=31, rows=(5, 9)), full[5:9])
    np.testing.assert_array_equal(orc.filter_f64(buf, mask, "mirror", w=31, rows=[0, 19]), full[[0, 19]])
    np.testing.assert_array_equal(orc.filter_f64(img, mask, "mirror", threads=3), full)


def test_body_invariance_eq1(orc):
    """Eq. (1) (reading A1): pixels with hx<=x<sx-hx, hy<=y<sy-hy need no border
    handling, so their outputs are identical under every pattern and constant."""
    img = synth.uniform_f32(24, 30, 8)
    mask = np.random.default_rng(2).random((5, 7))
    outs = [orc.filter_f64(img, mask, m, 0.9) for m in MODES] + [orc.filter_f64(img, mask, "constant", -3.0)]
    hy, hx = 2, 3
    for o in outs[1:]:
        np.testing.assert_array_equal(o[hy:-hy, hx:-hx], outs[0][hy:-hy, hx:-hx])
    assert not np.array_equal(outs[0], outs[3])     # the border does differ


@pytest.mark.parametrize("mode", MODES)
def test_constant_image_invariance(orc, mode):
    img = np.full((9, 11), 0.625, dtype=np.float32)
    mask = np.outer([1, 4, 6, 4, 1], [1, 4, 6, 4, 1]) / 256.0
    C = 0.625 if mode == "constant" else 7.0
    np.testing.assert_array_equal(orc.filter_f64(img, mask, mode, C), np.full((9, 11), 0.625))


def test_repeat_closed_form(orc):
    """Repeat == periodic tiling: filtering equals the centre crop of an unchecked
    ('valid') correlation of the 3x3-tiled image (window half-widths <= image size)."""
    img = synth.uniform_f32(6, 8, 9)
    mask = np.random.default_rng(4).random((5, 7))
    T = np.tile(img.astype(np.float64), (3, 3))
    valid = np.zeros((T.shape[0] - 4, T.shape[1] - 6))
    for j in range(5):
        for i in range(7):
            valid += mask[j, i] * T[j:j + valid.shape[0], i:i + valid.shape[1]]
    crop = valid[6 - 2:6 - 2 + 6, 8 - 3:8 - 3 + 8]
    np.testing.assert_allclose(orc.filter_f64(img, mask, "repeat"), crop, rtol=1e-12)


# ---------------------------------------------------------------- u8 integer-mask operator
def round_half_up_frac(acc, d):
    from fractions import Fraction
    return math.floor(Fraction(int(acc), int(d)) + Fraction(1, 2))


@pytest.mark.parametrize("mode", MODES)
def test_filter_u8_bruteforce(orc, mode):
    rng = np.random.default_rng(21)
    for (h, w) in [(1, 1), (2, 9), (5, 4), (8, 8)]:
        for (n, m, d) in [(3, 3, 16), (5, 5, 7), (1, 3, 3), (7, 5, 1)]:
            img = rng.integers(0, 256, (h, w), dtype=np.uint8)
            mask = rng.integers(-4, 9, (n, m)).astype(np.int32)
            got = orc.filter_u8(img, mask, d, mode, 77)
            acc = pad_correlate(img, mask, mode, 77)
            ref = np.array([[min(255, max(0, round_half_up_frac(a, d))) for a in row] for row in acc])
            np.testing.assert_array_equal(got, ref)


@pytest.mark.parametrize("m", [3, 5, 7])
@pytest.mark.parametrize("mode", MODES)
def test_u8_gaussian_separable_equals_2d(orc, m, mode):
    """Separable == 2-D (a7): the binomial mask b(x)b applied as two 1-D integer passes
    (np.pad path, exact integers, one rounding at the end) equals the 2-D oracle."""
    img = synth.uniform_u8(13, 17, 6)
    b = synth.binomial_row(m)
    mask2, S = orc.gaussian_u8_mask(m)
    assert S == int(b.sum()) ** 2
    rowp = pad_correlate(img, b[None, :].astype(np.int64), mode, 200)
    # the column pass reads the *unrounded* row-pass image with the same border map
    h, w = img.shape
    hy = m // 2
    kw = {"constant_values": 200 * int(b.sum())} if mode == "constant" else {}
    P = np.pad(rowp, ((hy, hy), (0, 0)), mode=NP_MODE[mode], **kw)
    acc = sum(int(b[j]) * P[j:j + h] for j in range(m))
    ref = np.clip((2 * acc + S) // (2 * S), 0, 255)
    np.testing.assert_array_equal(orc.filter_u8(img, mask2, S, mode, 200), ref)


@pytest.mark.parametrize("c", [0, 1, 127, 173, 255])
@pytest.mark.parametrize("m", [3, 5, 7])
def test_u8_gaussian_constant_invariance(orc, m, c):
    img = np.full((10, 12), c, dtype=np.uint8)
    mask, S = orc.gaussian_u8_mask(m)
    for mode in MODES:
        np.testing.assert_array_equal(orc.filter_u8(img, mask, S, mode, c), img)


# ---------------------------------------------------------------- Sobel, Laplace, Harris
def test_sobel_ramp_closed_form(orc):
    """In the body, I = a x + b y + c gives dx = 8a, dy = 8b (correlation, A9)."""
    y, x = np.mgrid[0:16, 0:20]
    img = (100 + 3 * x - 5 * y).astype(np.uint8)
    for mode in MODES:
        dx, dy, _ = orc.sobel(img, mode, 9)
        assert (dx[1:-1, 1:-1] == 24).all() and (dy[1:-1, 1:-1] == -40).all()


def test_sobel_constant_zero(orc):
    img = np.full((7, 9), 91, dtype=np.uint8)
    for mode in ["clamp", "mirror", "repeat"]:
        dx, dy, mag = orc.sobel(img, mode)
        assert not dx.any() and not dy.any() and not mag.any()
    dx, dy, mag = orc.sobel(img, "constant", 91)
    assert not dx.any() and not dy.any()


def test_sobel_mag_exhaustive(orc):
    """mag = min(255, round_half_up(sqrt(dx^2+dy^2))) over the whole int16 Sobel range,
    against float64 sqrt (exact enough below 2^22; ties are impossible for integers)."""
    v = np.arange(-1020, 1021, dtype=np.int32)
    dx, dy = np.meshgrid(v, v)
    got = orc.sobel_mag(dx, dy)
    ref = np.minimum(255, np.floor(np.sqrt(dx.astype(np.float64) ** 2 + dy.astype(np.float64) ** 2) + 0.5))
    np.testing.assert_array_equal(got, ref.astype(np.uint8))


@pytest.mark.parametrize("mode", MODES)
def test_sobel_bruteforce(orc, mode):
    img = synth.structured_u8(23, 29)
    dx, dy, mag = orc.sobel(img, mode, 45)
    kx = np.array([[-1, 0, 1], [-2, 0, 2], [-1, 0, 1]])
    np.testing.assert_array_equal(dx, pad_correlate(img, kx, mode, 45))
    np.testing.assert_array_equal(dy, pad_correlate(img, kx.T.copy(), mode, 45))
    ref = ndi.correlate(img.astype(np.float64), kx.astype(np.float64), mode=NDI_MODE[mode], cval=45)
    np.testing.assert_array_equal(dx, ref)


def test_laplace_closed_forms(orc):
    """Laplace 5x5 (a8): constant -> 0; I = x^2 -> 50; I = x^2 + y^2 -> 100 in the body."""
    y, x = np.mgrid[0:12, 0:14].astype(np.float32)
    lap = orc.LAPLACE5.astype(np.float64)
    o1 = orc.filter_f64(x ** 2, lap, "clamp")
    o2 = orc.filter_f64(x ** 2 + y ** 2, lap, "mirror")
    assert np.all(o1[2:-2, 2:-2] == 50.0) and np.all(o2[2:-2, 2:-2] == 100.0)
    img = np.full((9, 9), 200, dtype=np.uint8)
    for mode in ["clamp", "mirror", "repeat"]:
        assert not orc.laplace5_u8(img, mode).any()


@pytest.mark.parametrize("mode", MODES)
def test_laplace_u8_bruteforce(orc, mode):
    img = synth.structured_u8(19, 21)
    acc = pad_correlate(img, orc.LAPLACE5, mode, 30)
    np.testing.assert_array_equal(orc.laplace5_u8(img, mode, 30), np.clip(acc, 0, 255))


def harris_numpy(dx, dy, mode, C, thr):
    w = np.outer([1, 2, 1], [1, 2, 1]).astype(np.int64)
    kw = {"constant_values": C} if mode == "constant" else {}
    Px = np.pad(dx.astype(np.int64), 1, mode=NP_MODE[mode], **kw)
    Py = np.pad(dy.astype(np.int64), 1, mode=NP_MODE[mode], **kw)
    h, wd = dx.shape
    sxx = sum(w[j, i] * Px[j:j + h, i:i + wd] ** 2 for j in range(3) for i in range(3))
    syy = sum(w[j, i] * Py[j:j + h, i:i + wd] ** 2 for j in range(3) for i in range(3))
    sxy = sum(w[j, i] * Px[j:j + h, i:i + wd] * Py[j:j + h, i:i + wd] for j in range(3) for i in range(3))
    det, tr = sxx * syy - sxy * sxy, sxx + syy
    # R = det - k tr^2 with k = 0.04 = 1/25 (a10); compare 25 R > thr exactly via fractions-free ints
    return np.where(25 * det - tr * tr > thr, 255, 0).astype(np.uint8)


@pytest.mark.parametrize("mode", MODES)
def test_harris_bruteforce(orc, mode):
    dx = synth.random_i16(15, 18, 1)
    dy = synth.random_i16(15, 18, 2)
    for thr in [0, 10 ** 12, -(10 ** 12)]:
        np.testing.assert_array_equal(orc.harris(dx, dy, mode, -7, thr), harris_numpy(dx, dy, mode, -7, thr))


def test_harris_invariants(orc):
    z = np.zeros((8, 8), dtype=np.int16)
    assert not orc.harris(z, z, "clamp").any()
    img = synth.structured_u8(24, 24)
    dx, dy, _ = orc.sobel(img, "mirror")
    r = orc.harris(dx, dy, "mirror")
    dxt, dyt, _ = orc.sobel(np.ascontiguousarray(img.T), "mirror")
    np.testing.assert_array_equal(dxt, dy.T)       # transpose swaps the derivatives
    np.testing.assert_array_equal(orc.harris(dxt, dyt, "mirror"), r.T)
    assert r.any()                                  # the structured image has corners


# ---------------------------------------------------------------- Bilateral
def bilateral_numpy(img, win, sd, sr, mode, C):
    hw = win // 2
    kw = {"constant_values": C} if mode == "constant" else {}
    P = np.pad(img.astype(np.float64), hw, mode=NP_MODE[mode], **kw)
    h, w = img.shape
    I = img.astype(np.float64)
    num = np.zeros((h, w))
    den = np.zeros((h, w))
    for j in range(win):
        for i in range(win):
            q = P[j:j + h, i:i + w]
            s = math.exp(-((i - hw) ** 2 + (j - hw) ** 2) / (2 * sd * sd))
            r = np.exp(-((q - I) ** 2) / (2 * sr * sr))
            num += s * r * q
            den += s * r
    return num / den


@pytest.mark.parametrize("mode", MODES)
def test_bilateral_bruteforce(orc, mode):
    img = synth.structured_f32(14, 17)
    got = orc.bilateral(img, 5, 1.0, 0.1, mode, 0.5)
    np.testing.assert_allclose(got, bilateral_numpy(img, 5, 1.0, 0.1, mode, 0.5), rtol=1e-12, atol=1e-14)


def test_bilateral_special_cases(orc):
    img = synth.structured_f32(16, 18)
    np.testing.assert_array_equal(orc.bilateral(img, 1, 1.0, 0.1, "clamp"), img.astype(np.float64))
    c = np.full((9, 9), 0.3, dtype=np.float32)
    np.testing.assert_allclose(orc.bilateral(c, 7, 1.5, 0.1, "mirror"), np.float64(np.float32(0.3)), rtol=1e-14)
    # sigma_r -> inf: the normalised spatial Gaussian filter
    win, sd = 7, 1.5
    g = np.exp(-(np.arange(win) - 3.0) ** 2 / (2 * sd * sd))
    G = np.outer(g, g) / np.outer(g, g).sum()
    for mode in MODES:
        ref = ndi.correlate(img.astype(np.float64), G, mode=NDI_MODE[mode], cval=0.2)
        np.testing.assert_allclose(orc.bilateral(img, win, sd, 1e30, mode, 0.2), ref, rtol=1e-12)
    # sigma_d, sigma_r -> inf: box mean
    ref = ndi.uniform_filter(img.astype(np.float64), 5, mode="reflect")
    np.testing.assert_allclose(orc.bilateral(img, 5, 1e30, 1e30, "mirror"), ref, rtol=1e-12)


# ---------------------------------------------------------------- Atrous / Night
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("d", [1, 2, 4, 8])
def test_atrous_equals_dilated_mask(orc, mode, d):
    """Atrous with dilation d == correlation with the (2d+1)^2 mask holding h_i h_j at
    the dilated taps and zeros in the holes; d = 1 is the 3x3 binomial Gaussian."""
    img = synth.uniform_f32(21, 26, 12)
    h = np.array([0.25, 0.5, 0.25])
    M = np.zeros((2 * d + 1, 2 * d + 1))
    for j in range(3):
        for i in range(3):
            M[j * d, i * d] = h[j] * h[i]
    ref = ndi.correlate(img.astype(np.float64), M, mode=NDI_MODE[mode], cval=0.125)
    np.testing.assert_allclose(orc.atrous(img, d, mode, 0.125), ref, rtol=1e-13, atol=1e-15)


def test_night_constant(orc):
    img = np.full((20, 20), 0.5, dtype=np.float32)
    np.testing.assert_allclose(orc.night(img, "repeat"), 0.5 / 1.5, rtol=1e-7)
