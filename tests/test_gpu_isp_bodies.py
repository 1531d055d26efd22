"""GPU parity of every ISP region body against the oracle, with proof that the body ran.

The round-1 parity shapes mostly sent compiled-window launches to the NAIVE kernel
(misaligned widths, degenerate tiles), so ISP bodies were compared only with naive.
Here every shape is vector/TMA aligned (f32: width % 4 == 0; u8: width % 16 == 0),
spans several tile columns plus a partial last tile and several tile rows, and each
launch is checked through isp_last_plan() / isp_recent_plans():

  * the requested variant is the one that ran (TMA -> k_staged / k_tile, WARP ->
    Listing 5, BLOCK -> Listing 3, NAIVE), and
  * the plan is not degenerate (reading A3), so the nine-region dispatch ran.

Then the output must equal the oracle: bit-exact for integer / byte outputs, A28 for
f32 (|g - o| <= 1e-5 * max(|o|, sum |w * in|)), max-abs 1e-4 for the Bilateral, and
every variant bitwise equal to NAIVE (ISP == NAIVE invariant).
"""
import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

MODES = ["clamp", "mirror", "repeat", "constant"]
CODE = {"auto": 0, "block": 1, "warp": 2, "naive": 3, "tma": 4}
ISP_VARIANTS = ["tma", "warp", "block"]

# (h, w): aligned, >= 3 tile columns + a partial one, several tile rows
F32_SHAPES = [(70, 2052), (45, 4100)]
U8_SHAPES = [(70, 2064), (33, 4112)]


@pytest.fixture(scope="module")
def isp():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_ipps_qiaoth21_b200 as m
    m.lib()
    oracle.build_oracle()
    return m


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def check_f32(got, ref, scale, tol=1e-5):
    bound = tol * np.maximum(np.abs(ref), scale) + 1e-30
    err = np.abs(got.astype(np.float64) - ref)
    bad = err > bound
    assert not bad.any(), f"{bad.sum()} px off; worst err {err.max():.3e} at {np.unravel_index(err.argmax(), err.shape)}"


def ran(isp, v, has_tma=True):
    """Assert the last launch ran variant v on a non-degenerate plan; return the plan."""
    p = isp.isp_last_plan()
    assert not p["degenerate"], f"degenerate plan for {v}: {p}"
    want = CODE[v]
    if v == "tma" and not has_tma:
        want = CODE["block"]
    if v != "auto":
        assert p["choice"] == want, f"requested {v}, ran choice {p['choice']} ({p})"
    return p


def run_all(isp, call, has_tma=True):
    """Run call(v) for naive + the ISP variants + auto; return {v: host array}."""
    outs = {}
    for v in ["naive"] + ISP_VARIANTS + ["auto"]:
        r = call(v)
        ran(isp, v, has_tma)
        outs[v] = host(r) if not isinstance(r, tuple) else tuple(host(t) for t in r)
    return outs


def binomial_f32(m):
    b = synth.binomial_row(m).astype(np.float64)
    return (np.outer(b, b) / b.sum() ** 2).astype(np.float32)


# ---------------------------------------------------------------- f32, compiled windows
@pytest.mark.parametrize("staged", [False, True])
@pytest.mark.parametrize("mask_kind", ["binomial3", "binomial5", "binomial7", "rand3", "rand5", "rand7"])
@pytest.mark.parametrize("shape", F32_SHAPES)
def test_f32_compiled_bodies(isp, shape, mask_kind, staged, monkeypatch):
    """OpSepF32<3/5/7> (rank-1 masks) and OpConvF32<3/5/7> in the TMA-staged k_staged
    (staged, or any non-separable mask) or the band kernel k_sep_band (separable masks),
    k_stencil Listing 3 / Listing 5 bodies and naive, every border mode."""
    if staged:
        monkeypatch.setenv("ISP_F32_STAGED", "1")
    h, w = shape
    img = synth.uniform_f32(h, w, 100 + h)
    m = int(mask_kind[-1])
    mask = binomial_f32(m) if mask_kind.startswith("binomial") else \
        np.random.default_rng(m).standard_normal((m, m)).astype(np.float32)
    d = dev(img)
    for mode in MODES:
        ref, sc = oracle.filter_f64(img, mask, mode, 0.375, with_scale=True)
        outs = run_all(isp, lambda v: isp.isp_filter_ex(d, mask, mode, 0.375, variant=v))
        for v, o in outs.items():
            check_f32(o, ref, sc)
            np.testing.assert_array_equal(o, outs["naive"], err_msg=f"{v} != naive ({mode} {mask_kind})")


@pytest.mark.parametrize("staged", [False, True])
@pytest.mark.parametrize("m", [3, 5, 7])
def test_f32_separable_entry_bodies(isp, m, staged, monkeypatch):
    if staged:
        monkeypatch.setenv("ISP_F32_STAGED", "1")
    h, w = F32_SHAPES[0]
    img = synth.uniform_f32(h, w, 5)
    rng = np.random.default_rng(m)
    row, col = rng.standard_normal(m).astype(np.float32), rng.standard_normal(m).astype(np.float32)
    mask = np.outer(col.astype(np.float64), row.astype(np.float64))
    d = dev(img)
    for mode in MODES:
        ref, sc = oracle.filter_f64(img, mask, mode, -1.5, with_scale=True)
        outs = run_all(isp, lambda v: isp.isp_filter_sep_f32(d, row, col, mode, -1.5, variant=v))
        for v, o in outs.items():
            check_f32(o, ref, sc)
            np.testing.assert_array_equal(o, outs["naive"])


# ---------------------------------------------------------------- f32, runtime windows (direct / tiled)
@pytest.mark.parametrize("mask_kind", ["rand9", "rand5x3", "rand1x7", "rand13", "rand31"])
def test_f32_direct_bodies(isp, mask_kind):
    h, w = 70, 1036
    img = synth.uniform_f32(h, w, 41)
    dims = mask_kind[4:]
    mh, mw = (int(dims), int(dims)) if "x" not in dims else map(int, dims.split("x"))
    mask = np.random.default_rng(mh * 31 + mw).standard_normal((mh, mw)).astype(np.float32)
    d = dev(img)
    for mode in MODES:
        ref, sc = oracle.filter_f64(img, mask, mode, 0.25, with_scale=True)
        outs = run_all(isp, lambda v: isp.isp_filter_ex(d, mask, mode, 0.25, variant=v))
        for v, o in outs.items():
            check_f32(o, ref, sc)
            np.testing.assert_array_equal(o, outs["naive"], err_msg=f"{v} {mode} {mask_kind}")


# ---------------------------------------------------------------- u8 operators
@pytest.mark.parametrize("mask_kind", ["gauss3", "gauss5", "gauss7", "rand3", "rand5", "rand7", "laplace5", "rand9"])
@pytest.mark.parametrize("shape", U8_SHAPES)
def test_u8_bodies(isp, shape, mask_kind):
    """OpSepU8 / OpConvU8 in k_staged (u8 TMA), k_stencil Listing 3 / 5 and naive; the
    direct family for 9x9."""
    h, w = shape
    img = synth.uniform_u8(h, w, 200 + w)
    if mask_kind.startswith("gauss"):
        mask, div = oracle.gaussian_u8_mask(int(mask_kind[-1]))
    elif mask_kind == "laplace5":
        mask, div = oracle.LAPLACE5, 1
    else:
        k = int(mask_kind[-1])
        mask, div = np.random.default_rng(k).integers(-9, 10, (k, k)).astype(np.int32), 7 + k
    d = dev(img)
    for mode in MODES:
        ref = oracle.filter_u8(img, mask, div, mode, 77)
        outs = run_all(isp, lambda v: isp.isp_filter_u8(d, mask, div, mode, 77, variant=v),
                       has_tma=mask_kind != "rand9")   # no tiled kernel for runtime-window u8
        for v, o in outs.items():
            np.testing.assert_array_equal(o, ref, err_msg=f"{mask_kind} {mode} {v}")


@pytest.mark.parametrize("shape", U8_SHAPES)
def test_sobel_laplace_harris_bodies(isp, shape):
    """OpSobel, OpLaplace5 and OpHarris bodies (T/B/L/R/corners/Body) in every mode,
    streaming and TMA-staged."""
    h, w = shape
    img = synth.structured_u8(h, w, 11)
    d = dev(img)
    for mode in MODES:
        rdx, rdy, rmag = oracle.sobel(img, mode, 45)
        rlap = oracle.laplace5_u8(img, mode, 45)
        rhar = oracle.harris(rdx, rdy, mode, -3, 0)
        sob = run_all(isp, lambda v: isp.isp_sobel_u8(d, mode, 45, variant=v))
        for v, (dx, dy, mag) in sob.items():
            np.testing.assert_array_equal(dx, rdx, err_msg=f"dx {mode} {v}")
            np.testing.assert_array_equal(dy, rdy, err_msg=f"dy {mode} {v}")
            np.testing.assert_array_equal(mag, rmag, err_msg=f"mag {mode} {v}")
        lap = run_all(isp, lambda v: isp.isp_laplace5_u8(d, mode, 45, variant=v))
        for v, o in lap.items():
            np.testing.assert_array_equal(o, rlap, err_msg=f"laplace {mode} {v}")
        ddx, ddy = dev(rdx), dev(rdy)
        har = run_all(isp, lambda v: isp.isp_harris_u8(ddx, ddy, mode, -3, 0, variant=v))
        for v, o in har.items():
            np.testing.assert_array_equal(o, rhar, err_msg=f"harris {mode} {v}")


# ---------------------------------------------------------------- Bilateral
@pytest.mark.parametrize("win", [3, 13, 31])
def test_bilateral_bodies(isp, win):
    h, w = 70, 1036
    img = synth.structured_f32(h, w, 4)
    sd = (win - 1) / 4.0
    d = dev(img)
    for mode in MODES:
        ref = oracle.bilateral(img, win, sd, 0.1, mode, 0.5)
        outs = run_all(isp, lambda v: isp.isp_bilateral_f32(d, win, sd, 0.1, mode, 0.5, variant=v))
        for v, o in outs.items():
            assert np.abs(o - ref).max() <= 1e-4, (mode, v)
            np.testing.assert_array_equal(o, outs["naive"], err_msg=f"{v} {mode}")


# ---------------------------------------------------------------- Atrous / Night
@pytest.mark.parametrize("dil", [1, 2, 4, 8])
@pytest.mark.parametrize("shape", F32_SHAPES)
def test_atrous_bodies(isp, shape, dil):
    """Row-direct Atrous bodies incl. Body/T/B; no TMA kernel (TMA request runs BLOCK).
    Tolerance A28: the weights are non-negative and the data (and C) non-negative, so
    sum |w * in| = |o| and the bound is 1e-5 |o|."""
    h, w = shape
    img = synth.uniform_f32(h, w, 17)
    t = dev(img)
    for mode in MODES:
        ref = oracle.atrous(img, dil, mode, 0.75)
        outs = run_all(isp, lambda v: isp.isp_atrous_f32(t, dil, mode, 0.75, variant=v), has_tma=False)
        for v, o in outs.items():
            check_f32(o, ref, np.abs(ref))
            np.testing.assert_array_equal(o, outs["naive"])


def test_night_bodies(isp):
    """Night = Atrous d=1,2,4,8 + tone map, each pass non-degenerate ISP (isp_recent_plans).
    Each pass is within A28 of its exactly-rounded value and the passes are averages with
    non-negative weights (errors do not grow), so 4 passes stay within 4e-5 |o|."""
    h, w = F32_SHAPES[0]
    img = synth.uniform_f32(h, w, 4)
    d = dev(img)
    for mode in MODES:
        ref = oracle.night(img, mode, 0.25)
        outs = {}
        for v in ["naive", "warp", "block", "auto"]:
            isp.isp_clear_plans()
            outs[v] = host(isp.isp_night_f32(d, mode, 0.25, variant=v))
            plans = isp.isp_recent_plans()
            assert len(plans) == 4
            for p in plans:
                assert not p["degenerate"]
                if v != "auto":
                    assert p["choice"] == CODE[v]
        for v, o in outs.items():
            check_f32(o, ref, np.abs(ref), tol=4e-5)
            np.testing.assert_array_equal(o, outs["naive"])


# ---------------------------------------------------------------- multi-GPU strips (RowRange ISP)
def _strip_run(isp, img, H, W, halo, hy, nranks, r, mode, fill, local_call):
    sc = isp.isp_shard_schedule(H, r, nranks, halo, hy, mode)
    y0, sh = sc["y0"], sc["strip_h"]
    buf = np.full((sh + 2 * halo, W), fill, dtype=img.dtype)
    buf[halo:halo + sh] = img[y0:y0 + sh]
    for kind, peer, row, n in sc["ops"]:        # emulate the NCCL receives
        if kind == 1:
            g0 = y0 - halo + row
            buf[row:row + n] = img[[(g0 + k) % H for k in range(n)]]
    return y0, sh, local_call(dev(buf))


@pytest.mark.parametrize("sep", [False, True])
@pytest.mark.parametrize("nranks", [2, 3, 5, 8])
@pytest.mark.parametrize("m", [3, 5, 7, 9])
def test_strips_isp_f32(isp, nranks, m, sep):
    """Strip launches (RowRange, t_real / b_real = 0 at strip edges) of every rank on a
    2052-wide image run non-degenerate ISP bodies and reproduce the single-image result
    bitwise, with the halo rows filled as the NCCL schedule fills them; separable masks
    (sep) run the band kernel k_sep_band on the strips (TMA)."""
    H, W = 203, 2052
    img = synth.uniform_f32(H, W, 77)
    mask = binomial_f32(m) if sep else np.random.default_rng(m).random((m, m)).astype(np.float32)
    hy = m // 2
    halo = hy + 1
    full = dev(img)
    for mode in MODES:
        for v in ["tma", "warp", "naive"]:
            ref = host(isp.isp_filter_ex(full, mask, mode, 0.25, variant=v))
            got = np.full((H, W), np.nan, dtype=np.float32)
            for r in range(nranks):
                isp.isp_clear_plans()
                y0, sh, out = _strip_run(
                    isp, img, H, W, halo, hy, nranks, r, mode, np.nan,
                    lambda b: isp.isp_shard_filter_local_f32(b, H, halo, r, nranks, mask, mode, 0.25, variant=v))
                got[y0:y0 + sh] = host(out)
                main = isp.isp_recent_plans()[0]          # launch 0: the rows needing no halo
                assert not main["degenerate"], (mode, v, r, main)
                if m != 9 or v != "tma":
                    assert main["choice"] == CODE[v], (mode, v, r, main)
            np.testing.assert_array_equal(got, ref, err_msg=f"{mode} {v} P={nranks}")


@pytest.mark.parametrize("nranks", [2, 4, 8])
@pytest.mark.parametrize("m", [3, 5])
def test_strips_isp_u8(isp, nranks, m):
    """isp_shard_filter_local_u8: u8 Gaussian strips equal the oracle exactly."""
    H, W = 150, 2064
    img = synth.uniform_u8(H, W, 78)
    mask, div = oracle.gaussian_u8_mask(m)
    halo = m // 2 + 1
    for mode in MODES:
        ref = oracle.filter_u8(img, mask, div, mode, 9)
        for v in ["warp", "tma", "naive"]:
            got = np.zeros((H, W), dtype=np.uint8)
            for r in range(nranks):
                isp.isp_clear_plans()
                y0, sh, out = _strip_run(
                    isp, img, H, W, halo, m // 2, nranks, r, mode, 0,
                    lambda b: isp.isp_shard_filter_local_u8(b, H, halo, r, nranks, mask, div, mode, 9, variant=v))
                got[y0:y0 + sh] = host(out)
                main = isp.isp_recent_plans()[0]
                assert not main["degenerate"] and main["choice"] == CODE[v], (mode, v, r, main)
            np.testing.assert_array_equal(got, ref, err_msg=f"{mode} {v} P={nranks}")


# ---------------------------------------------------------------- Harris exactness at the threshold
def _harris_r25(dx, dy, mode, c, y, x):
    """Exact R25 at (y, x) in Python integers through the oracle's border map."""
    h, w = dx.shape
    wts = [1, 2, 1]
    sxx = syy = sxy = 0
    for j in range(3):
        for i in range(3):
            yy = oracle.border_index(mode, y + j - 1, h)
            xx = oracle.border_index(mode, x + i - 1, w)
            if yy < 0 or xx < 0:
                gx = gy = c
            else:
                gx, gy = int(dx[yy, xx]), int(dy[yy, xx])
            wt = wts[j] * wts[i]
            sxx += wt * gx * gx
            syy += wt * gy * gy
            sxy += wt * gx * gy
    return 25 * (sxx * syy - sxy * sxy) - (sxx + syy) ** 2


def test_harris_threshold_boundary(isp):
    """thr = R-1, R, R+1 around the true response of chosen pixels (large |R| ~ 1e15,
    derivatives near +-1020): the f32 sums / f64 response decide exactly as int64."""
    h, w = 40, 2064
    rng = np.random.default_rng(123)
    dx = rng.integers(-1020, 1021, (h, w)).astype(np.int16)
    dy = rng.integers(-1020, 1021, (h, w)).astype(np.int16)
    dx[:, ::7] = 1020
    dy[::5, :] = -1020
    ddx, ddy = dev(dx), dev(dy)
    picks = [(0, 0), (h - 1, w - 1), (17, 1030), (3, 700), (39, 5)]
    for mode in MODES:
        c = -1020 if mode == "constant" else 0
        for (y, x) in picks:
            R = _harris_r25(dx, dy, mode, c, y, x)
            for thr, want in ((R - 1, 255), (R, 0), (R + 1, 0)):
                ref = oracle.harris(dx, dy, mode, c, thr)
                assert ref[y, x] == want
                for v in ["tma", "warp", "naive"]:
                    got = host(isp.isp_harris_u8(ddx, ddy, mode, c, thr, variant=v))
                    ran(isp, v)
                    assert got[y, x] == want, (mode, v, y, x, thr)
                    np.testing.assert_array_equal(got, ref, err_msg=f"{mode} {v} thr={thr}")


def test_harris_flat_areas(isp):
    """All-zero window sums (flat image areas: t = 0, R25 = 0 exactly) decide in the f32
    path (the bound is 0 there only for thr = 0): R25 > thr for thr = 0, -1, 1 and far
    outside, next to textured spots and spots with dy = 0 (R25 = -Sxx^2 < 0), every mode
    and variant, and the fused pipeline on a piecewise-constant image -- bit-exact."""
    h, w = 37, 2064
    dx = np.zeros((h, w), dtype=np.int16)
    dy = np.zeros((h, w), dtype=np.int16)
    rng = np.random.default_rng(5)
    dx[10:14, 300:340] = rng.integers(-1020, 1021, (4, 40))
    dy[10:14, 300:340] = rng.integers(-1020, 1021, (4, 40))
    dx[20:23, 1000:1100] = 7          # dy = 0: R25 = -(Sxx)^2
    dx[0, :] = 1                      # edge row (T region) with tiny sums
    ddx, ddy = dev(dx), dev(dy)
    for mode in MODES:
        for c in ((0, 3) if mode == "constant" else (0,)):
            for thr in (0, -1, 1, -(10 ** 12), 10 ** 12):
                ref = oracle.harris(dx, dy, mode, c, thr)
                for v in ["tma", "warp", "naive"]:
                    got = host(isp.isp_harris_u8(ddx, ddy, mode, c, thr, variant=v))
                    ran(isp, v)
                    np.testing.assert_array_equal(got, ref, err_msg=f"{mode} {v} c={c} thr={thr}")
    img = np.full((64, 2048), 77, dtype=np.uint8)
    img[20:30, 500:520] = 200
    img[40:, :] = 10
    d = dev(img)
    for mode in MODES:
        rdx, rdy, _ = oracle.sobel(img, mode, 0)
        for thr in (0, -1, 1):
            want = oracle.harris(rdx, rdy, mode, 0, thr)
            for v in ["tma", "warp"]:
                _, _, har = isp.isp_pipeline_cfg3_u8(d, mode, 0, 0, thr, variant=v)
                np.testing.assert_array_equal(host(har), want, err_msg=f"fused {mode} {v} thr={thr}")


def test_harris_const_range(isp):
    d = dev(np.zeros((8, 16), dtype=np.int16))
    with pytest.raises(isp.IspError):
        isp.isp_harris_u8(d, d, "constant", 1021, 0)
    with pytest.raises(isp.IspError):
        isp.isp_harris_u8(d, d, "constant", -1021, 0)


# ---------------------------------------------------------------- Sobel magnitude near ties
def _sobel_block(X, Y, rng):
    """A 3x3 u8 block whose centre Sobel derivatives are exactly (X, Y) (a9: dx = (c-a) +
    2(f-d) + (i-g), dy = (g-a) + 2(h-b) + (i-c) over [[a,b,c],[d,e,f],[g,h,i]])."""
    for _ in range(200000):
        a, c, g, i = (int(t) for t in rng.integers(0, 256, 4))
        r1, r2 = X - (c - a) - (i - g), Y - (g - a) - (i - c)
        if r1 % 2 or r2 % 2 or abs(r1 // 2) > 255 or abs(r2 // 2) > 255:
            continue
        fd, hb = r1 // 2, r2 // 2
        d_, b_ = max(0, -fd), max(0, -hb)
        f_, h_ = d_ + fd, b_ + hb
        blk = np.array([[a, b_, c], [d_, 128, f_], [g, h_, i]])
        if blk.min() >= 0 and blk.max() <= 255:
            return blk.astype(np.uint8)
    raise AssertionError((X, Y))


def test_sobel_magnitude_near_ties(isp):
    """Magnitude rounding next to every half-integer: n = dx^2 + dy^2 within +-4 of
    (k + 1/2)^2 = k^2 + k + 1/4 for k = 1..255 (the tightest margins of the sqrt.approx
    rounding: 0.25/(2k+1) at n = k^2 + k).  Sobel
    derivatives of u8 images satisfy dx = dy (mod 2) (dx + dy = 2(i - a) + even terms),
    so only n = 0 (mod 4) or 2 (mod 8) occur: the test places every reachable n of the
    band, with both signs, at centres of isolated 3x3 blocks and compares the whole
    image with the oracle."""
    targets = []
    for k in range(1, 256):
        for n in range(k * k + k - 4, k * k + k + 5):
            for X in range(0, 257):
                r = n - X * X
                if r < 0:
                    break
                Y = int(round(r ** 0.5))
                if Y * Y == r and (X - Y) % 2 == 0:
                    sx, sy = (1, -1)[len(targets) % 2], (1, -1)[(len(targets) // 2) % 2]
                    targets.append((sx * X, sy * Y, n))
                    break
    assert len(targets) >= 150
    rng = np.random.default_rng(5)
    nb = len(targets)
    per_row = 680
    rows = -(-nb // per_row)
    img = np.zeros((3 * rows + 40, 3 * per_row + 24), dtype=np.uint8)   # 2064 wide: 16-B aligned rows
    centres = []
    for t, (X, Y, n) in enumerate(targets):
        by, bx = 3 + 3 * (t // per_row), 3 * (t % per_row)
        img[by:by + 3, bx:bx + 3] = _sobel_block(X, Y, rng)
        centres.append((by + 1, bx + 1, X, Y, n))
    d = dev(img)
    for mode in MODES:
        rdx, rdy, rmag = oracle.sobel(img, mode, 0)
        for (y, x, X, Y, n) in centres:
            assert int(rdx[y, x]) ** 2 + int(rdy[y, x]) ** 2 == n
        for v in ["tma", "warp", "naive"]:
            dx, dy, mag = isp.isp_sobel_u8(d, mode, 0, variant=v)
            ran(isp, v)
            np.testing.assert_array_equal(host(mag), rmag, err_msg=f"{mode} {v}")


# ---------------------------------------------------------------- peer-direct strips (N4)
@pytest.mark.parametrize("sep", [False, True])
@pytest.mark.parametrize("nranks", [2, 3, 8])
@pytest.mark.parametrize("m", [3, 7, 9])
def test_peer_strips_f32(isp, nranks, m, sep):
    """Peer-direct strips: every rank's buffer holds only its own rows,
    the neighbour rows are read from the neighbours' buffers (separate allocations, as
    IPC mappings would be), ONE launch per rank; the gathered result equals the
    single-image result bitwise, strip-edge block rows run T / B bodies (non-degenerate);
    separable masks (sep) run the band kernel, whose strip-edge bands select the buffer."""
    H, W = 203, 2052
    img = synth.uniform_f32(H, W, 79)
    mask = binomial_f32(m) if sep else np.random.default_rng(m).random((m, m)).astype(np.float32)
    full = dev(img)
    strips = []
    for r in range(nranks):
        y0, sh = isp.isp_shard_rows(H, r, nranks)
        strips.append(dev(img[y0:y0 + sh]))
    for mode in MODES:
        ring = mode == "repeat"
        for v in ["tma", "warp", "naive"]:
            ref = host(isp.isp_filter_ex(full, mask, mode, 0.25, variant=v))
            got = np.full((H, W), np.nan, dtype=np.float32)
            for r in range(nranks):
                y0, sh = isp.isp_shard_rows(H, r, nranks)
                prev = strips[r - 1] if r > 0 else (strips[-1] if ring else None)
                nxt = strips[r + 1] if r < nranks - 1 else (strips[0] if ring else None)
                isp.isp_clear_plans()
                out = isp.isp_shard_filter_peer_local_f32(strips[r], prev, nxt, H, r, nranks, mask, mode, 0.25,
                                                          variant=v)
                plans = isp.isp_recent_plans()
                assert len(plans) == 1 and not plans[0]["degenerate"], plans
                got[y0:y0 + sh] = host(out)
            np.testing.assert_array_equal(got, ref, err_msg=f"{mode} {v} P={nranks} m={m}")


@pytest.mark.parametrize("nranks", [2, 4])
def test_peer_strips_u8(isp, nranks):
    H, W = 150, 2064
    img = synth.uniform_u8(H, W, 80)
    mask, div = oracle.gaussian_u8_mask(5)
    strips = [dev(img[slice(*(lambda y, s: (y, y + s))(*isp.isp_shard_rows(H, r, nranks)))]) for r in range(nranks)]
    for mode in MODES:
        ring = mode == "repeat"
        ref = oracle.filter_u8(img, mask, div, mode, 9)
        for v in ["warp", "tma", "naive"]:
            got = np.zeros((H, W), dtype=np.uint8)
            for r in range(nranks):
                y0, sh = isp.isp_shard_rows(H, r, nranks)
                prev = strips[r - 1] if r > 0 else (strips[-1] if ring else None)
                nxt = strips[r + 1] if r < nranks - 1 else (strips[0] if ring else None)
                got[y0:y0 + sh] = host(isp.isp_shard_filter_peer_local_u8(strips[r], prev, nxt, H, r, nranks, mask,
                                                                          div, mode, 9, variant=v))
            np.testing.assert_array_equal(got, ref, err_msg=f"{mode} {v} P={nranks}")


# ---------------------------------------------------------------- tile-staged Laplace / Harris
@pytest.mark.parametrize("shape", [(260, 2064), (133, 400), (4096 // 8, 4096)])
def test_laplace_harris_tile_kernels(isp, shape):
    """The tile-staged ISP kernels of Laplace and Harris (tile_u8.cu; Body tiles unchecked,
    border tiles staged through the pattern, partial right / bottom tiles): bit-exact
    against the oracle in every mode, several Harris thresholds, the plan showing the
    tile variant (choice TMA, 128 x 32 tiles)."""
    h, w = shape
    img = synth.structured_u8(h, w, 12)
    d = dev(img)
    for mode in MODES:
        rlap = oracle.laplace5_u8(img, mode, 33)
        # Laplace: a width that is not a multiple of 8 (pitch still 16-B aligned) is not
        # band-eligible, so the tile kernel runs
        wt = w - 4
        got = host(isp.isp_laplace5_u8(d, mode, 33, variant="tma", w=wt))
        p = isp.isp_last_plan()
        assert p["choice"] == CODE["tma"] and p["tile_w"] == 128 and p["tile_h"] == 32, p
        np.testing.assert_array_equal(got[:, :wt], oracle.laplace5_u8(np.ascontiguousarray(img[:, :wt]), mode, 33),
                                      err_msg=f"laplace tile {mode}")
        got = host(isp.isp_laplace5_u8(d, mode, 33, variant="tma"))
        p = isp.isp_last_plan()
        assert p["choice"] == CODE["tma"] and p["tile_w"] == 512, p   # the band kernel
        np.testing.assert_array_equal(got, rlap, err_msg=f"laplace {mode}")
        rdx, rdy, _ = oracle.sobel(img, mode, 33)
        ddx, ddy = dev(rdx), dev(rdy)
        c = 700 if mode == "constant" else 0
        # Harris: a width that is not a multiple of 4 runs the tile kernel, else the band one
        wt = w - 2
        sdx, sdy = np.ascontiguousarray(rdx[:, :wt]), np.ascontiguousarray(rdy[:, :wt])
        for thr in (0, -(10 ** 7), 10 ** 9, 10 ** 12):
            got = host(isp.isp_harris_u8(ddx, ddy, mode, c, thr, variant="tma", w=wt,
                                         out=torch.empty((h, w), dtype=torch.uint8, device="cuda")))
            p = isp.isp_last_plan()
            assert p["choice"] == CODE["tma"] and p["tile_w"] == 128 and p["tile_h"] == 32, p
            np.testing.assert_array_equal(got[:, :wt], oracle.harris(sdx, sdy, mode, c, thr),
                                          err_msg=f"harris tile {mode} thr={thr}")
            rhar = oracle.harris(rdx, rdy, mode, c, thr)
            got = host(isp.isp_harris_u8(ddx, ddy, mode, c, thr, variant="tma"))
            p = isp.isp_last_plan()
            assert p["choice"] == CODE["tma"] and p["tile_w"] in (128, 256) and p["tile_h"] < 32, p   # band
            np.testing.assert_array_equal(got, rhar, err_msg=f"harris {mode} thr={thr}")
        # random int16 derivatives over the whole Sobel range
        rx = synth.random_i16(h, w, 5)
        ry = synth.random_i16(h, w, 6)
        np.testing.assert_array_equal(host(isp.isp_harris_u8(dev(rx), dev(ry), mode, -3, 10 ** 11, variant="tma")),
                                      oracle.harris(rx, ry, mode, -3, 10 ** 11), err_msg=f"harris random {mode}")


# ---------------------------------------------------------------- warp-strip band Laplace
@pytest.mark.parametrize("nw", [4, 2])
@pytest.mark.parametrize("shape", [(8, 32), (9, 48), (9, 264), (70, 2064), (33, 4112), (260, 528), (101, 512), (4096 // 8, 4096),
                                   (17, 784)])
def test_laplace_band_kernel(isp, shape, nw, monkeypatch):
    """The warp-strip streaming Laplace (band_u8.cu) at 16 and 8 pixels per lane: strips of
    512 / 256 columns (partial last strips down to one lane, a single strip that is both L
    and R), bands down to 6 rows (T and B in one band), all four modes and constants 0 / 255
    -- bit-exact against the oracle, the plan showing the band kernel ran (TMA choice,
    strip-wide tiles)."""
    monkeypatch.setenv("ISP_BAND_NW", str(nw))
    h, w = shape
    img = synth.structured_u8(h, w, 21)
    img[0, :] = 255
    img[:, -1] = 0
    d = dev(img)
    for mode in MODES:
        for c in ((0, 255) if mode == "constant" else (0,)):
            got = host(isp.isp_laplace5_u8(d, mode, c, variant="tma"))
            p = isp.isp_last_plan()
            # widths not a multiple of the lane's 4 nw pixels are not band-eligible (fallback)
            assert (p["choice"] == CODE["tma"] and p["tile_w"] == 128 * nw) == (w % (4 * nw) == 0), p
            np.testing.assert_array_equal(got, oracle.laplace5_u8(img, mode, c), err_msg=f"{mode} c={c}")
    # AUTO (Eq. 10 decides between the band kernel and the naive one): still exact
    np.testing.assert_array_equal(host(isp.isp_laplace5_u8(d, "mirror", 0)), oracle.laplace5_u8(img, "mirror", 0))


@pytest.mark.parametrize("groups", [1, 2])
@pytest.mark.parametrize("shape", [(8, 16), (9, 132), (9, 136), (70, 2064), (33, 4112), (101, 256), (4096 // 8, 4096), (17, 264)])
def test_harris_band_kernel(isp, shape, groups, monkeypatch):
    """The warp-strip streaming Harris (band_u8.cu): strips of 128 columns (partial last
    strips down to one lane, one strip that is both L and R), bands down to 4 rows, all
    modes, constants at the ends of the Sobel range, thresholds from far below to far
    above the responses, Sobel derivatives of a structured image and random int16 over the
    whole range -- bit-exact against the oracle's int64 definition; 4 (groups 1) and 8
    (groups 2) pixels per lane."""
    monkeypatch.setenv("ISP_HARRIS_G", str(groups))
    h, w = shape
    img = synth.structured_u8(h, w, 23)
    for mode in MODES:
        rdx, rdy, _ = oracle.sobel(img, mode, 9)
        rx = synth.random_i16(h, w, 31)
        ry = synth.random_i16(h, w, 32)
        for dx, dy in ((rdx, rdy), (rx, ry)):
            ddx, ddy = dev(dx), dev(dy)
            for c in ((-1020, 1020) if mode == "constant" else (0,)):
                for thr in (0, -(10 ** 9), 10 ** 8, 10 ** 13):
                    got = host(isp.isp_harris_u8(ddx, ddy, mode, c, thr, variant="tma"))
                    p = isp.isp_last_plan()
                    band = p["choice"] == CODE["tma"] and p["warp_w"] == 128 * groups and p["tile_h"] < 32
                    assert band == (w % (4 * groups) == 0), p   # partial lanes: not band-eligible
                    np.testing.assert_array_equal(got, oracle.harris(dx, dy, mode, c, thr),
                                                  err_msg=f"{mode} c={c} thr={thr}")


# ---------------------------------------------------------------- warp-strip band f32 (separable)
@pytest.mark.parametrize("m", [3, 5, 7])
@pytest.mark.parametrize("shape", [(8, 8), (9, 132), (70, 2052), (45, 4100), (300, 520), (4096 // 8, 4096)])
def test_sep_band_kernel(isp, shape, m):
    """k_sep_band (band_f32.cu), the TMA / AUTO kernel of whole-image separable f32 masks:
    strips of 128 columns (partial last strips down to one lane, one strip that is L and R),
    bands holding both image edges, binomial and random rank-1 masks, every mode -- A28
    against the oracle and bitwise equal to the naive kernel, the plan showing the band
    kernel (128-column tiles, TMA choice)."""
    h, w = shape
    img = synth.uniform_f32(h, w, 300 + m)
    rng = np.random.default_rng(77 + m)
    for mask in (binomial_f32(m), np.outer(rng.standard_normal(m), rng.standard_normal(m)).astype(np.float32)):
        d = dev(img)
        for mode in MODES:
            ref, sc = oracle.filter_f64(img, mask, mode, 0.625, with_scale=True)
            got = host(isp.isp_filter_ex(d, mask, mode, 0.625, variant="tma"))
            p = isp.isp_last_plan()
            assert p["choice"] == CODE["tma"] and p["tile_w"] == 128 and p["warp_w"] == 128, p
            check_f32(got, ref, sc)
            naive = host(isp.isp_filter_ex(d, mask, mode, 0.625, variant="naive"))
            np.testing.assert_array_equal(got, naive, err_msg=f"band != naive {mode} m={m}")


# ---------------------------------------------------------------- warp-strip band Sobel
@pytest.mark.parametrize("groups", [1, 2])
@pytest.mark.parametrize("shape", [(8, 16), (9, 132), (9, 136), (70, 2064), (45, 264), (4096 // 8, 4096)])
def test_sobel_band_kernel(isp, shape, groups, monkeypatch):
    """k_sob_band (band_u8.cu), the TMA / AUTO kernel of isp_sobel_u8: strips of 128
    columns (partial last strips down to one lane, one strip that is L and R), all modes and
    constants 0 / 255, every subset of the dx / dy / mag outputs -- bit-exact against the
    oracle, the plan showing the band kernel; 4 (groups 1) and 8 (groups 2) pixels per lane."""
    monkeypatch.setenv("ISP_SOBEL_G", str(groups))
    h, w = shape
    img = synth.structured_u8(h, w, 41)
    img[0, :] = 255
    img[:, -1] = 3
    d = dev(img)
    for mode in MODES:
        for c in ((0, 255) if mode == "constant" else (17,)):
            rdx, rdy, rmag = oracle.sobel(img, mode, c)
            for want in (("dx", "dy", "mag"), ("mag",), ("dx",), ("dy", "mag")):
                dx, dy, mag = isp.isp_sobel_u8(d, mode, c, variant="tma", want=want)
                p = isp.isp_last_plan()
                band = p["choice"] == CODE["tma"] and p["warp_w"] == 128 * groups and p["tile_h"] < 32
                assert band == (w % (4 * groups) == 0), p   # partial lanes: not band-eligible
                for name, got, ref in (("dx", dx, rdx), ("dy", dy, rdy), ("mag", mag, rmag)):
                    if name in want:
                        np.testing.assert_array_equal(host(got), ref, err_msg=f"{name} {mode} c={c} {want}")


# ---------------------------------------------------------------- warp-strip band separable u8
@pytest.mark.parametrize("nw", [2, 4])
@pytest.mark.parametrize("shape", [(8, 32), (9, 48), (9, 264), (70, 2064), (33, 4112), (260, 528), (4096 // 8, 4096)])
def test_sepu8_band_kernel(isp, shape, nw, monkeypatch):
    """k_sepu8_band (band_u8.cu), the TMA / AUTO kernel of normalised separable u8 masks: the
    3x3 / 16 and 5x5 / 256 binomials and a [1,2,1]^2 / 32 mask (result <= 127), all modes,
    strips of 256 columns with partial last strips -- bit-exact against the oracle, the plan
    showing the band kernel; a divisor that is not a power of two takes the generic path;
    8 (nw 2) and 16 (nw 4) pixels per lane."""
    monkeypatch.setenv("ISP_SEPU8_NW", str(nw))
    h, w = shape
    img = synth.uniform_u8(h, w, 51)
    img[0, :] = 255
    d = dev(img)
    b3 = synth.binomial_row(3).astype(np.int64)
    masks = [(oracle.gaussian_u8_mask(3)), (oracle.gaussian_u8_mask(5)), (np.outer(b3, b3).astype(np.int32), 32)]
    for mask, div in masks:
        for mode in MODES:
            ref = oracle.filter_u8(img, mask, div, mode, 201)
            got = host(isp.isp_filter_u8(d, mask, div, mode, 201, variant="tma"))
            p = isp.isp_last_plan()
            band = p["choice"] == CODE["tma"] and p["warp_w"] == 128 * nw and p["tile_h"] < 32
            assert band == (w % (4 * nw) == 0), p   # partial lanes: not band-eligible
            np.testing.assert_array_equal(got, ref, err_msg=f"{mode} div={div} m={mask.shape}")
    mask, _ = oracle.gaussian_u8_mask(5)
    got = host(isp.isp_filter_u8(d, mask, 300, "mirror", 0, variant="tma"))
    assert isp.isp_last_plan()["warp_w"] != 128 * nw
    np.testing.assert_array_equal(got, oracle.filter_u8(img, mask, 300, "mirror", 0))
