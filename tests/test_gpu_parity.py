"""GPU parity: the CUDA path (libisp.so through the Python binding) against the CPU
oracle, element by element on the same seeded inputs.

Bars (BASELINE.json north_star):
  * integer / byte outputs (u8 filters, Sobel, Laplace, Harris): bit-exact;
  * f32 linear filters: |gpu - oracle| <= 1e-5 * max(|oracle|, sum_taps |w * in|)
    (reading A28; the oracle accumulates in double);
  * Bilateral: max-abs <= 1e-4 on [0,1] data;
  * ISP_BLOCK, ISP_WARP, ISP_AUTO results are bitwise identical to ISP_NAIVE.
Sizes here: the FALLBACK shapes -- odd / misaligned widths (the planner sends them to
the naive kernel, which must still equal the oracle), tiny and degenerate plans (windows
larger than the image, reading A3) -- and BASELINE.json's full sizes on sampled rows in
the launch configuration bench.py times.  The aligned multi-tile shapes that run every
ISP region body (with the plan asserted) are in test_gpu_isp_bodies.py.
"""
import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

MODES = ["clamp", "mirror", "repeat", "constant"]
VARIANTS = ["auto", "tma", "block", "warp", "naive"]


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


def binomial_f32(m):
    b = synth.binomial_row(m).astype(np.float64)
    return (np.outer(b, b) / b.sum() ** 2).astype(np.float32)


# fallback shapes: misaligned widths (naive kernel) and tiny / degenerate plans
SHAPES = [(1, 1), (3, 5), (64, 64), (37, 517), (130, 1001), (257, 1031)]


# ---------------------------------------------------------------- generic f32 local operator
@pytest.mark.parametrize("mask_kind", ["binomial3", "binomial5", "binomial7", "rand3", "rand5", "rand7", "rand9",
                                       "rand5x3", "rand1x7"])
@pytest.mark.parametrize("shape", SHAPES)
def test_filter_f32(isp, shape, mask_kind):
    h, w = shape
    img = synth.uniform_f32(h, w, 100 + h)
    if mask_kind.startswith("binomial"):
        mask = binomial_f32(int(mask_kind[-1]))
    else:
        dims = mask_kind[4:]
        mh, mw = (int(dims), int(dims)) if "x" not in dims else map(int, dims.split("x"))
        mask = np.random.default_rng(7).standard_normal((mh, mw)).astype(np.float32)
    d = dev(img)
    for mode in MODES:
        ref, sc = oracle.filter_f64(img, mask, mode, 0.375, with_scale=True)
        outs = {}
        for v in VARIANTS:
            outs[v] = host(isp.isp_filter_ex(d, mask, mode, 0.375, variant=v))
            check_f32(outs[v], ref, sc)
        for v in VARIANTS[:-1]:
            np.testing.assert_array_equal(outs[v], outs["naive"], err_msg=f"{v} != naive ({mode})")


def test_filter_f32_north_star_calls(isp):
    img = synth.uniform_f32(300, 700, 3)
    mask = binomial_f32(5)
    d = dev(img)
    for mode in MODES:
        a = host(isp.isp_filter(d, mask, mode, 0.5))
        b = host(isp.isp_filter_naive(d, mask, mode, 0.5))
        np.testing.assert_array_equal(a, b)
        ref, sc = oracle.filter_f64(img, mask, mode, 0.5, with_scale=True)
        check_f32(a, ref, sc)


@pytest.mark.parametrize("m", [3, 5, 7, 9])
def test_filter_sep_f32(isp, m):
    img = synth.uniform_f32(150, 333, 5)
    rng = np.random.default_rng(m)
    row, col = rng.standard_normal(m).astype(np.float32), rng.standard_normal(m).astype(np.float32)
    mask = np.outer(col.astype(np.float64), row.astype(np.float64))
    d = dev(img)
    for mode in MODES:
        ref, sc = oracle.filter_f64(img, mask, mode, -1.5, with_scale=True)
        outs = [host(isp.isp_filter_sep_f32(d, row, col, mode, -1.5, variant=v)) for v in VARIANTS]
        for o in outs:
            check_f32(o, ref, sc)
            np.testing.assert_array_equal(o, outs[-1])


def test_misaligned_and_pitched(isp):
    h, w, pitch = 97, 301, 318          # pitch*4 not a multiple of 16, base offset by one element
    img = synth.uniform_f32(h, w, 9)
    buf = synth.pitched(img, pitch, fill=np.float32(np.nan))
    flat = torch.empty(h * pitch + 1, dtype=torch.float32, device="cuda")
    flat[1:] = torch.from_numpy(buf.ravel()).cuda()
    d = flat[1:].view(h, pitch)
    assert d.data_ptr() % 16 != 0
    for mname in ["binomial5", "rand5", "rand9"]:
        mask = binomial_f32(5) if mname == "binomial5" else \
            np.random.default_rng(2).standard_normal((int(mname[-1]),) * 2).astype(np.float32)
        aligned = host(isp.isp_filter_ex(dev(img), mask, "mirror"))
        for mode in MODES:
            ref, sc = oracle.filter_f64(buf, mask, mode, 0.25, w=w, with_scale=True)
            for v in VARIANTS:
                got = host(isp.isp_filter_ex(d, mask, mode, 0.25, variant=v, w=w))
                check_f32(got, ref, sc)
        # results do not depend on the alignment path
        np.testing.assert_array_equal(host(isp.isp_filter_ex(d, mask, "mirror", w=w)), aligned)


@pytest.mark.parametrize("shape,m", [((1, 1), 3), ((1, 1), 31), ((3, 5), 9), ((5, 3), 7), ((2, 40), 13),
                                     ((40, 2), 5), ((7, 7), 15)])
def test_window_larger_than_image(isp, shape, m):
    """Degenerate plans (A3): one block needs opposite checks; NAIVE with the general
    maps (Mirror period 2N, Repeat while loop) runs, for windows beyond the image."""
    h, w = shape
    img = synth.uniform_f32(h, w, 31)
    mask = np.random.default_rng(m).random((m, m)).astype(np.float32)
    d = dev(img)
    for mode in MODES:
        ref, sc = oracle.filter_f64(img, mask, mode, 2.0, with_scale=True)
        for v in VARIANTS:
            check_f32(host(isp.isp_filter_ex(d, mask, mode, 2.0, variant=v)), ref, sc)


# ---------------------------------------------------------------- u8 integer operators
@pytest.mark.parametrize("mask_kind", ["gauss3", "gauss5", "gauss7", "rand3", "rand5", "rand7", "rand9", "laplace5"])
@pytest.mark.parametrize("shape", SHAPES)
def test_filter_u8(isp, shape, mask_kind):
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
        outs = [host(isp.isp_filter_u8(d, mask, div, mode, 77, variant=v)) for v in VARIANTS]
        for v, o in zip(VARIANTS, outs):
            np.testing.assert_array_equal(o, ref, err_msg=f"{mask_kind} {mode} {v}")


@pytest.mark.parametrize("shape", [(1, 1), (2, 3), (64, 64), (77, 1000), (129, 4099)])
def test_sobel_laplace_harris(isp, shape):
    h, w = shape
    img = synth.structured_u8(h, w)
    d = dev(img)
    for mode in MODES:
        rdx, rdy, rmag = oracle.sobel(img, mode, 45)
        rlap = oracle.laplace5_u8(img, mode, 45)
        rhar = oracle.harris(rdx, rdy, mode, -3, 0)
        for v in VARIANTS:
            dx, dy, mag = isp.isp_sobel_u8(d, mode, 45, variant=v)
            np.testing.assert_array_equal(host(dx), rdx, err_msg=f"dx {mode} {v}")
            np.testing.assert_array_equal(host(dy), rdy, err_msg=f"dy {mode} {v}")
            np.testing.assert_array_equal(host(mag), rmag, err_msg=f"mag {mode} {v}")
            np.testing.assert_array_equal(host(isp.isp_laplace5_u8(d, mode, 45, variant=v)), rlap)
            har = isp.isp_harris_u8(dev(rdx), dev(rdy), mode, -3, 0, variant=v)
            np.testing.assert_array_equal(host(har), rhar, err_msg=f"harris {mode} {v}")


def test_sobel_partial_outputs(isp):
    img = synth.structured_u8(50, 90)
    rdx, rdy, rmag = oracle.sobel(img, "clamp")
    dx, dy, mag = isp.isp_sobel_u8(dev(img), "clamp", want=("mag",))
    assert dx is None and dy is None
    np.testing.assert_array_equal(host(mag), rmag)


def test_harris_thresholds(isp):
    dx = synth.random_i16(70, 130, 1)
    dy = synth.random_i16(70, 130, 2)
    for thr in [-(10 ** 13), 0, 10 ** 12, 10 ** 13]:
        ref = oracle.harris(dx, dy, "repeat", 11, thr)
        np.testing.assert_array_equal(host(isp.isp_harris_u8(dev(dx), dev(dy), "repeat", 11, thr)), ref)


# ---------------------------------------------------------------- Bilateral
@pytest.mark.parametrize("win", [1, 3, 5, 13, 31])
@pytest.mark.parametrize("shape", [(1, 1), (9, 11), (70, 133)])
def test_bilateral(isp, shape, win):
    h, w = shape
    img = synth.structured_f32(h, w)
    sd = max((win - 1) / 4.0, 0.5)
    d = dev(img)
    for mode in MODES:
        ref = oracle.bilateral(img, win, sd, 0.1, mode, 0.5)
        outs = [host(isp.isp_bilateral_f32(d, win, sd, 0.1, mode, 0.5, variant=v)) for v in VARIANTS]
        for v, o in zip(VARIANTS, outs):
            err = np.abs(o - ref).max()
            assert err <= 1e-4, (mode, v, err)
            np.testing.assert_array_equal(o, outs[-1])


# ---------------------------------------------------------------- Atrous / Night
@pytest.mark.parametrize("d", [1, 2, 4, 8])
@pytest.mark.parametrize("shape", [(3, 4), (40, 33), (150, 700)])
def test_atrous(isp, shape, d):
    h, w = shape
    img = synth.uniform_f32(h, w, 17)
    t = dev(img)
    for mode in MODES:
        ref = oracle.atrous(img, d, mode, 0.75)
        outs = [host(isp.isp_atrous_f32(t, d, mode, 0.75, variant=v)) for v in VARIANTS]
        for o in outs:
            check_f32(o, ref, np.abs(ref))        # A28: non-negative weights and data => scale |o|
            np.testing.assert_array_equal(o, outs[-1])


def test_night(isp):
    img = synth.uniform_f32(120, 260, 4)
    for mode in MODES:
        ref = oracle.night(img, mode, 0.25)
        got = host(isp.isp_night_f32(dev(img), mode, 0.25))
        check_f32(got, ref, np.abs(ref), tol=4e-5)   # 4 passes x A28 (see test_night_bodies)


# ---------------------------------------------------------------- BASELINE.json configs, full size
def sample_rows(h, k=16, seed=0):
    rng = np.random.default_rng(seed)
    rows = {0, 1, 2, 3, h // 2, h - 4, h - 3, h - 2, h - 1}
    rows |= set(int(r) for r in rng.integers(0, h, k))
    return sorted(r for r in rows if 0 <= r < h)


def test_cfg1_gauss3_u8_64(isp):
    img = synth.uniform_u8(64, 64, synth.CONFIG_SEEDS["cfg1"])
    mask, div = oracle.gaussian_u8_mask(3)
    ref = oracle.filter_u8(img, mask, div, "clamp")
    for v in VARIANTS:
        np.testing.assert_array_equal(host(isp.isp_filter_u8(dev(img), mask, div, "clamp", variant=v)), ref)


def test_cfg2_gauss5_f32_4096(isp):
    """The bench workload: 5x5 binomial f32 at 4096^2, all four modes, AUTO launch."""
    n = 4096
    img = synth.uniform_f32(n, n, synth.CONFIG_SEEDS["cfg2"])
    mask = binomial_f32(5)
    d = dev(img)
    rows = sample_rows(n)
    for mode in MODES:
        got = isp.isp_filter(d, mask, mode, 0.5)
        naive = isp.isp_filter_naive(d, mask, mode, 0.5)
        assert torch.equal(got, naive)
        ref, sc = oracle.filter_f64(img, mask, mode, 0.5, rows=rows, with_scale=True)
        check_f32(host(got)[rows], ref, sc)


def test_cfg3_pipeline_u8_4096(isp):
    n = 4096
    img = synth.structured_u8(n, n, synth.CONFIG_SEEDS["cfg3"])
    rows = sample_rows(n, seed=3)
    d = dev(img)
    dx, dy, mag = isp.isp_sobel_u8(d, "mirror")
    lap = isp.isp_laplace5_u8(d, "mirror")
    rdx, rdy, rmag = oracle.sobel(img, "mirror", threads=8)
    np.testing.assert_array_equal(host(dx), rdx)
    np.testing.assert_array_equal(host(dy), rdy)
    np.testing.assert_array_equal(host(mag), rmag)
    np.testing.assert_array_equal(host(lap)[rows], oracle.laplace5_u8(img, "mirror", rows=rows))
    har = isp.isp_harris_u8(dx, dy, "mirror")
    np.testing.assert_array_equal(host(har)[rows], oracle.harris(rdx, rdy, "mirror", rows=rows))


def test_cfg4_bilateral13_2048(isp):
    n = 2048
    img = synth.structured_f32(n, n, synth.CONFIG_SEEDS["cfg4"])
    rows = sample_rows(n, k=6, seed=4)
    d = dev(img)
    for mode in MODES:
        got = host(isp.isp_bilateral_f32(d, 13, 3.0, 0.1, mode, 0.5))[rows]
        ref = oracle.bilateral(img, 13, 3.0, 0.1, mode, 0.5, rows=rows)
        assert np.abs(got - ref).max() <= 1e-4


def test_cfg5_gauss7_f32_16384_single_gpu(isp):
    n = 16384
    g = torch.Generator(device="cuda").manual_seed(5)
    d = torch.rand((n, n), device="cuda", generator=g)
    # sampled rows plus the image's first / last three (the T / B regions of every kernel)
    rows = sorted(set(sample_rows(n, k=8, seed=5)) | {0, 1, 2, n - 3, n - 2, n - 1})
    band = sorted(set(r + k for r in rows for k in range(-3, 4) if 0 <= r + k < n) | {0, 1, 2, n - 3, n - 2, n - 1})
    mask = binomial_f32(7)
    cval = 0.25
    for mode in MODES:
        got = isp.isp_filter(d, mask, mode, cval)
        # oracle on the rows the sampled outputs depend on (plus the border rows the maps reach)
        sub = d[band].cpu().numpy()
        ref_full_rows = []
        for r in rows:
            ys = [oracle.border_index(mode, r + k, n) if mode != "constant" else r + k for k in range(-3, 4)]
            win = np.stack([sub[band.index(y)] if 0 <= y < n else np.full(n, cval, dtype=np.float32) for y in ys])
            # rows of `win` are already the mapped y taps (Constant: rows of C): row 3's output
            # uses exactly them; x is handled by the oracle's own border map
            out, sc = oracle.filter_f64(win, mask, mode, cval, rows=(3, 4), with_scale=True)
            ref_full_rows.append((out[0], sc[0]))
        ref = np.stack([r for r, _ in ref_full_rows])
        sc = np.stack([s for _, s in ref_full_rows])
        check_f32(host(got[rows]), ref, sc)


# ---------------------------------------------------------------- multi-GPU strips on one GPU
@pytest.mark.parametrize("nranks", [2, 3, 5, 8])
@pytest.mark.parametrize("m", [3, 5, 7, 9])
def test_strips_local_equal_full_image(isp, nranks, m):
    """Fallback strips: W = 333 is narrower than one ISP tile, so every strip launch is a
    degenerate plan (NAIVE); the strip/halo plumbing must still reproduce the
    single-image result bitwise.  The ISP strip bodies: test_gpu_isp_bodies.py."""
    H, W = 203, 333
    img = synth.uniform_f32(H, W, 77)
    mask = np.random.default_rng(m).random((m, m)).astype(np.float32)
    hy, halo = m // 2, m // 2 + 1
    full = dev(img)
    for mode in MODES:
        for v in VARIANTS:
            ref = host(isp.isp_filter_ex(full, mask, mode, 0.25, variant=v))
            got = np.full((H, W), np.nan, dtype=np.float32)
            for r in range(nranks):
                sc = isp.isp_shard_schedule(H, r, nranks, halo, hy, mode)
                y0, sh = sc["y0"], sc["strip_h"]
                buf = np.full((sh + 2 * halo, W), np.nan, dtype=np.float32)
                buf[halo:halo + sh] = img[y0:y0 + sh]
                for kind, peer, row, n in sc["ops"]:        # emulate the receives
                    if kind == 1:
                        g0 = y0 - halo + row                  # global rows this halo holds
                        buf[row:row + n] = img[[(g0 + k) % H for k in range(n)]]
                out = host(isp.isp_shard_filter_local_f32(dev(buf), H, halo, r, nranks, mask, mode, 0.25,
                                                          variant=v))
                got[y0:y0 + sh] = out
            np.testing.assert_array_equal(got, ref, err_msg=f"{mode} {v} P={nranks}")


def test_auto_follows_eq10(isp):
    """AUTO ("isp+m") takes the ISP kernel iff the model's G > 1 (Eq. 10, reading A20) with
    the B200-calibrated constants (A19, profiles/r02_counters.json) -- no other threshold;
    results identical to the oracle either way."""
    g5 = np.outer(synth.binomial_row(5), synth.binomial_row(5)).astype(np.int32)
    for n in (512, 1024, 4096):
        img = synth.structured_u8(n, n, 3)
        out = isp.isp_filter_u8(dev(img), g5, int(g5.sum()), "clamp", 7)
        torch.cuda.synchronize()
        plan = isp.isp_last_plan()
        if not plan["degenerate"]:
            assert (plan["choice"] != 3) == (plan["g"] > 1.0), plan
        rows = sample_rows(n, k=4, seed=n)
        np.testing.assert_array_equal(host(out)[rows], oracle.filter_u8(img, g5, int(g5.sum()), "clamp", 7, rows=rows))
