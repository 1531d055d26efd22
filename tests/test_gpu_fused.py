"""GPU parity of the fused cfg3 pipeline (isp_pipeline_cfg3_u8) against
the oracle COMPOSITION oracle.sobel -> oracle.laplace5_u8 -> oracle.harris: bit-exact on
every output, every border mode, ISP (auto) and naive staging, ragged shapes spanning
several 128x32 tiles, pitched images, and BASELINE.json configs[2] at full size.
Harris' border handling applies to the dx/dy images (remapped coordinates), which the
composition states by construction.
"""
import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

MODES = ["clamp", "mirror", "repeat", "constant"]


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


def composition(img, mode, c, hc, thr):
    rdx, rdy, rmag = oracle.sobel(img, mode, c)
    return rdx, rdy, rmag, oracle.laplace5_u8(img, mode, c), oracle.harris(rdx, rdy, mode, hc, thr)


@pytest.mark.parametrize("shape", [(1, 1), (2, 3), (5, 130), (33, 129), (64, 64), (70, 300), (131, 517), (8, 8),
                                   (9, 132), (70, 2064), (45, 260), (300, 1000)])
@pytest.mark.parametrize("kind", ["structured", "noise"])
def test_fused_matches_composition(isp, shape, kind):
    """auto / tma: the band kernel where w % 4 == 0 and h >= 8 (partial strips down to one
    lane, single-strip images, bands holding both image edges), else the tile / general
    kernels; warp: the tile-ISP kernel; naive: the general kernel."""
    h, w = shape
    img = synth.structured_u8(h, w, 5) if kind == "structured" else synth.uniform_u8(h, w, 5)
    d = dev(img)
    for mode in MODES:
        rdx, rdy, rmag, rlap, rhar = composition(img, mode, 45, -3, 0)
        for v in ["auto", "tma", "warp", "naive"]:
            dx = torch.empty((h, w), dtype=torch.int16, device="cuda")
            dy = torch.empty_like(dx)
            mag, lap, har = isp.isp_pipeline_cfg3_u8(d, mode, 45, -3, 0, dx=dx, dy=dy, variant=v)
            for name, got, ref in [("dx", dx, rdx), ("dy", dy, rdy), ("mag", mag, rmag), ("lap", lap, rlap),
                                   ("harris", har, rhar)]:
                np.testing.assert_array_equal(host(got), ref, err_msg=f"{name} {mode} {v} {shape} {kind}")


def test_fused_pitched_and_thresholds(isp):
    h, w, pitch = 97, 333, 352
    img = synth.uniform_u8(h, w, 9)
    d = dev(synth.pitched(img, pitch, 200))
    for mode in MODES:
        for thr in [-(10 ** 12), 0, 10 ** 11]:
            _, _, rmag, rlap, rhar = composition(img, mode, 7, 1020 if mode == "constant" else 0, thr)
            mag = torch.zeros((h, pitch), dtype=torch.uint8, device="cuda")
            lap, har = torch.zeros_like(mag), torch.zeros_like(mag)
            isp.isp_pipeline_cfg3_u8(d, mode, 7, 1020 if mode == "constant" else 0, thr, mag=mag, lap=lap,
                                     harris=har, w=w)
            np.testing.assert_array_equal(host(mag)[:, :w], rmag, err_msg=f"mag {mode}")
            np.testing.assert_array_equal(host(lap)[:, :w], rlap, err_msg=f"lap {mode}")
            np.testing.assert_array_equal(host(har)[:, :w], rhar, err_msg=f"harris {mode} {thr}")
            assert not host(mag)[:, w:].any()   # nothing written past the image width


def test_fused_equals_three_launches(isp):
    """Same bits as the unfused ISP pipeline on a multi-tile image (all modes)."""
    img = synth.uniform_u8(300, 1000, 11)
    d = dev(img)
    for mode in MODES:
        dx, dy, mag = isp.isp_sobel_u8(d, mode, 3)
        lap = isp.isp_laplace5_u8(d, mode, 3)
        har = isp.isp_harris_u8(dx, dy, mode, 5, 0)
        fm, fl, fh = isp.isp_pipeline_cfg3_u8(d, mode, 3, 5, 0)
        assert torch.equal(fm, mag) and torch.equal(fl, lap) and torch.equal(fh, har), mode


def test_fused_cfg3_4096(isp):
    """BASELINE.json configs[2] at full size, the launch bench_suite times: full-image
    oracle for Sobel, sampled rows for Laplace and Harris."""
    n = 4096
    img = synth.structured_u8(n, n, synth.CONFIG_SEEDS["cfg3"])
    rng = np.random.default_rng(3)
    rows = sorted({0, 1, 2, 31, 32, n - 33, n - 32, n - 2, n - 1} | {int(r) for r in rng.integers(0, n, 24)})
    d = dev(img)
    dx = torch.empty((n, n), dtype=torch.int16, device="cuda")
    dy = torch.empty_like(dx)
    mag, lap, har = isp.isp_pipeline_cfg3_u8(d, "mirror", dx=dx, dy=dy)
    rdx, rdy, rmag = oracle.sobel(img, "mirror", threads=8)
    np.testing.assert_array_equal(host(dx), rdx)
    np.testing.assert_array_equal(host(dy), rdy)
    np.testing.assert_array_equal(host(mag), rmag)
    np.testing.assert_array_equal(host(lap)[rows], oracle.laplace5_u8(img, "mirror", rows=rows))
    np.testing.assert_array_equal(host(har)[rows], oracle.harris(rdx, rdy, "mirror", rows=rows))


@pytest.mark.parametrize("variant", ["tma", "warp"])
@pytest.mark.parametrize("shape", [(70, 2064), (100, 1040), (66, 272), (129, 4112)])
@pytest.mark.parametrize("kind", ["structured", "noise"])
def test_fused_tile_isp_kernel(isp, shape, kind, variant):
    """The band kernel (tma: k_fused_band, remapped Harris ext by edge-lane permutes and ring
    copies) and the tile-ISP kernel (warp: k_fused_body, Body tiles unchecked, border tiles
    staged through the pattern with the ext fix-up at remapped coordinates) on aligned
    images with partial right / bottom strips and tiles: every output bit-exact against the
    oracle composition, all modes, several thresholds (the f32 Harris path with its exact
    f64 fallback)."""
    h, w = shape
    img = synth.structured_u8(h, w, 8) if kind == "structured" else synth.uniform_u8(h, w, 8)
    d = dev(img)
    for mode in MODES:
        hc = -1020 if mode == "constant" else 0
        for thr in ([0, 10 ** 9] if kind == "noise" else [0, -(10 ** 6), 10 ** 12]):
            rdx, rdy, rmag, rlap, rhar = composition(img, mode, 17, hc, thr)
            dx = torch.empty((h, w), dtype=torch.int16, device="cuda")
            dy = torch.empty_like(dx)
            mag, lap, har = isp.isp_pipeline_cfg3_u8(d, mode, 17, hc, thr, dx=dx, dy=dy, variant=variant)
            for name, got, ref in [("dx", dx, rdx), ("dy", dy, rdy), ("mag", mag, rmag), ("lap", lap, rlap),
                                   ("harris", har, rhar)]:
                np.testing.assert_array_equal(host(got), ref, err_msg=f"{name} {mode} {thr} {shape} {kind}")


def _r25(dx, dy, mode, c, y, x):
    """Exact R25 at (y, x) in Python integers, the dx / dy IMAGES read through the oracle's
    border map (Constant: the Harris constant outside)."""
    h, w = dx.shape
    wts = [1, 2, 1]
    sxx = syy = sxy = 0
    for j in range(3):
        for i in range(3):
            yy, xx = oracle.border_index(mode, y + j - 1, h), oracle.border_index(mode, x + i - 1, w)
            gx, gy = (c, c) if (yy < 0 or xx < 0) else (int(dx[yy, xx]), int(dy[yy, xx]))
            sxx += wts[j] * wts[i] * gx * gx
            syy += wts[j] * wts[i] * gy * gy
            sxy += wts[j] * wts[i] * gx * gy
    return 25 * (sxx * syy - sxy * sxy) - (sxx + syy) ** 2


def test_fused_band_pitched_and_threshold_boundary(isp):
    """The band kernel on a pitched image (w = 336 of a 352-byte pitch, outputs pitched too)
    and Harris thresholds at R-1, R, R+1 of chosen pixels (including border ones whose
    window reads remapped dx / dy): exact decisions and nothing written past the width."""
    h, w, pitch = 61, 336, 352
    img = synth.uniform_u8(h, w, 19)
    d = dev(synth.pitched(img, pitch, 99))
    for mode in MODES:
        hc = 1020 if mode == "constant" else 0
        rdx, rdy, rmag, rlap, _ = composition(img, mode, 5, hc, 0)
        for (y, x) in [(0, 0), (h - 1, w - 1), (30, 170), (1, w - 2)]:
            R = _r25(rdx, rdy, mode, hc, y, x)
            for thr in (R - 1, R, R + 1):
                mag = torch.zeros((h, pitch), dtype=torch.uint8, device="cuda")
                lap, har = torch.zeros_like(mag), torch.zeros_like(mag)
                isp.isp_pipeline_cfg3_u8(d, mode, 5, hc, thr, mag=mag, lap=lap, harris=har, w=w, variant="tma")
                ref = oracle.harris(rdx, rdy, mode, hc, thr)
                np.testing.assert_array_equal(host(har)[:, :w], ref, err_msg=f"harris {mode} thr={thr}")
                assert host(har)[y, x] == (255 if R > thr else 0)
                np.testing.assert_array_equal(host(mag)[:, :w], rmag, err_msg=f"mag {mode}")
                np.testing.assert_array_equal(host(lap)[:, :w], rlap, err_msg=f"lap {mode}")
                assert not host(mag)[:, w:].any() and not host(har)[:, w:].any()
