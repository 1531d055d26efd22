"""GPU parity of the two ablation variants:

  * ISP_SPLIT -- one kernel per region (P:L90 argues for ONE fat kernel): the nine region
    rectangles launched separately; same region bodies, so bitwise equal to NAIVE.
  * ISP_TEX -- texture-hardware border handling: taps read through a texture
    object whose address mode is the pattern; 2-D FMA order of the direct family.

Both against the oracle (A28 / bit-exact) in every border mode, with the plan asserted.
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


def check_f32(got, ref, scale, tol=1e-5):
    bound = tol * np.maximum(np.abs(ref), scale) + 1e-30
    err = np.abs(got.astype(np.float64) - ref)
    assert not (err > bound).any(), f"worst err {err.max():.3e}"


def binomial_f32(m):
    b = synth.binomial_row(m).astype(np.float64)
    return (np.outer(b, b) / b.sum() ** 2).astype(np.float32)


MASKS = {"binomial5": binomial_f32(5), "rand5": np.random.default_rng(5).standard_normal((5, 5)).astype(np.float32),
         "rand9": np.random.default_rng(9).standard_normal((9, 9)).astype(np.float32),
         "rand3x7": np.random.default_rng(37).standard_normal((7, 3)).astype(np.float32)}


@pytest.mark.parametrize("name", list(MASKS))
def test_split_f32(isp, name):
    mask = MASKS[name]
    img = synth.uniform_f32(70, 2052, 71)
    d = dev(img)
    for mode in MODES:
        ref, sc = oracle.filter_f64(img, mask, mode, 0.25, with_scale=True)
        naive = host(isp.isp_filter_ex(d, mask, mode, 0.25, variant="naive"))
        got = host(isp.isp_filter_ex(d, mask, mode, 0.25, variant="split"))
        p = isp.isp_last_plan()
        assert p["choice"] == isp.SPLIT and not p["degenerate"], p
        check_f32(got, ref, sc)
        np.testing.assert_array_equal(got, naive, err_msg=f"{name} {mode}")


def test_split_other_ops(isp):
    img = synth.structured_u8(70, 2064, 72)
    d = dev(img)
    g5, div = oracle.gaussian_u8_mask(5)
    for mode in MODES:
        np.testing.assert_array_equal(host(isp.isp_filter_u8(d, g5, div, mode, 5, variant="split")),
                                      oracle.filter_u8(img, g5, div, mode, 5))
        rdx, rdy, rmag = oracle.sobel(img, mode, 5)
        dx, dy, mag = isp.isp_sobel_u8(d, mode, 5, variant="split")
        assert isp.isp_last_plan()["choice"] == isp.SPLIT
        np.testing.assert_array_equal(host(mag), rmag)
        np.testing.assert_array_equal(host(isp.isp_laplace5_u8(d, mode, 5, variant="split")),
                                      oracle.laplace5_u8(img, mode, 5))
        np.testing.assert_array_equal(host(isp.isp_harris_u8(dev(rdx), dev(rdy), mode, 3, 0, variant="split")),
                                      oracle.harris(rdx, rdy, mode, 3, 0))
    f = synth.structured_f32(40, 1036, 73)
    for mode in MODES:
        ref = oracle.bilateral(f, 13, 3.0, 0.1, mode, 0.5)
        got = host(isp.isp_bilateral_f32(dev(f), 13, 3.0, 0.1, mode, 0.5, variant="split"))
        assert np.abs(got - ref).max() <= 1e-4


@pytest.mark.parametrize("name", list(MASKS))
@pytest.mark.parametrize("shape", [(70, 2048), (45, 328), (5, 8)])
def test_tex_f32(isp, name, shape):
    """Texture address modes reproduce the four patterns, windows larger than the image
    included (5x8 image, 9x9 window: wrap / mirror periods handled by the hardware).
    Widths keep rows on the device's texture pitch alignment (32 B)."""
    mask = MASKS[name]
    h, w = shape
    img = synth.uniform_f32(h, w, 74)
    d = dev(img)
    for mode in MODES:
        ref, sc = oracle.filter_f64(img, mask, mode, 0.25, with_scale=True)
        got = host(isp.isp_filter_ex(d, mask, mode, 0.25, variant="tex"))
        check_f32(got, ref, sc)


def test_tex_needs_pitch_alignment(isp):
    img = dev(synth.uniform_f32(16, 2052, 1))        # 8208-B rows: not a multiple of 32 B
    with pytest.raises(isp.IspError):
        isp.isp_filter_ex(img, MASKS["rand5"], "clamp", 0.0, variant="tex")


def test_tex_unsupported_elsewhere(isp):
    img = dev(synth.uniform_u8(16, 64, 1))
    g3, div = oracle.gaussian_u8_mask(3)
    with pytest.raises(isp.IspError):
        isp.isp_filter_u8(img, g3, div, "clamp", 0, variant="tex")
