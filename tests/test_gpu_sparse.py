"""GPU parity of sparse / irregular masks (the paper's future work
P:L394; reading A31): masks with all-zero edge rows / columns are cropped to their
non-zero footprint and the ISP bounds come from the footprint's reach on each side.

Checked against the oracle evaluated with the FULL (uncropped) mask -- zero taps add
exactly 0, so the oracle needs no notion of footprints -- at A28 (f32) / bit-exact (u8),
every border mode and variant, with the plan asserted: non-degenerate, the requested
variant, and Eq. (2) bounds equal to oracle/planner.bounds_reach for the plan's tile.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from oracle import planner as P

pytestmark = pytest.mark.gpu

MODES = ["clamp", "mirror", "repeat", "constant"]
CODE = {"auto": 0, "block": 1, "warp": 2, "naive": 3, "tma": 4}


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


def sparse_masks():
    rng = np.random.default_rng(31)
    out = {}
    m = rng.standard_normal((9, 9)).astype(np.float32)
    m[:, :5] = 0                                    # right half only: reach L = 0, R = 4
    out["right_half_9"] = m
    m = rng.standard_normal((7, 7)).astype(np.float32)
    m[:3, :] = 0                                    # bottom part: reach T = 0
    out["bottom_7"] = m
    m = np.zeros((7, 7), np.float32)
    m[1:6, 1:6] = rng.standard_normal((5, 5))       # zero ring: centred 5x5 (compiled path)
    out["ring_7to5"] = m
    m = np.zeros((13, 13), np.float32)
    m[6, 9:13] = rng.standard_normal(4)             # one row right of the centre (anchor outside)
    out["row_right_13"] = m
    m = np.zeros((5, 5), np.float32)
    m[0, 0], m[4, 1] = 1.0, -2.0                    # irregular corners
    out["corners_5"] = m
    return out


def check_plan(isp, v, shape, reach, want_choice=None):
    p = isp.isp_last_plan()
    assert not p["degenerate"], p
    if want_choice is not None:
        assert p["choice"] == want_choice, p
    h, w = shape
    b = P.bounds_reach(w, h, reach, p["tile_w"], max(p["tile_h"], 1))
    if p["choice"] in (1, 2, 3):      # uniform-tile plans: Eq. 2 with the footprint
        assert (p["bh_l"], p["bh_r"]) == (b["BH_L"], b["BH_R"]), (p, b)


@pytest.mark.parametrize("name", list(sparse_masks().keys()))
def test_sparse_f32(isp, name):
    mask = sparse_masks()[name]
    h, w = 70, 2052
    img = synth.uniform_f32(h, w, 61)
    d = dev(img)
    reach = P.mask_reach(mask)
    assert isp.isp_mask_reach(mask) == reach
    for mode in MODES:
        ref, sc = oracle.filter_f64(img, mask, mode, 0.25, with_scale=True)
        outs = {}
        for v in ["naive", "block", "warp", "tma", "auto"]:
            outs[v] = host(isp.isp_filter_ex(d, mask, mode, 0.25, variant=v))
            check_plan(isp, v, (h, w), reach, None if v in ("auto", "tma") else CODE[v])
            check_f32(outs[v], ref, sc)
        for v, o in outs.items():
            np.testing.assert_array_equal(o, outs["naive"], err_msg=f"{v} {mode} {name}")


def test_ring_crop_runs_compiled_window(isp):
    """A 7x7 mask with a zero ring is the 5x5 mask: same bits, compiled 5x5 kernels."""
    mask7 = sparse_masks()["ring_7to5"]
    mask5 = np.ascontiguousarray(mask7[1:6, 1:6])
    img = synth.uniform_f32(45, 4100, 3)
    d = dev(img)
    for mode in MODES:
        for v in ["tma", "warp", "naive"]:
            a = host(isp.isp_filter_ex(d, mask7, mode, 0.5, variant=v))
            pa = isp.isp_last_plan()
            b = host(isp.isp_filter_ex(d, mask5, mode, 0.5, variant=v))
            pb = isp.isp_last_plan()
            np.testing.assert_array_equal(a, b)
            assert pa == pb


@pytest.mark.parametrize("name", ["right_half_9", "bottom_7", "corners_5"])
def test_sparse_u8(isp, name):
    mask = np.rint(sparse_masks()[name] * 4).astype(np.int32)
    div = int(max(1, np.abs(mask).sum()))
    h, w = 70, 2064
    img = synth.uniform_u8(h, w, 62)
    d = dev(img)
    reach = P.mask_reach(mask)
    for mode in MODES:
        ref = oracle.filter_u8(img, mask, div, mode, 9)
        for v in ["naive", "block", "warp", "auto"]:
            got = host(isp.isp_filter_u8(d, mask, div, mode, 9, variant=v))
            check_plan(isp, v, (h, w), reach, None if v == "auto" else CODE[v])
            np.testing.assert_array_equal(got, ref, err_msg=f"{name} {mode} {v}")
