"""C-ABI library checks that need no GPU: libisp.so loads, exports every symbol that
include/isp.h declares, validates arguments before touching the device, and its
pure-host planner / model / shard schedule agree with the oracle's planner
(oracle/planner.py, pinned in test_planner_oracle.py)."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_ipps_qiaoth21_b200 as isp
from oracle import planner as P

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    txt = open(os.path.join(ROOT, "include", "isp.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(isp_\w+)\s*\(", txt)))


def test_library_exports_every_declared_symbol():
    L = isp.lib()
    syms = declared_symbols()
    assert len(syms) >= 25
    missing = [s for s in syms if not hasattr(L, s)]
    assert not missing, missing
    assert L.isp_version() == 1


FAKE_IN, FAKE_OUT = 1 << 40, 1 << 41   # never dereferenced: validation fails first


def call_filter(w=16, h=16, pitch=16, mw=3, mh=3, mode=0, out=FAKE_OUT, inp=FAKE_IN, out_pitch=None):
    m = (ctypes.c_float * (max(mw, 1) * max(mh, 1)))()
    return isp.lib().isp_filter_ex(inp, w, h, pitch, m, mw, mh, mode, 0.0, out,
                                   pitch if out_pitch is None else out_pitch, 0, None)


@pytest.mark.parametrize("kw", [dict(mw=4), dict(mh=0), dict(mw=33), dict(mode=4), dict(mode=-1), dict(w=0),
                                dict(h=0), dict(pitch=8), dict(out_pitch=8)])
def test_einval(kw):
    assert call_filter(**kw) == 1          # ISP_EINVAL
    assert isp.lib().isp_last_error()


def test_ealias():
    assert call_filter(inp=FAKE_IN, out=FAKE_IN + 64) == 3   # ISP_EALIAS
    assert b"overlap" in isp.lib().isp_last_error()


def test_u8_validation():
    L = isp.lib()
    m = (ctypes.c_int32 * 9)()
    assert L.isp_filter_u8(FAKE_IN, 8, 8, 8, m, 3, 3, 0, 0, 0, FAKE_OUT, 8, 0, None) == 1     # divisor 0
    assert L.isp_filter_u8(FAKE_IN, 8, 8, 8, m, 3, 3, 16, 3, 300, FAKE_OUT, 8, 0, None) == 1  # constant 300
    assert L.isp_atrous_f32(FAKE_IN, 8, 8, 8, 3, 0, 0.0, 0, FAKE_OUT, 8, 0, None) == 2       # dilation 3
    assert L.isp_bilateral_f32(FAKE_IN, 8, 8, 8, 5, 0.0, 0.1, 0, 0.0, FAKE_OUT, 8, 0, None) == 1


@pytest.mark.parametrize("w,h,m,n,tw,th,ww", [(4096, 4096, 5, 5, 512, 32, 128), (64, 64, 3, 3, 64, 8, 64),
                                              (64, 64, 3, 3, 32, 8, 32), (1001, 777, 7, 7, 512, 16, 128),
                                              (2048, 2048, 13, 13, 512, 32, 128), (100, 77, 7, 3, 16, 8, 8),
                                              (9, 9, 31, 31, 32, 8, 32)])
def test_plan_matches_oracle(w, h, m, n, tw, th, ww):
    got = isp.isp_plan(w, h, m, n, tile_w=tw, tile_h=th, warp_w=ww)
    b = P.bounds(w, h, m, n, tw, th)
    wb = P.warp_bounds(w, m, ww)
    assert (got["bh_l"], got["bh_r"], got["bh_t"], got["bh_b"]) == (b["BH_L"], b["BH_R"], b["BH_T"], b["BH_B"])
    assert (got["nx"], got["ny"]) == (b["NX"], b["NY"])
    assert (got["w_l"], got["w_r"]) == (wb["W_L"], wb["W_R"])
    assert bool(got["degenerate"]) == b["degenerate"]
    if not b["degenerate"]:
        nb = P.n_block(b)
        assert got["n_block"] == [nb[r] for r in P.REGIONS]


@pytest.mark.parametrize("form", [0, 1])
def test_model_matches_oracle(form):
    mp = isp.ModelParams(4.0, 20.0, 2.0, 0.75, 0.5, form)
    for (w, m, tw, th) in [(512, 13, 32, 4), (2048, 13, 128, 1), (4096, 5, 512, 32)]:
        got = isp.isp_plan(w, w, m, m, tile_w=tw, tile_h=th, warp_w=tw, params=mp)
        ref = P.model(w, w, m, m, tw, th, 4.0, 20.0, o_naive=0.75, o_isp=0.5, ipc_switch=2.0,
                      form="P" if form else "T", threads_per_block=32)
        for k_got, k_ref in [("n_naive", "N_naive"), ("n_isp", "N_ISP"), ("r_reduced", "R_reduced"), ("g", "G")]:
            assert got[k_got] == pytest.approx(ref[k_ref], rel=1e-12)
        assert (got["choice"] != 3) == (ref["choice"] == "isp")


def test_shard_rows_partition():
    for H in (1, 7, 64, 4096, 16384, 1001):
        for Pn in (1, 2, 3, 4, 8):
            if H < Pn:
                continue
            rows = [isp.isp_shard_rows(H, r, Pn) for r in range(Pn)]
            assert rows[0][0] == 0
            for (a, n), (b, _) in zip(rows, rows[1:]):
                assert a + n == b
            assert rows[-1][0] + rows[-1][1] == H


@pytest.mark.parametrize("mode", [0, 1, 2, 3])
@pytest.mark.parametrize("Pn", [1, 2, 3, 8])
def test_shard_schedule(mode, Pn):
    H, halo, hy = 512, 4, 3
    sc = [isp.isp_shard_schedule(H, r, Pn, halo, hy, mode) for r in range(Pn)]
    ring = mode == isp.REPEAT and Pn > 1
    sends, recvs = {}, {}
    for r, s in enumerate(sc):
        # launches tile the strip exactly, each launch's reads stay resident
        cover = sorted((l[0], l[0] + l[1]) for l in s["launch"] if l[1] > 0)
        assert cover[0][0] == s["y0"] and cover[-1][1] == s["y0"] + s["strip_h"]
        for (a0, a1), (b0, _) in zip(cover, cover[1:]):
            assert a1 == b0
        for (oy0, n, ylim, t_real, b_real, after) in s["launch"]:
            assert ylim <= s["y0"] + s["strip_h"] + (hy if s["next"] >= 0 else 0)
            if not after:   # overlapped with the exchange: must not read halo rows
                assert ylim <= s["y0"] + s["strip_h"]
                assert t_real or oy0 - hy >= s["y0"]
        assert (s["prev"] >= 0) == (r > 0 or ring)
        assert (s["next"] >= 0) == (r < Pn - 1 or ring)
        for kind, peer, row, n in s["ops"]:
            (sends if kind == 0 else recvs).setdefault((r, peer) if kind == 0 else (peer, r), []).append((row, n))
    # every send is matched, in order, by a receive of the same size on the peer
    assert sends.keys() == recvs.keys()
    for key in sends:
        assert [n for _, n in sends[key]] == [n for _, n in recvs[key]]


def test_pipeline_cfg3_validation():
    """isp_pipeline_cfg3_u8 argument checks (include/isp.h) fail before any device work."""
    L = isp.lib()
    F = FAKE_OUT

    def call(w=64, h=64, pitch=64, mode=1, c=0, hc=0, mag=F, lap=F + (1 << 20), har=F + (2 << 20), dx=None,
             op=64, inp=FAKE_IN):
        return L.isp_pipeline_cfg3_u8(inp, w, h, pitch, mode, c, hc, 0, dx, None, mag, lap, har, op, 0, None)
    assert call(w=0) == 1 and call(pitch=32) == 1 and call(op=32) == 1 and call(mode=4) == 1
    assert call(mag=None) == 1 and call(lap=None) == 1 and call(har=None) == 1
    assert call(c=256) == 1 and call(c=-1) == 1
    assert call(hc=1021) == 1 and call(hc=-1021) == 1       # outside the Sobel range
    assert call(mag=FAKE_IN + 100) == 3                     # EALIAS
    assert call(dx=FAKE_IN + 64 * 63) == 3                  # int16 output overlapping the image tail


def _balanced_y0s(h, ny, edge_w=64):
    """Block-row starts of the library's balanced one-wave split (isp_core.cuh block_rows:
    the first and last strip carry edge_w/256 of an interior strip's rows) -- the launch
    geometry the model is evaluated on, restated here independently of the library."""
    if ny <= 2:
        return [(by * h) // ny for by in range(ny + 1)]
    W = 2 * edge_w + 256 * (ny - 2)

    def cum(k):
        return 0 if k == 0 else W if k == ny else edge_w + 256 * (k - 1)
    return [(cum(k) * h) // W for k in range(ny + 1)]


@pytest.mark.parametrize("w,h,m", [(4096, 4096, 5), (2048, 1000, 7), (1000, 4096, 13), (4096, 512, 3)])
@pytest.mark.parametrize("form", [0, 1, 2, 3])
def test_model_balanced_split_matches_oracle(w, h, m, form):
    """Balanced one-wave plans (tile_h = 0): bounds from the real block-row starts and the
    model counting each block's real rows (round-1 counted 0 pixels per block there)."""
    mp = isp.ModelParams(4.0, 20.0, 2.0, 0.75, 0.5, form)
    got = isp.isp_plan(w, h, m, m, tile_w=512, tile_h=0, warp_w=512, params=mp)
    y0s = _balanced_y0s(h, got["ny"])
    b = P.bounds_rows(w, h, m, m, 512, y0s)
    assert (got["bh_t"], got["bh_b"], got["nx"], got["ny"]) == (b["BH_T"], b["BH_B"], b["NX"], b["NY"])
    ref = P.model(w, h, m, m, 512, None, 4.0, 20.0, o_naive=0.75, o_isp=0.5, ipc_switch=2.0,
                  form="TPSB"[form], threads_per_block=32, y0s=y0s)
    for k_got, k_ref in [("n_naive", "N_naive"), ("n_isp", "N_ISP"), ("r_reduced", "R_reduced"), ("g", "G")]:
        assert got[k_got] == pytest.approx(ref[k_ref], rel=1e-12), k_got
    assert got["n_isp"] > 0 and got["g"] < 100      # round 1: pix = 0 made G ~ 855


@pytest.mark.parametrize("form", [2, 3])
def test_model_form_s_matches_oracle(form):
    """Forms S (staged, A21) and B (band, A34) of the C model against the oracle planner."""
    mp = isp.ModelParams(4.0, 20.0, 2.0, 0.75, 0.5, form)
    for (w, m, tw, th) in [(512, 13, 32, 4), (2048, 13, 128, 1), (4096, 5, 512, 32), (4096, 7, 1024, 16),
                           (4096, 5, 128, 19), (1000, 3, 128, 7)]:
        got = isp.isp_plan(w, w, m, m, tile_w=tw, tile_h=th, warp_w=tw, params=mp)
        ref = P.model(w, w, m, m, tw, th, 4.0, 20.0, o_naive=0.75, o_isp=0.5, ipc_switch=2.0, form="SB"[form - 2],
                      threads_per_block=32)
        assert got["n_isp"] == pytest.approx(ref["N_ISP"], rel=1e-12)
        assert got["g"] == pytest.approx(ref["G"], rel=1e-12)


# ---------------------------------------------------------------- N3: sparse masks (reading A31)
def _sparse_masks(rng, n=40):
    out = []
    for _ in range(n):
        m, k = int(rng.choice([3, 5, 7, 9, 13])), int(rng.choice([1, 3, 5, 7, 9]))
        mask = np.where(rng.random((k, m)) < 0.4, rng.standard_normal((k, m)), 0.0)
        mask[:, : int(rng.integers(0, m // 2 + 1))] = 0
        mask[k - int(rng.integers(0, k // 2 + 1)):, :] = 0
        out.append(mask)
    return out


def test_mask_reach_matches_oracle():
    rng = np.random.default_rng(21)
    for mask in _sparse_masks(rng):
        assert isp.isp_mask_reach(mask.astype(np.float32)) == P.mask_reach(mask)
        assert isp.isp_mask_reach(np.sign(mask).astype(np.int32)) == P.mask_reach(mask)


def test_plan_reach_matches_oracle():
    rng = np.random.default_rng(22)
    for mask in _sparse_masks(rng):
        r = P.mask_reach(mask)
        for (w, h, tw, th) in [(4096, 4096, 512, 16), (300, 77, 128, 4), (40, 33, 32, 8)]:
            got = isp.isp_plan_reach(w, h, r, tw, th)
            b = P.bounds_reach(w, h, r, tw, th)
            assert (got["bh_l"], got["bh_r"], got["bh_t"], got["bh_b"], got["nx"], got["ny"]) == \
                (b["BH_L"], b["BH_R"], b["BH_T"], b["BH_B"], b["NX"], b["NY"])
            assert bool(got["degenerate"]) == b["degenerate"]
