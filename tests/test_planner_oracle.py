"""Pins for the planner oracle (oracle/planner.py): Eqs. (2), (7), (8), Listings 3/5, model.

Independent references: per-block brute force over every thread x tap (which checks a
block really needs), the paper's Listings 3 and 5 transcribed verbatim into
tests/golden/ and executed literally, and closed-form limits of the model.
"""
import os
import re

import numpy as np
import pytest

from oracle import planner as P

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _compile_listing(path):
    """Turn the transcribed CUDA listing into a Python function region(bx, by, wid, env)."""
    lines = [l.rstrip() for l in open(path) if l.strip() and not l.lstrip().startswith("#")]
    py = ["def region(bx, by, wid, BH_L, BH_R, BH_T, BH_B, W_L, W_R):"]
    # An `if (c)` without a same-line goto governs the following indented lines (Listing 5's
    # layout) or, if the next line is not indented, that single next line (Listing 3's).
    pending_single = False
    for k, l in enumerate(lines):
        ind = len(l) - len(l.lstrip())
        s = l.strip()
        s = s.replace("blockIdx.x", "bx").replace("blockIdx.y", "by").replace("warpID.x", "wid")
        s = s.replace("&&", "and")
        depth = 1 + (1 if ind > 0 else 0) + (1 if pending_single else 0)
        pending_single = False
        m = re.match(r"if \((.*)\)\s*(goto (\w+);)?$", s)
        if m:
            cond, tgt = m.group(1), m.group(3)
            if tgt:
                py.append("    " * depth + f"if {cond}: return '{tgt}'")
            else:
                py.append("    " * depth + f"if {cond}:")
                nxt = lines[k + 1]
                pending_single = (len(nxt) - len(nxt.lstrip())) <= ind
            continue
        m = re.match(r"goto (\w+);$", s)
        assert m, s
        py.append("    " * depth + f"return '{m.group(1)}'")
    env = {}
    exec("\n".join(py), env)
    return env["region"]


LISTING3 = _compile_listing(os.path.join(GOLDEN, "listing3.txt"))
LISTING5 = _compile_listing(os.path.join(GOLDEN, "listing5.txt"))

SHAPES = [(sx, sy, m, n, tx, ty)
          for (sx, sy) in [(7, 5), (16, 16), (23, 19), (39, 11)]
          for (m, n) in [(1, 1), (3, 3), (5, 3), (7, 9)]
          for (tx, ty) in [(1, 1), (4, 2), (8, 4), (16, 1)]]


@pytest.mark.parametrize("sx,sy,m,n,tx,ty", SHAPES)
def test_bounds_exact_vs_bruteforce(sx, sy, m, n, tx, ty):
    """Eq. (2) (reading A2) is conservative AND tight: a block needs the L check iff
    bx < BH_L, R iff bx >= BH_R, T iff by < BH_T, B iff by >= BH_B."""
    b = P.bounds(sx, sy, m, n, tx, ty)
    for by in range(b["NY"]):
        for bx in range(b["NX"]):
            need = P.needed_sides_bruteforce(sx, sy, m, n, tx, ty, bx, by)
            assert ("L" in need) == (bx < b["BH_L"])
            assert ("R" in need) == (bx >= b["BH_R"])
            assert ("T" in need) == (by < b["BH_T"])
            assert ("B" in need) == (by >= b["BH_B"])
            if not b["degenerate"]:
                reg, _ = P.listing3(bx, by, b)
                assert need <= P.REGION_SIDES[reg]
                assert need == P.REGION_SIDES[reg]          # and no superfluous check


def test_printed_eq2_misses_checks():
    """The literal Eq. (2) puts block 0 in Body for m=5, tx=32 although it
    needs the left check -- the reason for reading A2."""
    sx = sy = 128
    bp = P.bounds_printed(sx, sy, 5, 5, 32, 32)
    assert bp["BH_L"] == 0
    assert "L" in P.needed_sides_bruteforce(sx, sy, 5, 5, 32, 32, 0, 1)
    assert P.bounds(sx, sy, 5, 5, 32, 32)["BH_L"] == 1


def test_degenerate_flag():
    # cfg1 with a 64-wide tile: one block needs both the L and R check (A3).
    b = P.bounds(64, 64, 3, 3, 64, 8)
    assert b["degenerate"] and b["BH_R"] < b["BH_L"]
    assert not P.bounds(64, 64, 3, 3, 32, 8)["degenerate"]


@pytest.mark.parametrize("sx,sy,m,n,tx,ty", [s for s in SHAPES if not P.bounds(*s)["degenerate"]])
def test_listing3_matches_paper_text(sx, sy, m, n, tx, ty):
    b = P.bounds(sx, sy, m, n, tx, ty)
    for by in range(b["NY"]):
        for bx in range(b["NX"]):
            assert P.listing3(bx, by, b)[0] == LISTING3(bx, by, 0, b["BH_L"], b["BH_R"], b["BH_T"],
                                                        b["BH_B"], 0, 0)


@pytest.mark.parametrize("sx,sy,m,n,tx,ty", [s for s in SHAPES if not P.bounds(*s)["degenerate"]])
def test_eq8_counts(sx, sy, m, n, tx, ty):
    """Eq. (8a)/(8b) (reading A17) equal a Listing 3 enumeration; they sum to N_block (Eq. 7)."""
    b = P.bounds(sx, sy, m, n, tx, ty)
    nb = P.n_block(b)
    assert nb == P.n_block_enumerated(b)
    assert sum(nb.values()) == b["NX"] * b["NY"]
    assert all(v >= 0 for v in nb.values())


def test_n_switch_table():
    """Compares evaluated by Listing 3 under C short-circuit rules (A18)."""
    assert P.n_switch_table() == {"TL": 2, "TR": 3, "T": 3, "BL": 6, "BR": 8, "B": 8, "R": 8,
                                  "L": 9, "Body": 8}


@pytest.mark.parametrize("sx,wx,m", [(512, 32, 3), (100, 8, 5), (77, 4, 7), (64, 16, 9), (256, 128, 31)])
def test_warp_bounds_vs_bruteforce(sx, wx, m):
    """Warp-grained bounds (a3/A22): warp column g needs L iff g < W_L, R iff g >= W_R."""
    wb = P.warp_bounds(sx, m, wx)
    hx = m // 2
    for g in range(-(-sx // wx)):
        xs = range(g * wx, (g + 1) * wx)           # launched threads (A10)
        need_l = any(x - hx < 0 for x in xs)
        need_r = any(x + hx >= sx for x in xs)
        assert need_l == (g < wb["W_L"])
        assert need_r == (g >= wb["W_R"])


@pytest.mark.parametrize("sx,sy,m,n,tx,ty,wx", [(512, 64, 3, 3, 128, 4, 32), (300, 40, 5, 5, 64, 8, 16),
                                                (1000, 30, 7, 3, 256, 2, 64), (96, 96, 9, 9, 32, 8, 8)])
def test_listing5_matches_paper_and_is_safe(sx, sy, m, n, tx, ty, wx):
    """Listing 5 evaluated on global warp columns: the paper's text and the
    oracle agree, and each warp's region covers every check its pixels really need."""
    b = P.bounds(sx, sy, m, n, tx, ty)
    assert not b["degenerate"]
    wb = P.warp_bounds(sx, m, wx)
    wpb = tx // wx
    hx, hy = m // 2, n // 2
    for by in range(b["NY"]):
        for bx in range(b["NX"]):
            for w in range(wpb):
                g = bx * wpb + w
                reg, _ = P.listing5(bx, by, g, b, wb)
                # golden text uses `warpID.x > W_L` with W_L = last checked warp (A22)
                assert reg == LISTING5(bx, by, g, b["BH_L"], b["BH_R"], b["BH_T"], b["BH_B"],
                                       wb["W_L"] - 1, wb["W_R"])
                need = set()
                for y in range(by * ty, (by + 1) * ty):      # launched threads (A10)
                    for x in range(g * wx, (g + 1) * wx):
                        if x - hx < 0: need.add("L")
                        if x + hx >= sx: need.add("R")
                        if y - hy < 0: need.add("T")
                        if y + hy >= sy: need.add("B")
                assert need <= P.REGION_SIDES[reg], (bx, by, w, reg, need)


def test_listing5_paper_example():
    """block of 128 threads = 4 warps, 3x3 operator: only the leftmost warp needs the
    left check and only the rightmost the right check (one pixel per thread, wx = 32)."""
    sx, sy = 512, 64
    b = P.bounds(sx, sy, 3, 3, 128, 1)
    wb = P.warp_bounds(sx, 3, 32)
    regs = [P.listing5(g // 4, 5, g, b, wb)[0] for g in range(16)]
    assert regs[0] == "L" and regs[-1] == "R" and set(regs[1:-1]) == {"Body"}
    assert [P.listing3(g // 4, 5, b)[0] for g in range(16)][:4] == ["L"] * 4


def test_fig3_trend():
    """Fig. 3 / P:L173: for a 5x5 operator, smaller images have a lower share of Body blocks,
    and a larger block leaves fewer Body blocks at the same size."""
    for tile in [(32, 4), (128, 1), (128, 16)]:
        fr = [P.body_fraction(s, s, 5, 5, *tile) for s in (512, 1024, 2048, 4096)]
        assert fr == sorted(fr) and fr[0] < fr[-1] < 1.0
    assert P.body_fraction(512, 512, 5, 5, 256, 16) < P.body_fraction(512, 512, 5, 5, 32, 4)


def test_model_limits():
    """Eq. (9)/(10) limits: with a 1-pixel image border share -> 0, form T gives
    R -> (4c+k) m n / (ipc * n_sw(Body) + k m n) (threads = tx ty), approached monotonically;
    G scales with O_ISP / O_naive."""
    c, k, ipc = 4.0, 20.0, 2.0
    m = n = 13
    limit = (4 * c + k) * m * n / (ipc * 8 + k * m * n)
    rs = [P.model(s, s, m, n, 32, 4, c, k, ipc_switch=ipc)["R_reduced"] for s in (512, 1024, 2048, 4096, 16384)]
    assert rs == sorted(rs) and abs(rs[-1] - limit) / limit < 0.01 and rs[-1] < limit
    g = P.model(2048, 2048, m, n, 32, 4, c, k, o_naive=1.0, o_isp=0.5, ipc_switch=ipc)
    assert abs(g["G"] - 0.5 * g["R_reduced"]) < 1e-12
    # form P (switch charged per tap) predicts R ~ 1 for this calibration (reading A14)
    rp = P.model(4096, 4096, m, n, 32, 4, c, k, ipc_switch=ipc, form="P")["R_reduced"]
    assert abs(rp - (4 * c + k) / (ipc * 8 + k)) / rp < 0.02
    assert P.model(64, 64, 3, 3, 64, 8, c, k)["choice"] == "naive"      # degenerate


# ---------------------------------------------------------------- block rows of any height
def _needed_rows_bruteforce(sx, sy, m, n, tx, y0, y1, bx):
    """Which checks block (bx, rows [y0, y1)) needs: every launched thread x every tap."""
    hx, hy = m // 2, n // 2
    need = set()
    for y in range(y0, y1):
        for x in range(bx * tx, (bx + 1) * tx):
            for j in range(n):
                for i in range(m):
                    xx, yy = x + i - hx, y + j - hy
                    if xx < 0:
                        need.add("L")
                    if xx >= sx:
                        need.add("R")
                    if yy < 0:
                        need.add("T")
                    if yy >= sy:
                        need.add("B")
    return need


def test_bounds_rows_bruteforce():
    """bounds_rows (Eq. 2 for block rows of any height, e.g. the balanced one-wave split)
    is conservative and tight against per-thread enumeration: a block row < BH_T needs
    the T check and none >= BH_T does; likewise B."""
    rng = np.random.default_rng(3)
    for _ in range(60):
        sy = int(rng.integers(4, 40))
        n = int(rng.choice([1, 3, 5, 7]))
        cuts = sorted(set(int(c) for c in rng.integers(1, sy, int(rng.integers(1, 6)))))
        y0s = [0] + cuts + [sy]
        sx, m, tx = 8, 3, 8
        b = P.bounds_rows(sx, sy, m, n, tx, y0s)
        for by in range(len(y0s) - 1):
            need = _needed_rows_bruteforce(sx, sy, m, n, tx, y0s[by], y0s[by + 1], 0)
            assert ("T" in need) == (by < b["BH_T"]), (y0s, n, by, b)
            assert ("B" in need) == (by >= b["BH_B"]), (y0s, n, by, b)


@pytest.mark.parametrize("sx,sy,m,tx,ty", [(512, 512, 13, 32, 4), (300, 77, 5, 64, 8), (4096, 4096, 5, 512, 32)])
def test_bounds_rows_uniform_equals_eq2(sx, sy, m, tx, ty):
    NY = -(-sy // ty)
    y0s = [min(sy, by * ty) for by in range(NY + 1)]
    b, bu = P.bounds_rows(sx, sy, m, m, tx, y0s), P.bounds(sx, sy, m, m, tx, ty)
    # identical except where the uniform model's last partial tile ends past the image
    assert {k: b[k] for k in ("BH_L", "BH_R", "BH_T", "NX", "NY")} == {k: bu[k] for k in ("BH_L", "BH_R", "BH_T", "NX", "NY")}
    assert b["BH_B"] == bu["BH_B"] or (sy % ty and b["BH_B"] >= bu["BH_B"])


def test_model_rows_reduces_to_printed_form():
    """y0s of uniform full tiles give exactly the printed Eq. (5) sum."""
    for (s, m, tx, ty) in [(512, 13, 32, 4), (1024, 5, 128, 8)]:
        y0s = [by * ty for by in range(s // ty + 1)]
        for form in ("T", "P", "S"):
            a = P.model(s, s, m, m, tx, ty, 4.0, 20.0, form=form, threads_per_block=32)
            b = P.model(s, s, m, m, tx, ty, 4.0, 20.0, form=form, threads_per_block=32, y0s=y0s)
            assert a["N_ISP"] == pytest.approx(b["N_ISP"], rel=1e-12)


def test_model_form_s_closed_form():
    """Form S (reading A21) on a 3x3-block image: 8 border blocks (4 corners x 2 checks,
    4 edges x 1) pay n_check per staged element (tx+2hx)(ty+2hy); Body pays none;
    with n_check = 0 it equals form T with n_check = 0."""
    sx = sy = 48
    m = n = 5
    tx = ty = 16
    c, k, ipc, thr = 3.0, 7.0, 2.0, 64
    got = P.model(sx, sy, m, n, tx, ty, c, k, ipc_switch=ipc, form="S", threads_per_block=thr)
    sw = P.n_switch_table()
    E = (tx + 4) * (ty + 4)
    want = sum(sw[r] * ipc * thr for r in P.REGIONS) + (4 * 2 + 4 * 1) * c * E + 9 * k * m * n * tx * ty
    assert got["N_ISP"] == pytest.approx(want, rel=1e-12)
    a = P.model(sx, sy, m, n, tx, ty, 0.0, k, form="S", threads_per_block=thr)
    b = P.model(sx, sy, m, n, tx, ty, 0.0, k, form="T", threads_per_block=thr)
    assert a["N_ISP"] == pytest.approx(b["N_ISP"], rel=1e-12)


def test_model_form_b_closed_form():
    """Form B (reading A34, band kernels) on a 3x3-block image: the 8 border blocks pay
    n_check per STAGED ROW (ty + 2hy) per thread for each checked side (corners 2, edges 1),
    Body none -- written out by hand; and an 8x8 image of 2x2 corner blocks counted term by
    term (A18 switch costs TL 2, TR 3, BL 6, BR 8)."""
    sx = sy = 48
    m = n = 5
    tx = ty = 16
    c, k, ipc, thr = 3.0, 7.0, 2.0, 64
    got = P.model(sx, sy, m, n, tx, ty, c, k, ipc_switch=ipc, form="B", threads_per_block=thr)
    sw = P.n_switch_table()
    want = sum(sw[r] * ipc * thr for r in P.REGIONS) + (4 * 2 + 4 * 1) * c * thr * (ty + 4) + \
        9 * k * m * n * tx * ty
    assert got["N_ISP"] == pytest.approx(want, rel=1e-12)
    small = P.model(8, 8, 3, 3, 4, 4, 1.0, 1.0, ipc_switch=2.0, form="B")   # threads = tx * ty = 16
    assert small["N_ISP"] == pytest.approx((2 + 3 + 6 + 8) * 2 * 16 + 4 * 2 * 1 * 16 * 6 + 4 * 9 * 16, rel=1e-12)
    assert small["N_naive"] == 5 * 9 * 64
    # with n_check = 0 form B equals form T with n_check = 0 (only the checks differ)
    a = P.model(sx, sy, m, n, tx, ty, 0.0, k, form="B", threads_per_block=thr)
    b = P.model(sx, sy, m, n, tx, ty, 0.0, k, form="T", threads_per_block=thr)
    assert a["N_ISP"] == pytest.approx(b["N_ISP"], rel=1e-12)


# ---------------------------------------------------------------- N3: sparse masks (reading A31)
def test_mask_reach_examples():
    m = np.zeros((7, 7))
    m[3, 3] = 1
    assert P.mask_reach(m) == (0, 0, 0, 0)
    m[1, 5] = 2            # row 1 (2 above), column 5 (2 right)
    assert P.mask_reach(m) == (0, 2, 2, 0)
    m[6, 0] = -1           # row 6 (3 below), column 0 (3 left)
    assert P.mask_reach(m) == (3, 2, 2, 3)
    assert P.mask_reach(np.ones((5, 3))) == (1, 1, 2, 2)
    assert P.mask_reach(np.zeros((3, 3))) == (0, 0, 0, 0)


def test_bounds_reach_bruteforce():
    """Eq. (2) from the non-zero footprint is conservative AND tight: per-thread
    enumeration over the non-zero taps needs exactly the checks the bounds assign."""
    rng = np.random.default_rng(11)
    for _ in range(120):
        m, n = int(rng.choice([3, 5, 7, 9])), int(rng.choice([1, 3, 5, 7]))
        mask = (rng.random((n, m)) < 0.3).astype(float)
        # zero edge rows / columns on purpose
        if rng.random() < 0.5:
            mask[:, : int(rng.integers(0, m // 2 + 1))] = 0
        if rng.random() < 0.5:
            mask[: int(rng.integers(0, n // 2 + 1)), :] = 0
        sx, sy = int(rng.integers(6, 30)), int(rng.integers(6, 30))
        tx, ty = int(rng.choice([2, 4, 8])), int(rng.choice([1, 2, 4]))
        b = P.bounds_reach(sx, sy, P.mask_reach(mask), tx, ty)
        if b["degenerate"]:
            continue
        for by in range(b["NY"]):
            for bx in range(b["NX"]):
                need = P.needed_sides_mask_bruteforce(sx, sy, mask, tx, ty, bx, by)
                assert ("L" in need) == (bx < b["BH_L"])
                assert ("R" in need) == (bx >= b["BH_R"])
                assert ("T" in need) == (by < b["BH_T"])
                assert ("B" in need) == (by >= b["BH_B"])


def test_bounds_reach_dense_equals_eq2():
    for (sx, sy, m, n, tx, ty) in [(512, 512, 13, 13, 32, 4), (100, 77, 7, 3, 16, 8), (4096, 4096, 5, 5, 512, 32)]:
        hx, hy = m // 2, n // 2
        a = P.bounds_reach(sx, sy, (hx, hx, hy, hy), tx, ty)
        b = P.bounds(sx, sy, m, n, tx, ty)
        assert {k: a[k] for k in ("BH_L", "BH_R", "BH_T", "BH_B", "NX", "NY", "degenerate")} == \
               {k: b[k] for k in ("BH_L", "BH_R", "BH_T", "BH_B", "NX", "NY", "degenerate")}
