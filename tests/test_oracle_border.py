"""Pins for the oracle's border index map B_mode(i, N) (§III.A, Fig. 2).

The oracle (oracle/isp_oracle.c, orc_border_index) is checked against things other
than itself:
  * numpy.pad's index maps: edge (Clamp), symmetric (Mirror, reading A4), wrap
    (Repeat), constant (Constant) -- a library routine, for every pad width;
  * the paper's prose definitions as invariants: Repeat "is the same as to tile the
    image with itself along x- and y-dimensions periodically" -> np.tile;
    Mirror "returns the mirrored pixels at the border" -> reflection symmetry about
    the image edges; Clamp "returns the nearest valid pixel" -> argmin distance.
"""
import numpy as np
import pytest

NP_MODE = {"clamp": "edge", "mirror": "symmetric", "repeat": "wrap"}


@pytest.mark.parametrize("mode", ["clamp", "mirror", "repeat", "constant"])
@pytest.mark.parametrize("N", [1, 2, 3, 4, 5, 6])
def test_border_index_matches_np_pad(orc, mode, N):
    pad = 3 * N + 1
    idx = np.arange(N)
    if mode == "constant":
        ref = np.pad(idx, pad, mode="constant", constant_values=-1)
    else:
        ref = np.pad(idx, pad, mode=NP_MODE[mode])
    for i in range(-3 * N, 4 * N):
        assert orc.border_index(mode, i, N) == ref[i + pad], (mode, i, N)


@pytest.mark.parametrize("N", [1, 2, 3, 7])
def test_repeat_is_tiling(orc, N):
    # Repeat == tile the image with itself periodically.
    tiled = np.tile(np.arange(N), 9)          # covers [-4N, 5N)
    for i in range(-4 * N, 5 * N):
        assert orc.border_index("repeat", i, N) == tiled[i + 4 * N]


@pytest.mark.parametrize("N", [1, 2, 5, 8])
def test_mirror_symmetry(orc, N):
    # Symmetric reflection about x = -1/2 and x = N - 1/2 (edge pixel duplicated, A4).
    for i in range(-3 * N, 4 * N):
        b = orc.border_index("mirror", i, N)
        assert 0 <= b < N
        assert orc.border_index("mirror", -1 - i, N) == b
        assert orc.border_index("mirror", 2 * N - 1 - i, N) == b


@pytest.mark.parametrize("N", [1, 3, 6])
def test_clamp_nearest(orc, N):
    for i in range(-2 * N, 3 * N):
        b = orc.border_index("clamp", i, N)
        d = np.abs(np.arange(N) - i)
        assert d[b] == d.min()


def test_in_bounds_identity(orc):
    for mode in range(4):
        for i in range(7):
            assert orc.border_index(mode, i, 7) == i
