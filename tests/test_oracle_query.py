"""Pins for the SAT-consumer oracles (rectangle sums, box filter; SURVEY.md
Sec. 8(f) N4): brute-force loops, closed forms, and agreement with the
four-corner identity on the oracle SAT."""
import numpy as np
import pytest

import oracle

RNG = np.random.default_rng(11)


def test_rect_sums_bruteforce_and_clamping():
    A = RNG.integers(0, 256, (9, 13)).astype(np.uint8)
    rects = [(0, 0, 9, 13), (2, 3, 5, 7), (4, 4, 4, 9), (-3, -2, 2, 3), (7, 11, 20, 30), (5, 5, 3, 2)]
    got = oracle.rect_sums(A, rects)
    for (y0, x0, y1, x1), g in zip(rects, got):
        s = 0
        for y in range(max(y0, 0), min(y1, 9)):
            for x in range(max(x0, 0), min(x1, 13)):
                s += int(A[y, x])
        assert int(g) == s


def test_rect_sums_agree_with_four_corners_on_sat():
    A = RNG.random((40, 50))
    S = oracle.sat(A)
    Z = np.zeros((41, 51))
    Z[1:, 1:] = S
    rects = RNG.integers(0, 51, (200, 4))
    rects[:, 0] %= 41
    rects[:, 2] %= 41
    got = oracle.rect_sums(A, rects)
    for (y0, x0, y1, x1), g in zip(rects, got):
        if y1 <= y0 or x1 <= x0:
            assert g == 0.0
        else:
            four = Z[y1, x1] - Z[y0, x1] - Z[y1, x0] + Z[y0, x0]
            assert abs(g - four) <= 1e-12 * max(1.0, abs(Z).max())


@pytest.mark.parametrize("H,W,ry,rx", [(1, 1, 0, 0), (6, 9, 1, 2), (17, 5, 3, 0), (8, 8, 10, 10)])
def test_box_filter_all_ones_closed_form(H, W, ry, rx):
    A = np.ones((H, W), dtype=np.uint8)
    got = oracle.box_filter(A, ry, rx)
    y, x = np.mgrid[0:H, 0:W]
    cnt_y = np.minimum(y + ry, H - 1) - np.maximum(y - ry, 0) + 1
    cnt_x = np.minimum(x + rx, W - 1) - np.maximum(x - rx, 0) + 1
    assert np.array_equal(got, (cnt_y * cnt_x).astype(np.int32))


def test_box_filter_bruteforce_and_identity():
    A = RNG.integers(0, 256, (7, 10)).astype(np.uint8)
    assert np.array_equal(oracle.box_filter(A, 0, 0), A.astype(np.int32))
    got = oracle.box_filter(A, 2, 1)
    for y in range(7):
        for x in range(10):
            s = int(A[max(y - 2, 0):y + 3, max(x - 1, 0):x + 2].astype(np.int64).sum())
            assert got[y, x] == s
