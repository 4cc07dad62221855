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


# ---------------------------------------------------------------------------
# Multi-channel consumers: SAT + SAT of squares, integral histogram.

def test_sat_sq_bruteforce():
    """Direct rectangle sums of A and A^2 from the origin (Eq. 1 by its
    definition), exact integers."""
    A = RNG.integers(0, 256, (7, 11)).astype(np.uint8)
    SQ = oracle.sat_sq(A)
    for i in range(7):
        for j in range(11):
            blk = A[:i + 1, :j + 1].astype(np.int64)
            assert SQ[i, j, 0] == blk.sum()
            assert SQ[i, j, 1] == (blk * blk).sum()


def test_sat_sq_closed_form_and_wrap():
    """Constant c: S = c (i+1)(j+1), Q = c^2 (i+1)(j+1) mod 2^32 -- c = 255 on
    300 x 300 pushes Q past 2^32 (5.85e9)."""
    c = 255
    A = np.full((300, 300), c, dtype=np.uint8)
    SQ = oracle.sat_sq(A)
    ii, jj = np.meshgrid(np.arange(1, 301, dtype=np.int64), np.arange(1, 301, dtype=np.int64),
                         indexing="ij")
    wrap = lambda v: (v & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
    assert np.array_equal(SQ[..., 0], wrap(c * ii * jj))
    assert np.array_equal(SQ[..., 1], wrap(c * c * ii * jj))
    assert int(SQ[..., 1].view(np.uint32).max()) < c * c * 300 * 300  # it did wrap


def test_sat_sq_variance_identity():
    """A window's variance from the four corners of S and Q equals
    numpy's variance of the window (the Viola-Jones use)."""
    A = RNG.integers(0, 256, (40, 50)).astype(np.uint8)
    SQ = oracle.sat_sq(A).astype(np.int64)
    Z = np.zeros((41, 51, 2), dtype=np.int64)
    Z[1:, 1:] = SQ
    for (y0, x0, y1, x1) in [(0, 0, 40, 50), (3, 4, 27, 30), (10, 10, 12, 11)]:
        s, q = (Z[y1, x1] - Z[y0, x1] - Z[y1, x0] + Z[y0, x0])
        n = (y1 - y0) * (x1 - x0)
        var = q / n - (s / n) ** 2
        assert abs(var - A[y0:y1, x0:x1].astype(np.float64).var()) < 1e-6


def test_integral_histogram_bruteforce_and_partition():
    """Counts by direct counting over the prefix rectangle; the bins of a
    table that covers every value sum to (i+1)(j+1); a value mapped outside
    [0, nbins) is in no bin."""
    A = RNG.integers(0, 256, (6, 9)).astype(np.uint8)
    bin_of = RNG.integers(0, 5, 256)
    bin_of[7] = 200  # never counted
    A[2, 3] = 7
    Hh = oracle.integral_histogram(A, bin_of, 5)
    for k in range(5):
        for i in range(6):
            for j in range(9):
                assert Hh[k, i, j] == int(np.sum(bin_of[A[:i + 1, :j + 1]] == k))
    full = oracle.integral_histogram(A, np.arange(256) * 16 // 256, 16)
    ii, jj = np.meshgrid(np.arange(1, 7), np.arange(1, 10), indexing="ij")
    assert np.array_equal(full.sum(axis=0), ii * jj)
