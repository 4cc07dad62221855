"""Pins for the exclusive-SAT oracle (Eq. 2; NPP's nVal form,
PAPER.md:418-428): brute force on tiny inputs, closed forms, the border-free
four-corner rectangle identity, the Eq. 2 crop, and wrap mod 2^32."""
import numpy as np
import pytest

import oracle

RNG = np.random.default_rng(7)


def _img(dtype, shape):
    if dtype == np.uint8:
        return RNG.integers(0, 256, shape).astype(np.uint8)
    if dtype == np.float32:
        return (RNG.integers(0, 1 << 24, shape) * 2.0 ** -24).astype(np.float32)
    return RNG.random(shape)


@pytest.mark.parametrize("dtype", [np.uint8, np.float32, np.float64])
@pytest.mark.parametrize("shape", [(1, 1), (1, 6), (5, 1), (4, 7), (9, 5)])
@pytest.mark.parametrize("full", [True, False])
def test_exclusive_bruteforce(dtype, shape, full):
    A = _img(dtype, shape)
    nval = 0 if dtype == np.uint8 and shape == (1, 1) else (5 if dtype == np.uint8 else 0.25)
    got = oracle.sat_exclusive(A, full=full, nval=nval)
    ref = oracle.sat_exclusive_brute(A, full=full, nval=nval)
    H, W = shape
    assert got.shape == ((H + 1, W + 1) if full else (H, W))
    if dtype == np.uint8:
        assert np.array_equal(got, ref)
    else:
        np.testing.assert_allclose(got, ref, rtol=1e-15, atol=0)


@pytest.mark.parametrize("H,W", [(1, 1), (3, 300), (257, 5), (64, 64)])
def test_exclusive_all_ones_closed_form(H, W):
    """All-ones input: J(y, x) = x * y + nVal (Eq. 2), borders = nVal."""
    A = np.ones((H, W), dtype=np.uint8)
    J = oracle.sat_exclusive(A, full=True, nval=-3)
    y, x = np.mgrid[0:H + 1, 0:W + 1]
    assert np.array_equal(J, (x * y - 3).astype(np.int32))
    assert np.all(J[0, :] == -3) and np.all(J[:, 0] == -3)


def test_exclusive_rectangle_identity_without_border_cases():
    """The point of the (H+1) x (W+1) layout: ANY rectangle [y0, y1) x [x0, x1),
    including ones touching row 0 / column 0, is J(y1,x1) - J(y0,x1) - J(y1,x0)
    + J(y0,x0) with no special cases (PAPER.md:95 for the inclusive form)."""
    A = _img(np.uint8, (23, 31))
    J = oracle.sat_exclusive(A, full=True, nval=11).astype(np.int64)
    for _ in range(300):
        y0, y1 = sorted(RNG.integers(0, 24, 2))
        x0, x1 = sorted(RNG.integers(0, 32, 2))
        direct = int(A[y0:y1, x0:x1].astype(np.int64).sum())
        assert J[y1, x1] - J[y0, x1] - J[y1, x0] + J[y0, x0] == direct


@pytest.mark.parametrize("dtype", [np.uint8, np.float64])
def test_exclusive_eq2_is_crop_of_full(dtype):
    A = _img(dtype, (17, 19))
    full = oracle.sat_exclusive(A, full=True, nval=2)
    eq2 = oracle.sat_exclusive(A, full=False, nval=2)
    assert np.array_equal(eq2, full[:17, :19])


def test_exclusive_shift_of_inclusive_and_wrap():
    """J(y+1, x+1) = S(y, x) + nVal mod 2^32 (8u; reading R2), also past 2^31."""
    A = np.full((3000, 3000), 255, dtype=np.uint8)
    J = oracle.sat_exclusive(A, full=True, nval=1000)
    S = oracle.sat(A)
    assert np.array_equal(J[1:, 1:], (S.view(np.uint32) + np.uint32(1000)).view(np.int32))
    exact = 255 * 3000 * 3000 + 1000
    assert int(J[-1, -1].view(np.uint32)) == exact % (1 << 32)


def test_exclusive_empty_shapes():
    A = np.zeros((0, 5), dtype=np.uint8)
    J = oracle.sat_exclusive(A, full=True, nval=4)
    assert J.shape == (1, 6) and np.all(J == 4)
    assert oracle.sat_exclusive(A, full=False).shape == (0, 5)


def test_8u32f_reference_is_exact_sum():
    """oracle.sat_8u32f equals the brute-force integer rectangle sums (tiny)
    and the exact int64 cumsums past 2^32 (where 8u->32s wraps)."""
    A = RNG.integers(0, 256, (6, 9)).astype(np.uint8)
    ref = np.array([[int(A[:i + 1, :j + 1].astype(np.int64).sum()) for j in range(9)] for i in range(6)],
                   dtype=np.float64)
    assert np.array_equal(oracle.sat_8u32f(A), ref)
    B = np.full((300, 70000), 255, dtype=np.uint8)  # total 5.4e9 > 2^32
    got = oracle.sat_8u32f(B)
    assert got[-1, -1] == 255.0 * 300 * 70000


def test_32s_reference_bruteforce_and_8u_agreement():
    """oracle.sat_32s: brute force (Python ints, negative values, reported mod
    2^32) and equality with the independent 8u->32s recurrence oracle on
    inputs in [0, 255] (including past 2^31 where both wrap)."""
    A = RNG.integers(-2**31, 2**31, (5, 7), dtype=np.int64).astype(np.int32)
    got = oracle.sat_32s(A)
    for i in range(5):
        for j in range(7):
            s = int(A[:i + 1, :j + 1].astype(object).sum()) % (1 << 32)
            assert int(got[i, j].view(np.uint32)) == s
    B = np.full((3000, 3000), 255, dtype=np.uint8)
    assert np.array_equal(oracle.sat_32s(B.astype(np.int32)), oracle.sat(B))
