"""Pins of the CPU oracle against things other than itself (run with -m "not gpu").

Each test names the passage or mathematical fact it checks.  The oracle's
arithmetic is in oracle/sat_oracle.c; nothing here re-types its recurrence.
"""
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import satgen

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
RNG = np.random.default_rng(20181210)


def _load_golden(name):
    A, S, cur = [], [], None
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            if line in ("[A]", "[S]"):
                cur = A if line == "[A]" else S
                continue
            cur.append([int(v) for v in line.split()])
    return np.array(A), np.array(S)


# --- hand-worked golden fixture (Eq. 1) ----------
@pytest.mark.parametrize("dtype", [np.uint8, np.float32, np.float64])
def test_golden_handworked(dtype):
    A, S = _load_golden("sat_4x5_handworked.txt")
    got = oracle.sat(A.astype(dtype))
    np.testing.assert_array_equal(got, S.astype(got.dtype))
    np.testing.assert_array_equal(oracle.alg1(A.astype(dtype)), S.astype(got.dtype))


# --- brute force on tiny inputs (definition) ------------------
def _brute_int(A):
    H, W = A.shape
    out = np.empty((H, W), dtype=np.int64)
    for i in range(H):
        for j in range(W):
            out[i, j] = sum(int(v) for v in A[: i + 1, : j + 1].ravel())
    return out


def _brute_exact(A):
    """Exact rational rectangle sums (Fractions) for float inputs."""
    H, W = A.shape
    F = [[Fraction(float(v)) for v in row] for row in A]
    out = [[None] * W for _ in range(H)]
    for i in range(H):
        for j in range(W):
            out[i][j] = sum((F[y][x] for y in range(i + 1) for x in range(j + 1)), Fraction(0))
    return out


@pytest.mark.parametrize("shape", [(1, 1), (1, 17), (13, 1), (5, 7), (31, 33), (33, 31), (2, 33)])
def test_bruteforce_8u32s(shape):
    A = RNG.integers(0, 256, size=shape, dtype=np.uint8)
    ref = _brute_int(A)
    np.testing.assert_array_equal(oracle.sat(A).astype(np.int64), ref)  # no wrap at this size


@pytest.mark.parametrize("shape", [(1, 1), (1, 9), (7, 1), (6, 5), (12, 17)])
def test_bruteforce_32f(shape):
    A = satgen.generate(satgen.KIND_F32, *shape, seed=7)
    ref = _brute_exact(A)
    got = oracle.sat(A)
    for i in range(shape[0]):
        for j in range(shape[1]):
            # the fp64 recurrence on 24-bit inputs at this size is exact
            assert Fraction(float(got[i, j])) == ref[i][j]


@pytest.mark.parametrize("shape", [(1, 1), (3, 8), (9, 2), (10, 11)])
def test_bruteforce_64f_full_mantissa(shape):
    A = satgen.generate(satgen.KIND_F64, *shape, seed=11)
    ref = _brute_exact(A)
    got = oracle.sat(A)  # double-double recurrence, one rounding
    for i in range(shape[0]):
        for j in range(shape[1]):
            exact = ref[i][j]
            rounded = float(exact)  # correctly rounded exact value
            assert got[i, j] == rounded or abs(Fraction(float(got[i, j])) - exact) <= abs(exact) * Fraction(1, 2**52)


# --- closed forms ---------------------------------------------------------------
@pytest.mark.parametrize("H,W", [(1, 1), (7, 300), (300, 7), (257, 255), (1080, 1920)])
def test_all_ones_closed_form(H, W):
    """BASELINE.json north_star: all-ones input gives S(i,j) = (i+1)(j+1)."""
    i = np.arange(H, dtype=np.int64)[:, None]
    j = np.arange(W, dtype=np.int64)[None, :]
    ref = (i + 1) * (j + 1)
    for dt in (np.uint8, np.float32, np.float64):
        got = oracle.sat(np.ones((H, W), dtype=dt))
        np.testing.assert_array_equal(got.astype(np.int64), ref)


def test_constant_and_separable_closed_forms():
    H, W = 123, 77
    i = np.arange(H, dtype=np.int64)[:, None]
    j = np.arange(W, dtype=np.int64)[None, :]
    got = oracle.sat(np.full((H, W), 9, dtype=np.uint8)).astype(np.int64)
    np.testing.assert_array_equal(got, 9 * (i + 1) * (j + 1))
    # separable A(y,x) = f(y) g(x)  =>  S(i,j) = F(i) G(j) with F, G the prefix sums
    f = RNG.integers(0, 16, size=H)
    g = RNG.integers(0, 16, size=W)
    A = (f[:, None] * g[None, :]).astype(np.uint8)
    F = np.array([sum(int(v) for v in f[: k + 1]) for k in range(H)], dtype=np.int64)
    G = np.array([sum(int(v) for v in g[: k + 1]) for k in range(W)], dtype=np.int64)
    np.testing.assert_array_equal(oracle.sat(A).astype(np.int64), F[:, None] * G[None, :])


def test_all_255_wraps_mod_2_32():
    """Reading R2: 8u->32s output is the exact sum mod 2^32 (two's complement).

    255 (i+1)(j+1) first exceeds 2^31 near 2902^2; 3000^2 covers the wrap."""
    H = W = 3000
    got = oracle.sat(np.full((H, W), 255, dtype=np.uint8))
    i = np.arange(H, dtype=np.int64)[:, None]
    j = np.arange(W, dtype=np.int64)[None, :]
    ref = ((255 * (i + 1) * (j + 1)) & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
    assert (255 * H * W) > 2**31
    np.testing.assert_array_equal(got, ref)
    assert got[-1, -1] < 0  # wrapped into the negative range


# --- invariants ------------------------------------------------------------------
def test_rectangle_identity():
    """PAPER.md:95 (Fig. 1): rect sum = a + d - b - c with four SAT lookups."""
    H, W = 211, 173
    A = RNG.integers(0, 256, size=(H, W), dtype=np.uint8)
    S = oracle.sat(A).astype(np.int64)
    Sp = np.zeros((H + 1, W + 1), dtype=np.int64)
    Sp[1:, 1:] = S
    for _ in range(400):
        y0, y1 = sorted(RNG.integers(0, H, size=2))
        x0, x1 = sorted(RNG.integers(0, W, size=2))
        direct = int(A[y0 : y1 + 1, x0 : x1 + 1].astype(np.int64).sum())
        a, b, c, d = Sp[y0, x0], Sp[y0, x1 + 1], Sp[y1 + 1, x0], Sp[y1 + 1, x1 + 1]
        assert a + d - b - c == direct


def test_rectangle_identity_dyadic_64f_exact():
    H, W = 150, 190
    A = satgen.generate(satgen.KIND_F64, H, W, seed=3, mode=satgen.MODE_DYADIC24)
    S = oracle.sat(A)
    Sp = np.zeros((H + 1, W + 1))
    Sp[1:, 1:] = S
    for _ in range(200):
        y0, y1 = sorted(RNG.integers(0, H, size=2))
        x0, x1 = sorted(RNG.integers(0, W, size=2))
        direct = math.fsum(A[y0 : y1 + 1, x0 : x1 + 1].ravel())
        assert (Sp[y1 + 1, x1 + 1] - Sp[y0, x1 + 1]) - (Sp[y1 + 1, x0] - Sp[y0, x0]) == direct


@pytest.mark.parametrize("dtype", [np.uint8, np.float64])
def test_alg1_equals_recurrence(dtype):
    """PAPER.md:72-93 (Alg. 1) computes the same table (exact for ints/dyadics)."""
    H, W = 301, 517
    if dtype == np.uint8:
        A = RNG.integers(0, 256, size=(H, W), dtype=np.uint8)
    else:
        A = satgen.generate(satgen.KIND_F64, H, W, seed=5, mode=satgen.MODE_DYADIC24)
    np.testing.assert_array_equal(oracle.alg1(A), oracle.sat(A))


def test_alg1_close_32f():
    A = satgen.generate(satgen.KIND_F32, 400, 333, seed=8)
    np.testing.assert_allclose(oracle.alg1(A), oracle.sat(A), rtol=1e-13)


def test_inverse_difference_recovers_input_even_when_wrapped():
    H, W = 3100, 3100  # wraps mod 2^32 (255-heavy input)
    A = np.full((H, W), 255, dtype=np.uint8)
    A[::7, ::3] = RNG.integers(0, 256, size=A[::7, ::3].shape, dtype=np.uint8)
    S = oracle.sat(A).view(np.uint32).astype(np.int64)
    Sp = np.zeros((H + 1, W + 1), dtype=np.int64)
    Sp[1:, 1:] = S
    D = (Sp[1:, 1:] - Sp[:-1, 1:] - Sp[1:, :-1] + Sp[:-1, :-1]) & 0xFFFFFFFF
    np.testing.assert_array_equal(D, A.astype(np.int64))


def test_transpose_symmetry():
    A = RNG.integers(0, 256, size=(97, 45), dtype=np.uint8)
    np.testing.assert_array_equal(oracle.sat(np.ascontiguousarray(A.T)), oracle.sat(A).T)


def test_numpy_cumsum_crosscheck():
    """Special case that reduces to a library routine: cumsum over both axes."""
    A = RNG.integers(0, 256, size=(640, 480), dtype=np.uint8)
    ref = np.cumsum(np.cumsum(A.astype(np.int64), axis=0), axis=1)
    np.testing.assert_array_equal(oracle.sat(A).astype(np.int64), ref)
    B = satgen.generate(satgen.KIND_F32, 300, 200, seed=1)
    refb = np.cumsum(np.cumsum(B.astype(np.float64), axis=0), axis=1)
    np.testing.assert_allclose(oracle.sat(B), refb, rtol=1e-13)


def test_linearity_mod_2_32():
    A = RNG.integers(0, 128, size=(3000, 3000), dtype=np.uint8)
    B = RNG.integers(0, 128, size=(3000, 3000), dtype=np.uint8)
    lhs = oracle.sat((A + B).astype(np.uint8)).view(np.uint32)
    rhs = oracle.sat(A).view(np.uint32) + oracle.sat(B).view(np.uint32)  # uint32 wraps
    np.testing.assert_array_equal(lhs, rhs)


def test_dyadic_64f_is_exact():
    """Reading R6: 24-bit dyadic inputs keep every partial sum exact while
    H*W <= 2^29, so the SAT equals the integer SAT scaled by 2^-24."""
    H, W = 1024, 1536
    A = satgen.generate(satgen.KIND_F64, H, W, seed=9, mode=satgen.MODE_DYADIC24)
    K = np.rint(A * 16777216.0).astype(np.int64)
    exact = np.cumsum(np.cumsum(K, axis=0), axis=1)
    np.testing.assert_array_equal(oracle.sat(A), exact.astype(np.float64) / 16777216.0)
    np.testing.assert_array_equal(oracle.sat_64f_plain(A), oracle.sat(A))


def test_double_double_beats_plain_fp64():
    """Reading R4: plain fp64 recurrence error grows ~u*sqrt(ij); the dd
    oracle stays at ~1 ulp of the exact sum (checked via exact integers)."""
    H, W = 1024, 1024
    # inputs k * 2^-53 with k < 2^53: exact sums fit in Python ints
    A = satgen.generate(satgen.KIND_F64, H, W, seed=21)
    K = (A * 9007199254740992.0).astype(np.uint64).astype(object)
    rows = [0, 511, 1023]
    # exact column sums up to row i, then prefix over x, for the sampled rows
    colsum = np.zeros(W, dtype=object)
    exact_rows = {}
    for i in range(H):
        colsum = colsum + K[i]
        if i in rows:
            exact_rows[i] = np.cumsum(colsum)
    dd = oracle.sat(A)
    plain = oracle.sat_64f_plain(A)
    for i in rows:
        ex = np.array([float(Fraction(int(v), 2**53)) for v in exact_rows[i]])
        rel_dd = np.max(np.abs(dd[i] - ex) / ex)
        rel_plain = np.max(np.abs(plain[i] - ex) / ex)
        assert rel_dd <= 2.3e-16
        assert rel_plain <= 2e-12


@pytest.mark.parametrize("pair", [0, 1, 2])
def test_gen_rows_matches_full(pair):
    """The streaming, generator-fed form agrees with the array form."""
    H, W = 333, 257
    kind = {0: satgen.KIND_U8, 1: satgen.KIND_F32, 2: satgen.KIND_F64}[pair]
    A = satgen.generate(kind, H, W, seed=42, img=3)
    full = oracle.sat(A)
    rows = [0, 1, 100, 331, 332]
    got = oracle.sat_gen_rows(pair, H, W, rows, seed=42, img=3)
    np.testing.assert_array_equal(got, full[rows])


def test_empty_is_noop():
    assert oracle.sat(np.zeros((0, 5), dtype=np.uint8)).shape == (0, 5)
    assert oracle.sat(np.zeros((5, 0), dtype=np.float32)).shape == (5, 0)
