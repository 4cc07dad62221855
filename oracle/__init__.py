"""CPU oracle for the 2D inclusive summed-area table -- TEST INFRASTRUCTURE.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` leg may import this package.  The product path
(``paper_conf_cluster_chenwttm18_b200``) never imports it and shares no code
with it (the seeded input generator ``satgen`` is the only common module).

The arithmetic lives in ``sat_oracle.c`` (see its header for the paper
passages each function follows); this module is ctypes marshalling only.

Pairs: 0 = 8u->32s (int32 output, wrap mod 2^32), 1 = 32f->32f (fp64 output of
an fp64 recurrence), 2 = 64f->64f (fp64 output of a double-double recurrence).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

PAIR_8U32S, PAIR_32F32F, PAIR_64F64F = 0, 1, 2
IN_DTYPE = {PAIR_8U32S: np.uint8, PAIR_32F32F: np.float32, PAIR_64F64F: np.float64}
OUT_DTYPE = {PAIR_8U32S: np.int32, PAIR_32F32F: np.float64, PAIR_64F64F: np.float64}

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")
SRC_PATH = os.path.join(_HERE, "sat_oracle.c")

_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain -O2, no fast-math, no contraction)."""
    if force or not os.path.exists(LIB_PATH) or os.path.getmtime(LIB_PATH) < os.path.getmtime(SRC_PATH):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", "-o", LIB_PATH, SRC_PATH])
    return LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB_PATH)
        i64, vp = ctypes.c_int64, ctypes.c_void_p
        L.oracle_sat.argtypes = [ctypes.c_int, vp, i64, i64, i64, vp, i64]
        L.oracle_sat_64f_plain.argtypes = [vp, i64, i64, i64, vp, i64]
        L.oracle_sat_gen_rows.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_uint64, i64,
                                          ctypes.c_double, i64, i64, vp, i64, vp]
        L.oracle_alg1_8u32s.argtypes = [vp, i64, i64, i64, vp, i64]
        L.oracle_alg1_f64.argtypes = [ctypes.c_int, vp, i64, i64, i64, vp, i64]
        for f in (L.oracle_sat, L.oracle_sat_64f_plain, L.oracle_sat_gen_rows, L.oracle_alg1_8u32s,
                  L.oracle_alg1_f64):
            f.restype = ctypes.c_int
        _lib = L
    return _lib


def pair_of(a: np.ndarray) -> int:
    return {np.dtype(np.uint8): PAIR_8U32S, np.dtype(np.float32): PAIR_32F32F,
            np.dtype(np.float64): PAIR_64F64F}[a.dtype]


def _check(rc: int, what: str):
    if rc != 0:
        raise RuntimeError(f"{what} failed with oracle status {rc}")


def sat(A: np.ndarray) -> np.ndarray:
    """Inclusive SAT of a 2-D host image (row stride may be padded)."""
    assert A.ndim == 2 and (A.size == 0 or A.strides[1] == A.itemsize)
    pair = pair_of(A)
    H, W = A.shape
    S = np.empty((H, W), dtype=OUT_DTYPE[pair])
    if A.size == 0:
        return S
    _check(lib().oracle_sat(pair, A.ctypes.data, H, W, A.strides[0], S.ctypes.data, S.strides[0]),
           "oracle_sat")
    return S


def sat_batched(A: np.ndarray) -> np.ndarray:
    return np.stack([sat(a) for a in A]) if A.ndim == 3 else sat(A)


def sat_64f_plain(A: np.ndarray) -> np.ndarray:
    """Plain fp64 recurrence for 64f input (sanity form; reading R4)."""
    assert A.dtype == np.float64 and A.ndim == 2 and A.strides[1] == 8
    H, W = A.shape
    S = np.empty((H, W), dtype=np.float64)
    _check(lib().oracle_sat_64f_plain(A.ctypes.data, H, W, A.strides[0], S.ctypes.data,
                                      S.strides[0]), "oracle_sat_64f_plain")
    return S


def alg1(A: np.ndarray) -> np.ndarray:
    """Algorithm 1 of the paper."""
    assert A.ndim == 2 and A.strides[1] == A.itemsize
    H, W = A.shape
    pair = pair_of(A)
    if pair == PAIR_8U32S:
        J = np.empty((H, W), dtype=np.int32)
        _check(lib().oracle_alg1_8u32s(A.ctypes.data, H, W, A.strides[0], J.ctypes.data,
                                       J.strides[0]), "oracle_alg1_8u32s")
    else:
        J = np.empty((H, W), dtype=np.float64)
        _check(lib().oracle_alg1_f64(pair, A.ctypes.data, H, W, A.strides[0], J.ctypes.data,
                                     J.strides[0]), "oracle_alg1_f64")
    return J


def sat_gen_rows(pair: int, H: int, W: int, rows, seed: int = 0, img: int = 0, mode: int = 0,
                 value: float = 0.0) -> np.ndarray:
    """Selected rows of the SAT of the satgen image (seed, img); O(W) memory."""
    rows = np.ascontiguousarray(np.asarray(rows, dtype=np.int64))
    out = np.empty((len(rows), W), dtype=OUT_DTYPE[pair])
    _check(lib().oracle_sat_gen_rows(pair, mode, seed, img, value, H, W, rows.ctypes.data,
                                     len(rows), out.ctypes.data), "oracle_sat_gen_rows")
    return out


def sat_exclusive(A: np.ndarray, full: bool = True, nval=0) -> np.ndarray:
    """Exclusive SAT, PAPER.md:63-68 (Eq. 2): J(y, x) = 0 where x = 0 or y = 0,
    else sum_{j < y} sum_{i < x} I(j, i); plus NPP's offset nVal on every
    element (nppi_statistics_functions.h, nppiIntegral: pDst(j,i) = nVal +
    sum_{l<j} sum_{k<i} pSrc(l,k)).

    full=True: the (H+1) x (W+1) layout of NPP / OpenCV,
    whose last row/column hold the totals; full=False: Eq. 2 as printed, the
    same H x W size as I (reading R7 of DESIGN.md).  Built from the inclusive
    oracle: J(y+1, x+1) = S(y, x) (Eq. 1 vs Eq. 2).  8u: int64 sum + nVal,
    reported mod 2^32 as int32 (reading R2); floats: fp64 (64f: the
    double-double inclusive result, + nVal rounded once).
    """
    assert A.ndim == 2
    pair = pair_of(A)
    H, W = A.shape
    S = sat(A) if A.size else np.empty((H, W), dtype=OUT_DTYPE[pair])
    if pair == PAIR_8U32S:
        J = np.zeros((H + 1, W + 1), dtype=np.int64)
        J[1:, 1:] = S.astype(np.int64)
        J = (J + int(nval)) & 0xFFFFFFFF
        J = J.astype(np.uint32).view(np.int32)
    else:
        J = np.zeros((H + 1, W + 1), dtype=np.float64)
        J[1:, 1:] = S
        J = J + float(nval)
    return J if full else np.ascontiguousarray(J[:H, :W])


def sat_exclusive_brute(A: np.ndarray, full: bool = True, nval=0) -> np.ndarray:
    """Eq. 2 evaluated literally (tiny inputs only): every element is the
    direct sum over its rectangle {j < y, i < x}, exact (Python ints /
    fractions of the fp values), + nVal."""
    from fractions import Fraction
    H, W = A.shape
    Hn, Wn = (H + 1, W + 1) if full else (H, W)
    pair = pair_of(A)
    vals = [[int(v) if pair == PAIR_8U32S else Fraction(float(v)) for v in row] for row in A]
    out = np.zeros((Hn, Wn), dtype=np.int32 if pair == PAIR_8U32S else np.float64)
    for y in range(Hn):
        for x in range(Wn):
            s = sum((vals[j][i] for j in range(y) for i in range(x)), 0)
            if pair == PAIR_8U32S:
                out[y, x] = np.uint32((s + int(nval)) & 0xFFFFFFFF).view(np.int32)
            else:
                out[y, x] = float(s + Fraction(float(nval)))
    return out


def rect_sums(A: np.ndarray, rects) -> np.ndarray:
    """Direct sums of A over half-open rectangles [y0, y1) x [x0, x1) (clamped),
    straight from the input -- the quantity the four-corner identity of
    PAPER.md:95 recovers from a SAT.  8u: int64 sum reported mod 2^32 (int32)."""
    H, W = A.shape
    pair = pair_of(A)
    out = []
    for y0, x0, y1, x1 in np.asarray(rects, dtype=np.int64).reshape(-1, 4):
        y0, y1 = min(max(y0, 0), H), min(max(y1, 0), H)
        x0, x1 = min(max(x0, 0), W), min(max(x1, 0), W)
        blk = A[y0:y1, x0:x1]
        if pair == PAIR_8U32S:
            v = int(blk.astype(np.int64).sum()) if y1 > y0 and x1 > x0 else 0
            out.append(np.uint32(v & 0xFFFFFFFF).view(np.int32))
        else:
            out.append(float(blk.astype(np.float64).sum()) if y1 > y0 and x1 > x0 else 0.0)
    return np.array(out, dtype=np.int32 if pair == PAIR_8U32S else np.float64)


def box_filter(A: np.ndarray, ry: int, rx: int) -> np.ndarray:
    """Box sums out(y, x) = sum of A over [y-ry, y+ry] x [x-rx, x+rx] clipped to
    the image, as a sum of shifted copies of the zero-padded input (no SAT
    involved).  8u: exact int64, reported mod 2^32; floats: fp64."""
    H, W = A.shape
    pair = pair_of(A)
    P = np.zeros((H + 2 * ry, W + 2 * rx), dtype=np.int64 if pair == PAIR_8U32S else np.float64)
    P[ry:ry + H, rx:rx + W] = A
    out = np.zeros((H, W), dtype=P.dtype)
    for dy in range(2 * ry + 1):
        for dx in range(2 * rx + 1):
            out += P[dy:dy + H, dx:dx + W]
    if pair == PAIR_8U32S:
        return (out & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
    return out


def sat_8u32f(A: np.ndarray) -> np.ndarray:
    """Reference for the 8u->32f pair (NPP's nppiIntegral_8u32f):
    the EXACT inclusive sums of the uint8 image, as fp64 (the double-double
    recurrence of `sat` is exact for integer sums below 2^53); the GPU's fp32
    result is judged against it with the 32f bar (1e-4 relative)."""
    assert A.dtype == np.uint8
    return sat(np.ascontiguousarray(A, dtype=np.float64))


def sat_32s(A: np.ndarray) -> np.ndarray:
    """Reference for the 32s->32s pair: the exact inclusive sums of an int32
    image reported mod 2^32 as int32 (reading R2, as for 8u->32s).  Sums run
    in uint64 (numpy cumsum as the library step, Eq. 1 written as the two
    one-dimensional prefix sums it factors into); uint64 wraps mod 2^64, so
    the low 32 bits are exact for any size."""
    assert A.dtype == np.int32 and A.ndim == 2
    S = A.astype(np.int64).astype(np.uint64).cumsum(axis=0, dtype=np.uint64).cumsum(axis=1, dtype=np.uint64)
    return (S & np.uint64(0xFFFFFFFF)).astype(np.uint32).view(np.int32)


# ---------------------------------------------------------------------------
# Multi-channel consumers.  Both are Eq. 1
# applied channel by channel to a per-pixel vector f(A):

def sat_sq(A: np.ndarray):
    """SAT and SAT of squares of a uint8 image (Viola-Jones variance
    normalisation, PAPER.md:18-24 [2]): S = sum_{y<=i, x<=j} A(y, x) and
    Q = sum_{y<=i, x<=j} A(y, x)^2, both exact and reported mod 2^32 as int32
    (reading R2).  Returns an [..., H, W, 2] int32 array (S, Q interleaved).
    Q reuses sat_32s on the squared image (squares <= 65025 fit int32)."""
    assert A.dtype == np.uint8
    if A.ndim == 3:
        return np.stack([sat_sq(a) for a in A])
    S = sat(np.ascontiguousarray(A))
    Q = sat_32s(np.ascontiguousarray(A.astype(np.int32) ** 2))
    return np.stack([S, Q], axis=-1)


def integral_histogram(A: np.ndarray, bin_of: np.ndarray, nbins: int) -> np.ndarray:
    """Integral histogram ([34], [38]): H_k(i, j) = number of
    pixels (y <= i, x <= j) whose value falls in bin k, bin = bin_of[value],
    for k < nbins; counts exact mod 2^32 as int32.  Returns [nbins, H, W]
    (bin-major; the library's interleaved 4-bin groups are compared after a
    transpose).  Each bin is the SAT (`sat`, the int64 recurrence) of its
    0/1 indicator image."""
    assert A.dtype == np.uint8 and A.ndim == 2
    b = np.asarray(bin_of, dtype=np.int64)[A]
    return np.stack([sat(np.ascontiguousarray((b == k).astype(np.uint8))) for k in range(nbins)])
