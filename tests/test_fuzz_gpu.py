"""Seeded randomised parity: many random (pair, shape, batch, pitch, offset)
cases through `sat_compute` / `sat_compute_batched` / `sat_compute_exclusive`
against the CPU oracle, with sentinel-filled output padding that must stay
untouched.

The shapes are drawn around the kernel's tile edges (TW = 128 / 256 columns,
TH = 16 / 32 rows, so +-1 of a multiple) and elsewhere uniformly; a quarter of
the cases start the input at an element offset that breaks 16-byte alignment
(the generic, non-TMA path).  Bars are BASELINE.json's: bit-exact for the
integer pairs (8u->32s, 32s->32s; wrap mod 2^32, reading R2), max relative
error 1e-4 for 32f and 8u->32f (against the exact sums), 1e-12 for 64f.
"""
import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu

N_CASES = 120
# pair -> (input numpy dtype, output numpy dtype, tolerance); pair numbers as in libsat.h
PAIRS = {
    0: (np.uint8, np.int32, 0.0),
    1: (np.float32, np.float32, 1e-4),
    2: (np.float64, np.float64, 1e-12),
    3: (np.uint8, np.float32, 1e-4),
    4: (np.int32, np.int32, 0.0),
}
SENTINEL = {np.int32: -123456789, np.float32: -7.25, np.float64: -7.25}


def _t():
    import torch
    return torch


def _sat():
    import paper_conf_cluster_chenwttm18_b200 as sat
    return sat


def _tdt(d):
    torch = _t()
    return {np.uint8: torch.uint8, np.float32: torch.float32, np.float64: torch.float64,
            np.int32: torch.int32}[d]


def _dim(rng, edges):
    if rng.random() < 0.5:
        return int(max(1, rng.choice(edges) * rng.integers(1, 4) + rng.integers(-1, 2)))
    return int(rng.integers(1, 1400))


def _host_input(pair, N, H, W, seed, rng):
    tin = PAIRS[pair][0]
    if tin is np.int32:
        return rng.integers(-2**31, 2**31 - 1, size=(N, H, W), dtype=np.int64).astype(np.int32)
    kind = satgen.KIND_OF_DTYPE[np.dtype(tin)]
    return np.stack([satgen.generate(kind, H, W, seed=seed, img=n) for n in range(N)])


def _reference(pair, A):
    if pair == 3:
        return oracle.sat_8u32f(A)
    if pair == 4:
        return oracle.sat_32s(A)
    return oracle.sat(A)


def _check(got, ref, tol, what):
    if tol == 0.0:
        assert np.array_equal(got, ref), f"{what}: {int((got != ref).sum())} mismatches"
        return
    g = got.astype(np.float64)
    nz = ref != 0
    assert np.all(g[~nz] == 0), f"{what}: nonzero where the oracle is 0"
    if nz.any():
        worst = float(np.max(np.abs(g[nz] - ref[nz]) / np.abs(ref[nz])))
        assert worst <= tol, f"{what}: max rel err {worst:.3e} > {tol:.0e}"


def _case(i):
    rng = np.random.default_rng(90_000 + i)
    pair = int(rng.choice(list(PAIRS)))
    H = _dim(rng, [16, 32, 64])
    W = _dim(rng, [128, 256])
    N = int(rng.choice([1, 1, 2, 3]))
    in_pad = int(rng.choice([0, 0, 3, 16, 40]))
    out_pad = int(rng.choice([0, 0, 4, 8, 17]))
    offset = int(rng.choice([0, 0, 0, 1]))  # element offset: 1 breaks 16-byte alignment
    return rng, pair, N, H, W, in_pad, out_pad, offset


@pytest.mark.parametrize("i", range(N_CASES))
def test_fuzz_inclusive(i):
    torch, sat = _t(), _sat()
    rng, pair, N, H, W, in_pad, out_pad, offset = _case(i)
    tin, tout, tol = PAIRS[pair]
    A = _host_input(pair, N, H, W, 90_000 + i, rng)
    # input: [N, H, W + in_pad] buffer, the image starting `offset` elements in
    flat = torch.zeros(N * H * (W + in_pad) + offset, dtype=_tdt(tin), device="cuda")
    x = flat[offset:].view(N, H, W + in_pad)[:, :, :W]
    x.copy_(torch.from_numpy(A))
    ybuf = torch.full((N, H, W + out_pad), SENTINEL[tout], dtype=_tdt(tout), device="cuda")
    y = ybuf[:, :, :W]
    sat.sat(x if N > 1 else x[0], out=y if N > 1 else y[0])
    torch.cuda.synchronize()
    what = f"case {i}: pair {pair} N={N} {H}x{W} in_pad={in_pad} out_pad={out_pad} off={offset}"
    got = y.cpu().numpy()
    for n in range(N):
        _check(got[n], _reference(pair, A[n]), tol, f"{what} img {n}")
    if out_pad:
        pad = ybuf[:, :, W:].cpu().numpy()
        assert np.all(pad == np.asarray(SENTINEL[tout], dtype=tout)), f"{what}: padding written"


@pytest.mark.parametrize("i", range(0, N_CASES, 3))
def test_fuzz_exclusive(i):
    torch, sat = _t(), _sat()
    rng, pair, _, H, W, _, _, _ = _case(i)
    tin, tout, tol = PAIRS[pair]
    A = _host_input(pair, 1, H, W, 91_000 + i, rng)[0]
    full = bool(rng.integers(0, 2))
    x = torch.from_numpy(A).cuda()
    e = sat.sat_exclusive(x, full=full, out_dtype=_tdt(tout))
    torch.cuda.synchronize()
    inc = _reference(pair, A)
    # Eq. 2: the exclusive SAT is the inclusive one shifted by a row and a column
    ref = np.zeros((H + 1, W + 1), dtype=inc.dtype)
    ref[1:, 1:] = inc
    if not full:
        ref = ref[:H, :W]
    _check(e.cpu().numpy(), ref, tol, f"exclusive case {i}: pair {pair} {H}x{W} full={full}")
