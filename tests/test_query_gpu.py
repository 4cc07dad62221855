"""GPU parity of the SAT consumers (sat_rect_sums, sat_box_filter; SURVEY.md
Sec. 8(f) N4) against oracles that sum the INPUT directly (no SAT).

Tolerances: 8u->32s is bit-exact (the four-corner identity holds mod 2^32, so
any rectangle whose true sum is < 2^32 is exact even where the SAT wrapped).
For floats a rectangle sum is a difference of four SAT values, each within
the SAT bar (rel. 1e-4 for 32f, 1e-12 for 64f), so the derived bound is
absolute: |got - ref| <= 4 * bar * max|S| (cancellation: a small rectangle far
from the origin keeps only the SAT's absolute accuracy)."""
import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu
BAR = {np.uint8: 0.0, np.float32: 1e-4, np.float64: 1e-12}


def _t():
    import torch
    return torch


def _sat():
    import paper_conf_cluster_chenwttm18_b200 as sat
    return sat


def _tdt(d):
    torch = _t()
    return {np.uint8: torch.uint8, np.float32: torch.float32, np.float64: torch.float64}[d]


def _check(got, ref, d, smax, what):
    if BAR[d] == 0.0:
        assert np.array_equal(got, ref), f"{what}: {np.count_nonzero(got != ref)} mismatches"
    else:
        err = np.max(np.abs(got.astype(np.float64) - ref)) if got.size else 0.0
        assert err <= 4 * BAR[d] * smax, f"{what}: abs err {err} > {4 * BAR[d] * smax}"


@pytest.mark.parametrize("d", [np.uint8, np.float32, np.float64])
def test_rect_sums_parity(d):
    torch, sat = _t(), _sat()
    H, W = 513, 1031
    x = torch.empty((H, W), dtype=_tdt(d), device="cuda")
    satgen.fill_device(x, seed=41)
    S = sat.sat(x)
    rng = np.random.default_rng(3)
    r = np.stack([rng.integers(-5, H + 5, 4000), rng.integers(-5, W + 5, 4000),
                  rng.integers(-5, H + 5, 4000), rng.integers(-5, W + 5, 4000)], 1).astype(np.int32)
    r[:100, 2] = r[:100, 0]  # empty rows
    got = sat.rect_sums(S, torch.from_numpy(r).cuda())
    torch.cuda.synchronize()
    ref = oracle.rect_sums(x.cpu().numpy(), r)
    _check(got.cpu().numpy(), ref, d, float(S.abs().max()), f"rect_sums {d.__name__}")


def test_rect_sums_exact_where_the_sat_wraps():
    """16384^2 8u: the SAT wraps past 2^32; rectangles with true sums < 2^32
    (up to ~16.8M pixels here) are still bit-exact."""
    torch, sat = _t(), _sat()
    H = W = 16384
    x = torch.empty((H, W), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=1001)
    S = sat.sat(x)
    rng = np.random.default_rng(5)
    y0 = rng.integers(0, H - 4096, 300)
    x0 = rng.integers(0, W - 4096, 300)
    hh = rng.integers(1, 4096, 300)
    ww = rng.integers(1, 4096, 300)
    r = np.stack([y0, x0, y0 + hh, x0 + ww], 1).astype(np.int32)
    got = sat.rect_sums(S, torch.from_numpy(r).cuda()).cpu().numpy()
    A = x.cpu().numpy()
    ref = oracle.rect_sums(A, r)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("d", [np.uint8, np.float32, np.float64])
@pytest.mark.parametrize("ry,rx", [(0, 0), (1, 2), (5, 3), (40, 70)])
def test_box_filter_parity(d, ry, rx):
    torch, sat = _t(), _sat()
    H, W = 300, 517
    x = torch.empty((H, W), dtype=_tdt(d), device="cuda")
    satgen.fill_device(x, seed=42)
    S = sat.sat(x)
    got = sat.box_filter(S, ry, rx)
    torch.cuda.synchronize()
    ref = oracle.box_filter(x.cpu().numpy(), ry, rx)
    _check(got.cpu().numpy(), ref, d, float(S.abs().max()), f"box {d.__name__} r=({ry},{rx})")


def test_box_filter_full_size_sampled_rows():
    """16384^2 8u, radius 8: sampled interior and border rows against the
    oracle run on the rows' input neighbourhood."""
    torch, sat = _t(), _sat()
    H = W = 16384
    ry = rx = 8
    x = torch.empty((H, W), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=1001)
    S = sat.sat(x)
    B = sat.box_filter(S, ry, rx)
    torch.cuda.synchronize()
    for y in (0, 3, 4000, 12345, H - 1):
        lo, hi = max(y - ry, 0), min(y + ry + 1, H)
        blk = x[lo:hi].cpu().numpy()
        ref = oracle.box_filter(blk, ry, rx)[y - lo]
        assert np.array_equal(B[y].cpu().numpy(), ref), f"row {y}"


def test_invalid_arguments_of_consumers_and_exclusive():
    """sat_compute_exclusive / sat_rect_sums / sat_box_filter validate
    synchronously and launch nothing on failure (libsat.h conventions)."""
    import ctypes
    torch, sat = _t(), _sat()
    L = sat.lib()
    x = torch.zeros((64, 64), dtype=torch.uint8, device="cuda")
    S = torch.zeros((64, 64), dtype=torch.int32, device="cuda")
    out = torch.full((65, 68), 5, dtype=torch.int32, device="cuda")
    p = sat.Plan(0, 64, 64, 1)
    h = p.handle
    nv = ctypes.c_int32(1)
    rects = torch.zeros((4, 4), dtype=torch.int32, device="cuda")
    qo = torch.full((4,), 5, dtype=torch.int32, device="cuda")
    cases = [
        (L.sat_compute_exclusive(h, x.data_ptr(), out.data_ptr(), 64, 64, 64, 64 * 4, 1, ctypes.byref(nv), 0, None), 1),  # pitch < (w+1)*4
        (L.sat_compute_exclusive(h, x.data_ptr(), out.data_ptr(), 64, 64, 64, 272, 2, ctypes.byref(nv), 0, None), 1),    # full not 0/1
        (L.sat_compute_exclusive(h, x.data_ptr(), out.data_ptr(), 64, 64, 64, 272, 1, ctypes.byref(nv), 1, None), 1),    # pair
        (L.sat_compute_exclusive(h, x.data_ptr(), x.data_ptr(), 16, 16, 64, 256, 1, None, 0, None), 2),                  # overlap
        (L.sat_rect_sums(h, S.data_ptr(), 64, 64, 255, rects.data_ptr(), 4, qo.data_ptr(), 0, None), 1),                  # sat pitch
        (L.sat_rect_sums(h, S.data_ptr(), 64, 64, 256, rects.data_ptr(), -1, qo.data_ptr(), 0, None), 1),                 # n < 0
        (L.sat_rect_sums(h, S.data_ptr(), 64, 64, 256, rects.data_ptr() + 4, 4, qo.data_ptr(), 0, None), 1),              # misaligned rects
        (L.sat_box_filter(h, S.data_ptr(), out.data_ptr(), 64, 64, 256, 272, -1, 2, 0, None), 1),                         # radius
        (L.sat_box_filter(h, S.data_ptr(), S.data_ptr(), 64, 64, 256, 256, 1, 1, 0, None), 2),                            # overlap
        (L.sat_box_filter(h, S.data_ptr(), out.data_ptr(), 64, 64, 256, 272, 1, 1, 2, None), 1),                          # pair
    ]
    for i, (got, want) in enumerate(cases):
        assert got == want, f"case {i}: status {got}, want {want}"
    torch.cuda.synchronize()
    assert bool((out == 5).all()) and bool((qo == 5).all())
    p.close()
