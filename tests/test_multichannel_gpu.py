"""Multi-channel SAT consumers on the GPU, parity
with the oracle:

* SAT_8U_SQ -- one read of a uint8 image produces the SAT S and the SAT of
  squares Q (Viola-Jones variance normalisation, PAPER.md:18-24 [2]) in the
  same single pass, both exact mod 2^32 (bit-exact vs oracle.sat_sq);
* SAT_8U_HIST4 -- the integral histogram ([34], [38]), four bins per
  single-pass launch, bit-exact vs oracle.integral_histogram;
* window queries on both (four corners): sums, variances, bin counts.
"""
import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu

SHAPES = [(1, 1), (1, 300), (300, 1), (31, 33), (32, 128), (33, 129), (64, 65), (999, 1001),
          (1080, 1920), (4097, 4099)]


def _t():
    import torch
    return torch


def _sat():
    import paper_conf_cluster_chenwttm18_b200 as sat
    return sat


def _img(H, W, seed, N=None):
    torch = _t()
    x = torch.empty((N, H, W) if N else (H, W), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=seed)
    return x


@pytest.mark.parametrize("shape", SHAPES)
def test_sat_sq_parity(shape):
    torch, sat = _t(), _sat()
    H, W = shape
    x = _img(H, W, seed=H * 7 + W)
    y = sat.sat_sq(x)
    torch.cuda.synchronize()
    assert y.shape == (H, W, 2)
    ref = oracle.sat_sq(x.cpu().numpy())
    assert np.array_equal(y.cpu().numpy(), ref)


def test_sat_sq_wraps_and_batch():
    """All-255 at 2000^2: Q reaches 2.6e11 (wraps mod 2^32 ~ 60 times) --
    bit-exact; and a batch of 9 frames whose clusters straddle frames."""
    torch, sat = _t(), _sat()
    x = torch.full((2000, 2000), 255, dtype=torch.uint8, device="cuda")
    y = sat.sat_sq(x)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy(), oracle.sat_sq(x.cpu().numpy()))
    xb = _img(1080, 700, seed=5, N=9)
    yb = sat.sat_sq(xb)
    torch.cuda.synchronize()
    assert np.array_equal(yb.cpu().numpy(), oracle.sat_sq(xb.cpu().numpy()))


@pytest.mark.parametrize("cluster", ["5", "4", "8"])
def test_sat_sq_cluster_sizes_and_generic_path(monkeypatch, cluster):
    torch, sat = _t(), _sat()
    monkeypatch.setenv("SAT_CLUSTER", cluster)
    x = _img(2100, 777, seed=3)
    assert np.array_equal(sat.sat_sq(x).cpu().numpy(), oracle.sat_sq(x.cpu().numpy()))
    monkeypatch.setenv("SAT_FORCE_GENERIC", "1")
    xs = x[:, 1:700]  # unaligned input rows: the plain-load path
    assert np.array_equal(sat.sat_sq(xs).cpu().numpy(), oracle.sat_sq(xs.cpu().numpy()))


def test_sat_sq_full_size_16384sq():
    """Every element at 16384^2 (both channels wrap) in the bench's launch configuration."""
    torch, sat = _t(), _sat()
    x = _img(16384, 16384, seed=1001)
    y = sat.sat_sq(x)
    torch.cuda.synchronize()
    xs = x.cpu().numpy()
    del x
    ref = oracle.sat_sq(xs)
    for r0 in range(0, 16384, 2048):
        assert np.array_equal(y[r0:r0 + 2048].cpu().numpy(), ref[r0:r0 + 2048]), f"rows {r0}"


def test_window_variance_from_sat_sq():
    """Viola-Jones use: window sums of A and A^2 by four corners on the GPU,
    exact, and the variances they give equal numpy's."""
    torch, sat = _t(), _sat()
    H, W = 1000, 1300
    x = _img(H, W, seed=17)
    SQ = sat.sat_sq(x)
    rng = np.random.default_rng(3)
    y0 = rng.integers(0, H - 24, 500)
    x0 = rng.integers(0, W - 24, 500)
    rects = np.stack([y0, x0, y0 + 24, x0 + 24], axis=1).astype(np.int32)
    got = sat.rect_sums(SQ, torch.from_numpy(rects).cuda()).cpu().numpy().astype(np.int64)
    A = x.cpu().numpy().astype(np.int64)
    for (a, b, c, d), (s, q) in zip(rects, got):
        win = A[a:c, b:d]
        assert s == win.sum() and q == (win * win).sum()
        assert abs((q / 576 - (s / 576) ** 2) - win.astype(np.float64).var()) < 1e-6


@pytest.mark.parametrize("shape", [(1, 1), (33, 65), (999, 1001), (1080, 1920)])
@pytest.mark.parametrize("bins", [4, 16, 7])
def test_integral_histogram_parity(shape, bins):
    torch, sat = _t(), _sat()
    H, W = shape
    x = _img(H, W, seed=bins + H)
    y = sat.integral_histogram(x, bins=bins)
    torch.cuda.synchronize()
    ref = oracle.integral_histogram(x.cpu().numpy(), np.arange(256) * bins // 256, bins)
    got = y.cpu().numpy()  # [groups, H, W, 4] -> bin-major
    got = np.moveaxis(got, 3, 1).reshape(-1, H, W)[:bins]
    assert np.array_equal(got, ref)


def test_integral_histogram_arbitrary_table_and_queries():
    """A random byte-to-bin table (values mapped past the last bin are not
    counted); window histograms by four corners equal direct counts."""
    torch, sat = _t(), _sat()
    H, W = 700, 900
    x = _img(H, W, seed=23)
    rng = np.random.default_rng(9)
    table = rng.integers(0, 12, 256)
    table[rng.integers(0, 256, 20)] = 40  # outside the 12 bins
    y = sat.integral_histogram(x, bins=12, bin_of=table)
    torch.cuda.synchronize()
    ref = oracle.integral_histogram(x.cpu().numpy(), table, 12)
    got = np.moveaxis(y.cpu().numpy(), 3, 1).reshape(-1, H, W)[:12]
    assert np.array_equal(got, ref)
    rects = np.array([[0, 0, H, W], [10, 20, 300, 400], [650, 800, 700, 900]], dtype=np.int32)
    A = x.cpu().numpy()
    for g in range(3):
        cnt = sat.rect_sums(y[g], torch.from_numpy(rects).cuda()).cpu().numpy()
        for (a, b, c, d), row in zip(rects, cnt):
            for k in range(4):
                assert row[k] == int(np.sum(table[A[a:c, b:d]] == 4 * g + k))


def test_multichannel_unsupported_entry_points():
    """The multi-channel pairs refuse the carry-in / exclusive / chained /
    row-banded entry points instead of computing something else."""
    torch, sat = _t(), _sat()
    L = sat.lib()
    p = sat.Plan(sat.PAIR_8U_SQ, 64, 64, 1)
    x = torch.zeros((64, 64), dtype=torch.uint8, device="cuda")
    o = torch.zeros((64, 64, 2), dtype=torch.int32, device="cuda")
    c = torch.zeros((64, 2), dtype=torch.int32, device="cuda")
    assert L.sat_compute_band(p.handle, x.data_ptr(), o.data_ptr(), 64, 64, 64, 512, c.data_ptr(),
                              sat.PAIR_8U_SQ, None) == 2
    assert L.sat_compute_exclusive(p.handle, x.data_ptr(), o.data_ptr(), 63, 63, 64, 512, 1, None,
                                   sat.PAIR_8U_SQ, None) == 2
    h = sat.Plan(sat.PAIR_8U_HIST4, 64, 64, 1)
    o4 = torch.zeros((64, 64, 4), dtype=torch.int32, device="cuda")
    assert L.sat_compute(h.handle, x.data_ptr(), o4.data_ptr(), 64, 64, 64, 1024,
                         sat.PAIR_8U_HIST4, None) == 1  # bins needed
    torch.cuda.synchronize()
    p.close()
    h.close()


# ---------------------------------------------------------------------------
# Seeded randomised cases: shapes around the tile edges (TW = 128 / 64,
# TH = 32), batches, pitched rows (input offset breaking 16-byte alignment ->
# the generic load path), random bin tables; sentinel-padded outputs must stay
# untouched.

@pytest.mark.parametrize("case", range(24))
def test_multichannel_fuzz(case):
    torch, sat = _t(), _sat()
    rng = np.random.default_rng(7000 + case)
    hist = case % 2 == 1
    edges = [64, 32] if hist else [128, 32]
    dim = lambda: int(max(1, rng.choice(edges) * rng.integers(1, 5) + rng.integers(-1, 2))) \
        if rng.random() < 0.5 else int(rng.integers(1, 900))
    H, W = dim(), dim()
    N = int(rng.integers(2, 5)) if (not hist and rng.random() < 0.3) else 1
    off = int(rng.integers(1, 16)) if rng.random() < 0.25 else 0
    pitch = W + off + int(rng.integers(0, 32))
    base = torch.empty((N, H, pitch), dtype=torch.uint8, device="cuda")
    satgen.fill_device(base, seed=case)
    x = base[:, :, off:off + W] if N > 1 else base[0, :, off:off + W]
    if hist:
        table = rng.integers(0, 9, 256)
        y = sat.integral_histogram(x, bins=9, bin_of=table)
        torch.cuda.synchronize()
        ref = oracle.integral_histogram(x.cpu().numpy(), table, 9)
        got = np.moveaxis(y.cpu().numpy(), 3, 1).reshape(-1, H, W)[:9]
        assert np.array_equal(got, ref), f"hist case {case} {H}x{W}"
    else:
        K = 2
        opitch = W + int(rng.integers(0, 8))
        obuf = torch.full((N, H, opitch, K), -5, dtype=torch.int32, device="cuda")
        out = obuf[:, :, :W, :] if N > 1 else obuf[0, :, :W, :]
        sat.sat_sq(x, out=out)
        torch.cuda.synchronize()
        ref = oracle.sat_sq(x.cpu().numpy())
        assert np.array_equal(out.cpu().numpy(), ref), f"sq case {case} {N}x{H}x{W} off {off}"
        assert torch.all(obuf[:, :, W:, :] == -5), "padding written"
