"""Chained row bands (sat_compute_band_chained): each
band's kernel publishes its bottom row per chunk into the next band's chain
buffer, whose top clusters wait for it.  On one GPU the "ranks" run in order
on one stream (the same device code that peers run concurrently on separate
GPUs); results against the oracle, bars as everywhere."""
import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu
TOL = {np.uint8: 0.0, np.float32: 1e-4, np.float64: 1e-12}


def _t():
    import torch
    return torch


def _sat():
    import paper_conf_cluster_chenwttm18_b200 as sat
    return sat


def _tdt(d):
    torch = _t()
    return {np.uint8: torch.uint8, np.float32: torch.float32, np.float64: torch.float64}[d]


def _check(got, ref, d, what):
    if TOL[d] == 0.0:
        assert np.array_equal(got, ref), f"{what}: {np.count_nonzero(got != ref)} mismatches"
    else:
        rel = np.max(np.abs(got.astype(np.float64) - ref) / np.maximum(np.abs(ref), 1e-300))
        assert rel <= TOL[d], f"{what}: rel err {rel}"


def _run_chain(d, H, W, P, epochs=(1,), short=None, monkeypatch=None):
    torch, sat = _t(), _sat()
    if short is not None:
        monkeypatch.setenv("SAT_SHORT", short)
    x = torch.empty((H, W), dtype=_tdt(d), device="cuda")
    satgen.fill_device(x, seed=77 + P)
    pair = sat.pair_of_dtype(x.dtype)
    bufs = [sat.new_chain_buffer(pair, W) for _ in range(P - 1)]
    out = torch.empty((H, W), dtype=sat.out_dtype(pair), device="cuda")
    for ep in epochs:
        out.fill_(0)
        for r in range(P):
            r0, r1 = sat.band_partition(H, P, r)
            sat.sat_band_chained(x[r0:r1], bufs[r - 1] if r > 0 else None,
                                 bufs[r] if r < P - 1 else None, ep, out=out[r0:r1])
        torch.cuda.synchronize()
        _check(out.cpu().numpy(), oracle.sat(x.cpu().numpy()), d, f"P={P} {H}x{W} epoch {ep}")


@pytest.mark.parametrize("d", [np.uint8, np.float32, np.float64])
@pytest.mark.parametrize("P", [2, 3, 8])
def test_chained_bands(d, P):
    _run_chain(d, 1001, 1537, P)


def test_chained_bands_epoch_reuse_and_tiny_bands():
    """Buffers reused with increasing epochs; bands of one row and of one
    chunk; W a multiple of the tile width."""
    _run_chain(np.uint8, 37, 512, 5, epochs=(1, 2, 3))
    _run_chain(np.float64, 9, 64, 9)
    _run_chain(np.float32, 300, 1, 4)


@pytest.mark.parametrize("short", ["0", "1"])
def test_chained_bands_both_band_heights(monkeypatch, short):
    _run_chain(np.uint8, 700, 3000, 3, short=short, monkeypatch=monkeypatch)


def test_chained_full_size_8u_16384sq_sampled():
    """16384^2 8u in 4 chained bands (the sums wrap): sampled rows vs the
    streaming oracle, including the rows on both sides of each band edge."""
    torch, sat = _t(), _sat()
    H = W = 16384
    P = 4
    x = torch.empty((H, W), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=1001)
    out = torch.empty((H, W), dtype=torch.int32, device="cuda")
    bufs = [sat.new_chain_buffer(0, W) for _ in range(P - 1)]
    for r in range(P):
        r0, r1 = sat.band_partition(H, P, r)
        sat.sat_band_chained(x[r0:r1], bufs[r - 1] if r > 0 else None,
                             bufs[r] if r < P - 1 else None, 1, out=out[r0:r1])
    torch.cuda.synchronize()
    rows = [0, 4095, 4096, 8191, 8192, 12287, 12288, H - 1]
    ref = oracle.sat_gen_rows(0, H, W, rows, seed=1001)
    assert np.array_equal(out[rows].cpu().numpy(), ref)


def test_chained_invalid_arguments():
    import ctypes
    torch, sat = _t(), _sat()
    L = sat.lib()
    x = torch.zeros((64, 64), dtype=torch.uint8, device="cuda")
    o = torch.zeros((64, 64), dtype=torch.int32, device="cuda")
    b = sat.new_chain_buffer(0, 64)
    p = sat.Plan(0, 64, 64, 1)
    assert L.sat_compute_band_chained(p.handle, x.data_ptr(), o.data_ptr(), 64, 64, 64, 256,
                                      None, b.data_ptr(), 0, 0, None) == 1  # epoch 0
    assert L.sat_compute_band_chained(p.handle, x.data_ptr(), o.data_ptr(), 0, 64, 64, 256,
                                      None, b.data_ptr(), 1, 0, None) == 1  # empty band
    assert L.sat_compute_band_chained(p.handle, x.data_ptr(), o.data_ptr(), 64, 64, 64, 256,
                                      None, b.data_ptr() + 8, 1, 0, None) == 1  # alignment
    assert sat.chain_bytes(0, 257) == 2 * 256 * 4 * 2
    p.close()


@pytest.mark.parametrize("d", [np.uint8, np.float32])
def test_chained_bands_concurrent_streams(monkeypatch, d):
    """The bands run CONCURRENTLY on separate streams (as peers do on separate
    GPUs): each kernel's persistent grid is capped (SAT_MAX_CLUSTERS) so that
    all bands are co-resident whatever order the hardware starts them in, and
    the lower bands' top clusters really wait inside the kernel for chunks
    still being produced above them."""
    torch, sat = _t(), _sat()
    P = 3
    monkeypatch.setenv("SAT_MAX_CLUSTERS", "16")  # 3 x 16 clusters x 4 CTAs <= 2 CTAs/SM x 148
    monkeypatch.setenv("SAT_SHORT", "0")
    H, W = 3 * 2048, 8192
    x = torch.empty((H, W), dtype=_tdt(d), device="cuda")
    satgen.fill_device(x, seed=91)
    pair = sat.pair_of_dtype(x.dtype)
    bufs = [sat.new_chain_buffer(pair, W) for _ in range(P - 1)]
    out = torch.empty((H, W), dtype=sat.out_dtype(pair), device="cuda")
    plans = [sat.Plan(pair, H, W, 1) for _ in range(P)]
    streams = [torch.cuda.Stream() for _ in range(P)]
    torch.cuda.synchronize()
    for r in reversed(range(P)):  # lowest band first: it must wait for the others
        r0, r1 = sat.band_partition(H, P, r)
        with torch.cuda.stream(streams[r]):
            sat.sat_band_chained(x[r0:r1], bufs[r - 1] if r > 0 else None,
                                 bufs[r] if r < P - 1 else None, 1, out=out[r0:r1],
                                 plan=plans[r], stream=streams[r])
    torch.cuda.synchronize()
    _check(out.cpu().numpy(), oracle.sat(x.cpu().numpy()), d, "concurrent chain")
