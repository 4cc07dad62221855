"""Chained row bands (sat_compute_band_chained): each
band's kernel publishes its bottom row per chunk into the next band's link,
whose top clusters wait for it; the lower band acknowledges each chunk so the
upper band may reuse the slot two epochs later.  On one GPU the "ranks" run in
order on one stream, or concurrently on separate streams (the same device code
that peers run on separate GPUs); results against the oracle, bars as
everywhere."""
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


def _links(sat, pair, W, P):
    return [sat.new_chain_buffer(pair, W) for _ in range(P)]


def _band(sat, x, out, links, r, P, ep, **kw):
    return sat.sat_band_chained(x, links[r], links[r - 1] if r > 0 else None,
                                links[r + 1] if r < P - 1 else None, ep, out=out, **kw)


def _run_chain(d, H, W, P, epochs=(1,), short=None, monkeypatch=None):
    torch, sat = _t(), _sat()
    if short is not None:
        monkeypatch.setenv("SAT_SHORT", short)
    pair = sat.pair_of_dtype(_tdt(d))
    links = _links(sat, pair, W, P)
    out = torch.empty((H, W), dtype=sat.out_dtype(pair), device="cuda")
    for ep in epochs:
        x = torch.empty((H, W), dtype=_tdt(d), device="cuda")
        satgen.fill_device(x, seed=77 + P + ep)  # new data every epoch: slots must not mix
        out.fill_(0)
        for r in range(P):
            r0, r1 = sat.band_partition(H, P, r)
            _band(sat, x[r0:r1], out[r0:r1], links, r, P, ep)
        torch.cuda.synchronize()
        _check(out.cpu().numpy(), oracle.sat(x.cpu().numpy()), d, f"P={P} {H}x{W} epoch {ep}")


@pytest.mark.parametrize("d", [np.uint8, np.float32, np.float64])
@pytest.mark.parametrize("P", [2, 3, 8])
def test_chained_bands(d, P):
    _run_chain(d, 1001, 1537, P)


def test_chained_bands_epoch_reuse_and_tiny_bands():
    """Links reused with increasing epochs (both slots, acknowledgements);
    bands of one row and of one chunk; W a multiple of the tile width."""
    _run_chain(np.uint8, 37, 512, 5, epochs=(1, 2, 3, 4, 5, 6))
    _run_chain(np.float32, 700, 900, 3, epochs=(1, 2, 3))
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
    links = _links(sat, 0, W, P)
    for r in range(P):
        r0, r1 = sat.band_partition(H, P, r)
        _band(sat, x[r0:r1], out[r0:r1], links, r, P, 1)
    torch.cuda.synchronize()
    rows = [0, 4095, 4096, 8191, 8192, 12287, 12288, H - 1]
    ref = oracle.sat_gen_rows(0, H, W, rows, seed=1001)
    assert np.array_equal(out[rows].cpu().numpy(), ref)


def test_chained_invalid_arguments():
    torch, sat = _t(), _sat()
    L = sat.lib()
    x = torch.zeros((64, 64), dtype=torch.uint8, device="cuda")
    o = torch.zeros((64, 64), dtype=torch.int32, device="cuda")
    b = sat.new_chain_buffer(0, 64)
    c = sat.new_chain_buffer(0, 64)
    p = sat.Plan(0, 64, 64, 1)
    args = (p.handle, x.data_ptr(), o.data_ptr(), 64, 64, 64, 256)
    assert L.sat_compute_band_chained(*args, b.data_ptr(), None, c.data_ptr(), 0, 0, None) == 1  # epoch 0
    assert L.sat_compute_band_chained(p.handle, x.data_ptr(), o.data_ptr(), 0, 64, 64, 256,
                                      b.data_ptr(), None, c.data_ptr(), 1, 0, None) == 1  # empty band
    assert L.sat_compute_band_chained(*args, b.data_ptr(), None, c.data_ptr() + 16, 1, 0, None) == 1  # alignment
    assert L.sat_compute_band_chained(*args, None, None, c.data_ptr(), 1, 0, None) == 1  # no own link
    # 257 columns = 2 chunks of 256: 256 bytes of ack words + 2 slots of 2 x 256 x 8 bytes
    assert sat.chain_bytes(0, 257) == 256 + 2 * (2 * 256 * 4 * 2)
    p.close()


def test_chained_missing_upstream_band_times_out():
    """A band whose band above never runs: its bounded wait runs out, the launch
    finishes (no hung GPU) and sat_plan_status reports SAT_ERR_TIMEOUT; the plan
    works normally afterwards."""
    torch, sat = _t(), _sat()
    H, W = 256, 1000
    x = torch.ones((H, W), dtype=torch.uint8, device="cuda")
    links = _links(sat, 0, W, 2)
    p = sat.Plan(0, H, W, 1)
    p.set_timeout(20_000_000)  # 20 ms
    sat.sat_band_chained(x, links[1], links[0], None, 1, plan=p)  # band 1 of 2; band 0 never runs
    with pytest.raises(sat.SatError) as ei:
        p.status()
    assert ei.value.status == 6  # SAT_ERR_TIMEOUT
    p.status()  # cleared
    y = sat.sat(x, plan=p)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy(), oracle.sat(x.cpu().numpy()))
    p.close()


def test_chained_flow_control_concurrent_epochs(monkeypatch):
    """Two bands on two streams, three epochs each, the lower stream enqueued
    late: the upper band's epoch-3 kernel must wait (on the device) for the
    lower band to acknowledge epoch 1 of every chunk before reusing the slot.
    Every epoch has its own input; every output checked."""
    torch, sat = _t(), _sat()
    monkeypatch.setenv("SAT_MAX_CLUSTERS", "16")  # both bands co-resident
    monkeypatch.setenv("SAT_SHORT", "0")
    H, W, P, E = 2 * 1024, 6000, 2, 3
    pair = 0
    links = _links(sat, pair, W, P)
    xs = []
    for e in range(E):
        x = torch.empty((H, W), dtype=torch.uint8, device="cuda")
        satgen.fill_device(x, seed=500 + e)
        xs.append(x)
    outs = [torch.zeros((H, W), dtype=torch.int32, device="cuda") for _ in range(E)]
    plans = [sat.Plan(pair, H, W, 1) for _ in range(P)]
    streams = [torch.cuda.Stream() for _ in range(P)]
    torch.cuda.synchronize()
    for r in range(P):  # upper band's three epochs first, then the lower band's
        r0, r1 = sat.band_partition(H, P, r)
        for e in range(E):
            with torch.cuda.stream(streams[r]):
                _band(sat, xs[e][r0:r1], outs[e][r0:r1], links, r, P, e + 1, plan=plans[r],
                      stream=streams[r])
    torch.cuda.synchronize()
    for pl in plans:
        pl.status()
    for e in range(E):
        assert np.array_equal(outs[e].cpu().numpy(), oracle.sat(xs[e].cpu().numpy())), f"epoch {e + 1}"


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
    links = _links(sat, pair, W, P)
    out = torch.empty((H, W), dtype=sat.out_dtype(pair), device="cuda")
    plans = [sat.Plan(pair, H, W, 1) for _ in range(P)]
    streams = [torch.cuda.Stream() for _ in range(P)]
    torch.cuda.synchronize()
    for r in reversed(range(P)):  # lowest band first: it must wait for the others
        r0, r1 = sat.band_partition(H, P, r)
        with torch.cuda.stream(streams[r]):
            _band(sat, x[r0:r1], out[r0:r1], links, r, P, 1, plan=plans[r], stream=streams[r])
    torch.cuda.synchronize()
    _check(out.cpu().numpy(), oracle.sat(x.cpu().numpy()), d, "concurrent chain")
