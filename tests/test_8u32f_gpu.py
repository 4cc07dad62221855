"""GPU parity of the 8u->32f pair (NPP's nppiIntegral_8u32f):
uint8 input, fp32 output accumulated in fp32, judged with the 32f bar (max
relative error 1e-4) against the EXACT sums (oracle.sat_8u32f)."""
import ctypes

import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu
TOL = 1e-4


def _t():
    import torch
    return torch


def _sat():
    import paper_conf_cluster_chenwttm18_b200 as sat
    return sat


def _rel(got, ref):
    got = got.astype(np.float64)
    nz = ref != 0
    assert np.all(got[~nz] == 0)
    return float(np.max(np.abs(got[nz] - ref[nz]) / ref[nz])) if nz.any() else 0.0


def _img(H, W, seed, n=None):
    torch = _t()
    x = torch.empty((n, H, W) if n else (H, W), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=seed)
    return x


SHAPES = [(1, 1), (1, 300), (300, 1), (33, 129), (32, 128), (512, 512), (999, 1001), (1080, 1920),
          (4097, 4099)]


@pytest.mark.parametrize("shape", SHAPES)
def test_8u32f_parity(shape):
    torch, sat = _t(), _sat()
    x = _img(*shape, seed=301)
    y = sat.sat(x, out_dtype=torch.float32)
    torch.cuda.synchronize()
    assert y.dtype == torch.float32
    assert _rel(y.cpu().numpy(), oracle.sat_8u32f(x.cpu().numpy())) <= TOL


@pytest.mark.parametrize("env", [{}, {"SAT_CLUSTER": "5"}, {"SAT_CLUSTER": "8"}, {"SAT_SHORT": "1"},
                                 {"SAT_FORCE_GENERIC": "1"}])
def test_8u32f_launch_variants(monkeypatch, env):
    torch, sat = _t(), _sat()
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    x = _img(777, 2050, seed=302)
    y = sat.sat(x, out_dtype=torch.float32)
    torch.cuda.synchronize()
    assert _rel(y.cpu().numpy(), oracle.sat_8u32f(x.cpu().numpy())) <= TOL


def test_8u32f_batched_pitched_and_in_band():
    torch, sat = _t(), _sat()
    x = _img(100, 300, seed=303, n=5)
    y = sat.sat(x, out_dtype=torch.float32)
    big = torch.zeros((120, 333), dtype=torch.uint8, device="cuda")
    big[7:107, 5:305] = x[0]
    o = torch.empty((100, 320), dtype=torch.float32, device="cuda")[:, :300]
    sat.sat(big[7:107, 5:305], out=o)
    torch.cuda.synchronize()
    xs = x.cpu().numpy()
    for i in range(5):
        assert _rel(y[i].cpu().numpy(), oracle.sat_8u32f(xs[i])) <= TOL
    assert _rel(o.cpu().numpy(), oracle.sat_8u32f(xs[0])) <= TOL


def test_8u32f_full_size_sampled_rows_past_2_32():
    """16384^2: the exact sums reach 3.4e10 (8u->32s wraps there, 8u->32f
    rounds); sampled rows against exact int64 sums."""
    torch, sat = _t(), _sat()
    H = W = 16384
    x = _img(H, W, seed=1001)
    y = sat.sat(x, out_dtype=torch.float32)
    torch.cuda.synchronize()
    for r in (0, 31, 32, 8191, H - 1):
        exact = x[:r + 1].to(torch.int64).sum(0).cumsum(0).cpu().numpy().astype(np.float64)
        assert _rel(y[r].cpu().numpy(), exact) <= TOL, f"row {r}"


def test_8u32f_exclusive_matches_npp():
    """Exclusive (H+1) x (W+1) 8u->32f against nppiIntegral_8u32f_C1R (both
    fp32: compared with the 32f bar, relative to the exact sums)."""
    torch, sat = _t(), _sat()
    try:
        npp = ctypes.CDLL("libnppist.so.12")
    except OSError:
        pytest.skip("NPP not available")

    class Size(ctypes.Structure):
        _fields_ = [("width", ctypes.c_int), ("height", ctypes.c_int)]

    f = npp.nppiIntegral_8u32f_C1R
    f.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p, ctypes.c_int, Size, ctypes.c_float]
    H, W = 1999, 3001
    x = _img(H, W, seed=304)
    npp_out = torch.empty((H + 1, W + 1), dtype=torch.float32, device="cuda")
    torch.cuda.synchronize()
    assert f(x.data_ptr(), W, npp_out.data_ptr(), (W + 1) * 4, Size(W, H), 0.0) == 0
    ours = sat.sat_exclusive(x, full=True, out_dtype=torch.float32)
    torch.cuda.synchronize()
    ref = oracle.sat_exclusive(x.cpu().numpy().astype(np.float64), full=True)
    assert _rel(ours.cpu().numpy(), ref) <= TOL
    assert _rel(npp_out.cpu().numpy(), ref) <= TOL


def test_8u32f_dist_virtual_ranks_and_chain():
    torch, sat = _t(), _sat()
    H, W = 1001, 1999
    x = _img(H, W, seed=305)
    ref = oracle.sat_8u32f(x.cpu().numpy())
    P = 3
    spans = [sat.band_partition(H, P, r) for r in range(P)]
    gathered = torch.stack([sat.dist_colsum(x[a:b], pair=3) for a, b in spans])
    for r, (a, b) in enumerate(spans):
        carry = sat.dist_carry(gathered, r, 3)
        y = sat.sat_band(x[a:b], carry_in=carry if r > 0 else None, out_dtype=torch.float32)
        torch.cuda.synchronize()
        assert _rel(y.cpu().numpy(), ref[a:b]) <= TOL, f"colsum rank {r}"
    links = [sat.new_chain_buffer(3, W) for _ in range(P)]
    out = torch.empty((H, W), dtype=torch.float32, device="cuda")
    for r, (a, b) in enumerate(spans):
        sat.sat_band_chained(x[a:b], links[r], links[r - 1] if r > 0 else None,
                             links[r + 1] if r < P - 1 else None, 1, out=out[a:b])
    torch.cuda.synchronize()
    assert _rel(out.cpu().numpy(), ref) <= TOL


def test_8u32f_box_filter_on_float_sat():
    torch, sat = _t(), _sat()
    x = _img(300, 517, seed=306)
    S = sat.sat(x, out_dtype=torch.float32)
    B = sat.box_filter(S, 3, 5)
    torch.cuda.synchronize()
    ref = oracle.box_filter(x.cpu().numpy(), 3, 5).view(np.uint32).astype(np.float64)
    err = np.max(np.abs(B.cpu().numpy().astype(np.float64) - ref))
    assert err <= 4 * TOL * float(S.max())


def test_8u32f_host_streamed_path():
    torch, sat = _t(), _sat()
    xh = torch.empty((1500, 2100), dtype=torch.uint8).pin_memory()
    xd = _img(1500, 2100, seed=307)
    xh.copy_(xd.cpu())
    oh = torch.empty((1500, 2100), dtype=torch.float32).pin_memory()
    y = sat.sat_host(xh, out=oh)
    assert _rel(y.numpy(), oracle.sat_8u32f(xh.numpy())) <= TOL
