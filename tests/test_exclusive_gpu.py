"""GPU parity of the exclusive SAT (sat_compute_exclusive; Eq. 2,
NPP's (H+1) x (W+1) layout with nVal) against the CPU oracle, element by
element; bars as for the inclusive path (8u bit-exact, 32f 1e-4, 64f 1e-12).
Shapes span several tiles with ragged tails, W a multiple of the tile width
(the last column lies past the last chunk's vectors), 16-byte aligned and
unaligned output rows (vector vs scalar shifted stores), and empty inputs."""
import ctypes

import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu

TOL = {np.uint8: 0.0, np.float32: 1e-4, np.float64: 1e-12}
NVAL = {np.uint8: 7, np.float32: 0.5, np.float64: 0.25}


def _t():
    import torch
    return torch


def _sat():
    import paper_conf_cluster_chenwttm18_b200 as sat
    return sat


def _tdt(d):
    torch = _t()
    return {np.uint8: torch.uint8, np.float32: torch.float32, np.float64: torch.float64}[d]


def check(got, ref, d, what):
    if TOL[d] == 0.0:
        assert np.array_equal(got, ref), f"{what}: {np.count_nonzero(got != ref)} mismatches, first " \
            f"{np.argwhere(got != ref)[:1].tolist()}"
    else:
        g = got.astype(np.float64)
        nz = ref != 0
        assert np.all(g[~nz] == ref[~nz]), what
        rel = np.max(np.abs(g[nz] - ref[nz]) / np.abs(ref[nz])) if nz.any() else 0.0
        assert rel <= TOL[d], f"{what}: rel err {rel}"


SHAPES = [(1, 1), (1, 300), (300, 1), (37, 513), (64, 256), (33, 128), (70, 64), (129, 1031), (517, 640)]


@pytest.mark.parametrize("d", [np.uint8, np.float32, np.float64])
@pytest.mark.parametrize("shape", SHAPES)
@pytest.mark.parametrize("full", [True, False])
def test_exclusive_parity(d, shape, full):
    torch, sat = _t(), _sat()
    H, W = shape
    x = torch.empty((H, W), dtype=_tdt(d), device="cuda")
    satgen.fill_device(x, seed=31)
    nv = NVAL[d]
    got = sat.sat_exclusive(x, full=full, nval=nv)
    torch.cuda.synchronize()
    ref = oracle.sat_exclusive(x.cpu().numpy(), full=full, nval=nv)
    check(got.cpu().numpy(), ref, d, f"{d.__name__} {shape} full={full}")


@pytest.mark.parametrize("d", [np.uint8, np.float32, np.float64])
def test_exclusive_unaligned_pitched_output(d):
    """Output rows not 16-B aligned (scalar shifted stores) inside a larger
    buffer: nothing outside the (H+1) x (W+1) window is touched."""
    torch, sat = _t(), _sat()
    H, W = 97, 700
    x = torch.empty((H, W), dtype=_tdt(d), device="cuda")
    satgen.fill_device(x, seed=32)
    out_dt = sat.out_dtype(sat.pair_of_dtype(x.dtype))
    big = torch.full((H + 3, W + 9), 99, dtype=out_dt, device="cuda")
    win = big[1:H + 2, 1:W + 2]
    sat.sat_exclusive(x, full=True, nval=NVAL[d], out=win)
    torch.cuda.synchronize()
    ref = oracle.sat_exclusive(x.cpu().numpy(), full=True, nval=NVAL[d])
    b = big.cpu().numpy()
    check(b[1:H + 2, 1:W + 2], ref, d, "window")
    mask = np.ones(b.shape, dtype=bool)
    mask[1:H + 2, 1:W + 2] = False
    assert np.all(b[mask] == 99), "wrote outside the output window"


@pytest.mark.parametrize("shape", [(0, 5), (5, 0), (0, 0)])
def test_exclusive_empty(shape):
    torch, sat = _t(), _sat()
    x = torch.empty(shape, dtype=torch.uint8, device="cuda")
    J = sat.sat_exclusive(x, full=True, nval=3)
    torch.cuda.synchronize()
    assert tuple(J.shape) == (shape[0] + 1, shape[1] + 1)
    assert bool((J == 3).all())
    assert tuple(sat.sat_exclusive(x, full=False).shape) == shape


def test_exclusive_full_size_sampled_rows():
    """16384^2 8u (BASELINE configs[1] at its largest size; the sums wrap past
    2^31): sampled output rows against the oracle's streamed rows, plus the
    nVal border."""
    torch, sat = _t(), _sat()
    H = W = 16384
    x = torch.empty((H, W), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=1001)
    nv = 12345
    J = sat.sat_exclusive(x, full=True, nval=nv)
    torch.cuda.synchronize()
    rows = [0, 1, 31, 32, 4095, 8191, 12288, H - 1]
    ref = oracle.sat_gen_rows(0, H, W, rows, seed=1001)
    got = J[[r + 1 for r in rows]].cpu().numpy()
    assert np.all(got[:, 0] == nv)
    want = (ref.view(np.uint32) + np.uint32(nv)).view(np.int32)
    assert np.array_equal(got[:, 1:], want)
    assert bool((J[0] == nv).all())


def test_exclusive_matches_npp():
    """Independent library check: nppiIntegral_8u32s_C1R (CUDA NPP, the
    paper's comparison library) on the same input and nVal."""
    torch, sat = _t(), _sat()
    try:
        npp = ctypes.CDLL("libnppist.so.12")
    except OSError:
        pytest.skip("NPP not available")

    class Size(ctypes.Structure):
        _fields_ = [("width", ctypes.c_int), ("height", ctypes.c_int)]

    f = npp.nppiIntegral_8u32s_C1R
    f.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p, ctypes.c_int, Size, ctypes.c_int32]
    H, W = 1999, 3001
    x = torch.empty((H, W), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=33)
    ref = torch.empty((H + 1, W + 1), dtype=torch.int32, device="cuda")
    torch.cuda.synchronize()
    assert f(x.data_ptr(), W, ref.data_ptr(), (W + 1) * 4, Size(W, H), -17) == 0
    got = sat.sat_exclusive(x, full=True, nval=-17)
    torch.cuda.synchronize()
    assert torch.equal(got, ref)
