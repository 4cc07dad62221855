"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bars (BASELINE.json north_star): 8u->32s bit-exact; 32f max relative error
<= 1e-4; 64f max relative error <= 1e-12 (64f inputs on a 24-bit dyadic grid
must be bit-exact, reading R6).  Inputs are seeded satgen images.
"""
import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu

TOL = {np.uint8: 0.0, np.float32: 1e-4, np.float64: 1e-12}
KIND = {np.uint8: satgen.KIND_U8, np.float32: satgen.KIND_F32, np.float64: satgen.KIND_F64}


def _torch():
    import torch
    return torch


def _sat():
    import paper_conf_cluster_chenwttm18_b200 as sat
    return sat


def tdtype(np_dtype):
    torch = _torch()
    return {np.uint8: torch.uint8, np.float32: torch.float32, np.float64: torch.float64}[np_dtype]


def check(got: np.ndarray, ref: np.ndarray, np_dtype, what=""):
    tol = TOL[np_dtype]
    if tol == 0.0:
        if not np.array_equal(got, ref):
            bad = np.argwhere(got != ref)
            i, j = bad[0]
            raise AssertionError(f"{what}: {len(bad)} mismatches, first at {(i, j)}: "
                                 f"got {got[i, j]} ref {ref[i, j]}")
        return
    g = got.astype(np.float64)
    nz = ref != 0
    assert np.all(g[~nz] == 0), f"{what}: nonzero where the oracle is 0"
    rel = np.abs(g[nz] - ref[nz]) / np.abs(ref[nz])
    worst = float(rel.max()) if rel.size else 0.0
    assert worst <= tol, f"{what}: max rel err {worst:.3e} > {tol:.0e}"


def gen(np_dtype, H, W, seed, img=0, mode=satgen.MODE_UNIFORM, value=0.0):
    torch = _torch()
    x = torch.empty((H, W), dtype=tdtype(np_dtype), device="cuda")
    satgen.fill_device(x, seed=seed, img0=img, mode=mode, value=value)
    return x


SHAPES = [(1, 1), (1, 300), (300, 1), (31, 33), (32, 256), (33, 257), (64, 255), (512, 512),
          (999, 1001), (1080, 1920), (4097, 4099)]


@pytest.mark.parametrize("np_dtype", [np.uint8, np.float32, np.float64])
@pytest.mark.parametrize("shape", SHAPES)
def test_parity_shapes(np_dtype, shape):
    torch = _torch()
    sat = _sat()
    H, W = shape
    x = gen(np_dtype, H, W, seed=1001 + H + W)
    y = sat.sat(x)
    torch.cuda.synchronize()
    check(y.cpu().numpy(), oracle.sat(x.cpu().numpy()), np_dtype, f"{np_dtype.__name__} {shape}")


@pytest.mark.parametrize("np_dtype", [np.uint8, np.float32, np.float64])
def test_padded_pitches_and_sentinels(np_dtype):
    """Byte pitches larger than a row; the output padding must stay untouched."""
    torch = _torch()
    sat = _sat()
    H, W = 777, 1000
    xin = torch.empty((H, W + 48), dtype=tdtype(np_dtype), device="cuda")
    satgen.fill_device(xin, seed=5)
    x = xin[:, :W]
    out_dt = sat.out_dtype(sat.pair_of_dtype(x.dtype))
    big = torch.full((H, W + 40), -7, dtype=out_dt, device="cuda")
    out = big[:, :W]
    sat.sat(x, out=out)
    torch.cuda.synchronize()
    check(out.cpu().numpy(), oracle.sat(x.cpu().numpy()), np_dtype, "padded")
    assert torch.all(big[:, W:] == -7)


@pytest.mark.parametrize("np_dtype", [np.uint8, np.float32, np.float64])
def test_misaligned_base_uses_generic_path(np_dtype):
    torch = _torch()
    sat = _sat()
    H, W = 300, 701
    xin = torch.empty((H, W + 3), dtype=tdtype(np_dtype), device="cuda")
    satgen.fill_device(xin, seed=6)
    x = xin[:, 1:W + 1]  # base not 16-byte aligned, pitch (W+3)*es not a multiple of 16
    out_dt = sat.out_dtype(sat.pair_of_dtype(x.dtype))
    outbig = torch.zeros((H, W + 1), dtype=out_dt, device="cuda")
    out = outbig[:, 1:]
    sat.sat(x, out=out)
    torch.cuda.synchronize()
    check(out.cpu().numpy(), oracle.sat(x.cpu().numpy()), np_dtype, "misaligned")
    assert torch.all(outbig[:, 0] == 0)


@pytest.mark.parametrize("np_dtype", [np.uint8, np.float32, np.float64])
def test_batched_with_gaps(np_dtype):
    torch = _torch()
    sat = _sat()
    N, H, W = 5, 211, 517
    xin = torch.empty((N, H + 3, W + 16), dtype=tdtype(np_dtype), device="cuda")
    satgen.fill_device(xin, seed=77)
    x = xin[:, :H, :W]
    out_dt = sat.out_dtype(sat.pair_of_dtype(x.dtype))
    obig = torch.full((N, H + 2, W + 8), 3, dtype=out_dt, device="cuda")
    out = obig[:, :H, :W]
    sat.sat(x, out=out)
    torch.cuda.synchronize()
    xn = x.cpu().numpy()
    on = out.cpu().numpy()
    for n in range(N):
        check(on[n], oracle.sat(np.ascontiguousarray(xn[n])), np_dtype, f"batch img {n}")
    assert torch.all(obig[:, H:, :] == 3) and torch.all(obig[:, :, W:] == 3)


@pytest.mark.parametrize("np_dtype", [np.float32, np.float64])
def test_in_place(np_dtype):
    torch = _torch()
    sat = _sat()
    x = gen(np_dtype, 1000, 1500, seed=8)
    ref = oracle.sat(x.cpu().numpy())
    sat.sat(x, out=x)
    torch.cuda.synchronize()
    check(x.cpu().numpy(), ref, np_dtype, "in place")


def test_all_255_wraps_bit_exact():
    """Reading R2 at a size whose sums exceed 2^31 (255 * 4096 * 4096 > 2^31)."""
    torch = _torch()
    sat = _sat()
    H = W = 4096
    x = gen(np.uint8, H, W, seed=0, mode=satgen.MODE_CONST, value=255)
    y = sat.sat(x).cpu().numpy()
    i = np.arange(H, dtype=np.int64)[:, None]
    j = np.arange(W, dtype=np.int64)[None, :]
    ref = ((255 * (i + 1) * (j + 1)) & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
    np.testing.assert_array_equal(y, ref)


def test_all_ones_closed_form_float():
    torch = _torch()
    sat = _sat()
    H, W = 2049, 3001
    for dt in (np.float32, np.float64):
        x = gen(dt, H, W, seed=0, mode=satgen.MODE_CONST, value=1.0)
        y = sat.sat(x).cpu().numpy().astype(np.float64)
        i = np.arange(H, dtype=np.float64)[:, None]
        j = np.arange(W, dtype=np.float64)[None, :]
        np.testing.assert_array_equal(y, (i + 1) * (j + 1))  # all < 2^24: exact in fp32


def test_dyadic_64f_bit_exact():
    torch = _torch()
    sat = _sat()
    x = gen(np.float64, 1024, 1536, seed=9, mode=satgen.MODE_DYADIC24)
    y = sat.sat(x).cpu().numpy()
    np.testing.assert_array_equal(y, oracle.sat(x.cpu().numpy()))


def test_8u_repeat_determinism():
    torch = _torch()
    sat = _sat()
    x = gen(np.uint8, 2048, 3000, seed=10)
    first = sat.sat(x).clone()
    for _ in range(50):
        assert torch.equal(sat.sat(x), first)


def test_rectangle_queries_on_gpu_result():
    """four-corner box sums from the GPU table equal direct sums."""
    torch = _torch()
    sat = _sat()
    x = gen(np.uint8, 1500, 1700, seed=12)
    S = sat.sat(x).cpu().numpy().astype(np.int64)
    A = x.cpu().numpy().astype(np.int64)
    Sp = np.zeros((S.shape[0] + 1, S.shape[1] + 1), dtype=np.int64)
    Sp[1:, 1:] = S
    rng = np.random.default_rng(3)
    for _ in range(300):
        y0, y1 = sorted(rng.integers(0, A.shape[0], size=2))
        x0, x1 = sorted(rng.integers(0, A.shape[1], size=2))
        assert Sp[y1 + 1, x1 + 1] - Sp[y0, x1 + 1] - Sp[y1 + 1, x0] + Sp[y0, x0] == \
            A[y0:y1 + 1, x0:x1 + 1].sum()


@pytest.mark.parametrize("np_dtype", [np.uint8, np.float32, np.float64])
def test_band_with_carry_in(np_dtype):
    torch = _torch()
    sat = _sat()
    H, W, r0 = 900, 1300, 333
    x = gen(np_dtype, H, W, seed=13)
    ref = oracle.sat(x.cpu().numpy())
    out_dt = sat.out_dtype(sat.pair_of_dtype(x.dtype))
    carry = torch.from_numpy(np.ascontiguousarray(ref[r0 - 1])).to(device="cuda", dtype=out_dt)
    y = sat.sat_band(x[r0:], carry_in=carry)
    torch.cuda.synchronize()
    check(y.cpu().numpy(), ref[r0:], np_dtype, "band")


@pytest.mark.parametrize("np_dtype", [np.uint8, np.float32, np.float64])
def test_host_streamed_path(np_dtype):
    torch = _torch()
    sat = _sat()
    H, W = 6000, 4000  # several streamed bands for every pair
    xh = torch.empty((H, W), dtype=tdtype(np_dtype)).pin_memory()
    satgen.fill_host(xh.numpy(), seed=14)
    y = sat.sat_host(xh)
    check(y.numpy(), oracle.sat(xh.numpy()), np_dtype, "host path")


@pytest.mark.parametrize("np_dtype", [np.uint8, np.float32, np.float64])
@pytest.mark.parametrize("P", [2, 3, 8])
def test_dist_virtual_ranks(np_dtype, P):
    """The row-banded multi-GPU algebra on one GPU: per-band column totals,
    a local 'all-gather', the carry row per rank, the band SAT with carry-in."""
    torch = _torch()
    sat = _sat()
    H, W = 1001, 1999
    x = gen(np_dtype, H, W, seed=15)
    ref = oracle.sat(x.cpu().numpy())
    pair = sat.pair_of_dtype(x.dtype)
    spans = [sat.band_partition(H, P, r) for r in range(P)]
    gathered = torch.stack([sat.dist_colsum(x[a:b]) for a, b in spans])
    for r, (a, b) in enumerate(spans):
        carry = sat.dist_carry(gathered, r, pair)
        y = sat.sat_band(x[a:b], carry_in=carry if r > 0 else None)
        torch.cuda.synchronize()
        check(y.cpu().numpy(), ref[a:b], np_dtype, f"rank {r}/{P}")


def test_invalid_arguments_launch_nothing():
    torch = _torch()
    sat = _sat()
    L = sat.lib()
    x = gen(np.uint8, 64, 64, seed=1)
    out = torch.full((64, 64), 5, dtype=torch.int32, device="cuda")
    p = sat.Plan(sat.PAIR_8U_32S, 64, 64, 1)
    h = p.handle
    s = None
    cases = [
        (L.sat_compute(h, x.data_ptr(), out.data_ptr(), 64, 64, 63, 256, 0, s), 1),  # in pitch < w
        (L.sat_compute(h, x.data_ptr(), out.data_ptr(), 64, 64, 64, 255, 0, s), 1),  # out pitch
        (L.sat_compute(h, x.data_ptr(), out.data_ptr(), 65, 64, 64, 256, 0, s), 1),  # > plan h
        (L.sat_compute(h, x.data_ptr(), out.data_ptr(), 64, 64, 64, 256, 1, s), 1),  # pair
        (L.sat_compute(h, None, out.data_ptr(), 64, 64, 64, 256, 0, s), 1),          # NULL
        (L.sat_compute(h, x.data_ptr(), out.data_ptr(), -1, 64, 64, 256, 0, s), 1),  # negative
        (L.sat_compute(h, x.data_ptr(), x.data_ptr(), 16, 16, 64, 256, 0, s), 2),    # overlap
        (L.sat_compute(h, x.data_ptr(), out.data_ptr(), 0, 64, 64, 256, 0, s), 0),   # empty
    ]
    for got, want in cases:
        assert got == want
    torch.cuda.synchronize()
    assert torch.all(out == 5)
    p.close()


# ---------------------------------------------------------------------------
# Full BASELINE.json sizes, in the bench's launch configuration: EVERY element
# against the oracle (compared in row blocks to bound host temporaries), except
# 65536^2 (34 GB), which is checked on a whole chunk column of every row plus
# 128 full rows on both sides of band / cluster / wave edges.

def check_blocks(y, ref: np.ndarray, np_dtype, what, block=2048):
    """Element-by-element check of a CUDA tensor against the oracle array."""
    H = ref.shape[0]
    for r0 in range(0, H, block):
        r1 = min(H, r0 + block)
        check(y[r0:r1].cpu().numpy(), ref[r0:r1], np_dtype, f"{what} rows {r0}:{r1}")


FULL = [
    ("8u 16384^2", np.uint8, 16384, 16384),
    ("32f 16384^2", np.float32, 16384, 16384),
    ("8u 8192^2", np.uint8, 8192, 8192),
    ("32f 8192^2", np.float32, 8192, 8192),
    ("64f 16384^2", np.float64, 16384, 16384),
    ("64f 4096x65536", np.float64, 4096, 65536),
    ("64f 65536x4096", np.float64, 65536, 4096),
    ("8u 4096x65536", np.uint8, 4096, 65536),
    ("32f 65536x4096", np.float32, 65536, 4096),
]


@pytest.mark.parametrize("name,np_dtype,H,W", FULL, ids=[f[0] for f in FULL])
def test_full_size_every_element(name, np_dtype, H, W):
    torch = _torch()
    sat = _sat()
    seed = 1001
    x = gen(np_dtype, H, W, seed=seed)
    y = sat.sat(x)
    torch.cuda.synchronize()
    ref = oracle.sat(x.cpu().numpy())
    del x
    check_blocks(y, ref, np_dtype, name)


def test_full_size_65536sq_32f():
    """BASELINE.json config 4 on one GPU (34 GB of in+out): the first chunk
    column (x < 128) of EVERY row -- the SAT of the image's first 128 columns,
    computed by the oracle on that sub-image -- plus 128 full rows straddling
    the edges of 1024-row blocks (band, cluster and look-back boundaries) and
    the first / last rows."""
    torch = _torch()
    sat = _sat()
    H = W = 65536
    x = gen(np.float32, H, W, seed=1004)
    y = sat.sat(x)
    torch.cuda.synchronize()
    del x
    torch.cuda.empty_cache()
    sub = satgen.generate(satgen.KIND_F32, H, 128, seed=1004)
    check_blocks(y[:, :128], oracle.sat(sub), np.float32, "32f 65536^2 columns 0:128", block=8192)
    rows = sorted({0, 1, H - 1} | {r for k in range(1, 64) for r in (1024 * k - 1, 1024 * k)})
    got = y[rows].cpu().numpy()
    del y
    torch.cuda.empty_cache()
    assert len(rows) >= 64
    check(got, oracle.sat_gen_rows(1, H, W, rows, seed=1004), np.float32, "32f 65536^2 rows")


def test_full_size_batch_1024_frames():
    """BASELINE.json config 3: 1024 frames of 1920x1080, 8u->32s, every
    element of every frame bit-exact."""
    torch = _torch()
    sat = _sat()
    N, H, W = 1024, 1080, 1920
    x = torch.empty((N, H, W), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=1002)
    y = sat.sat(x)
    torch.cuda.synchronize()
    for n0 in range(0, N, 64):  # 64 frames at a time
        xs = x[n0:n0 + 64].cpu().numpy()
        ys = y[n0:n0 + 64].cpu().numpy()
        ref = oracle.sat_batched(xs)
        if not np.array_equal(ys, ref):
            bad = np.argwhere(ys != ref)[0]
            raise AssertionError(f"frame {n0 + bad[0]} row {bad[1]} col {bad[2]} differs")


# ---------------------------------------------------------------------------
# Launch-configuration variants: cluster sizes (bands per thread-block
# cluster) and the generic (non-TMA) load path, selected per launch.

@pytest.mark.parametrize("cluster", ["5", "4", "8"])
@pytest.mark.parametrize("np_dtype", [np.uint8, np.float32, np.float64])
@pytest.mark.parametrize("shape", [(1, 1), (33, 257), (999, 1001), (1080, 1920), (4099, 4097)])
def test_parity_cluster_sizes(monkeypatch, cluster, np_dtype, shape):
    torch = _torch()
    sat = _sat()
    monkeypatch.setenv("SAT_CLUSTER", cluster)
    H, W = shape
    x = gen(np_dtype, H, W, seed=2001 + H)
    y = sat.sat(x)
    torch.cuda.synchronize()
    check(y.cpu().numpy(), oracle.sat(x.cpu().numpy()), np_dtype, f"CL={cluster} {shape}")


@pytest.mark.parametrize("cluster", ["5", "4", "8"])
def test_batched_partial_clusters(monkeypatch, cluster):
    """34 bands per 1080-row frame: clusters straddle frames (segmented scan)."""
    torch = _torch()
    sat = _sat()
    monkeypatch.setenv("SAT_CLUSTER", cluster)
    N, H, W = 7, 1080, 700
    x = torch.empty((N, H, W), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=31)
    y = sat.sat(x).cpu().numpy()
    xn = x.cpu().numpy()
    for n in range(N):
        check(y[n], oracle.sat(xn[n]), np.uint8, f"CL={cluster} frame {n}")


@pytest.mark.parametrize("np_dtype", [np.uint8, np.float32, np.float64])
def test_generic_load_path_forced(monkeypatch, np_dtype):
    torch = _torch()
    sat = _sat()
    monkeypatch.setenv("SAT_FORCE_GENERIC", "1")
    x = gen(np_dtype, 777, 1333, seed=41)
    y = sat.sat(x)
    torch.cuda.synchronize()
    check(y.cpu().numpy(), oracle.sat(x.cpu().numpy()), np_dtype, "generic")


@pytest.mark.parametrize("short", ["0", "1"])
@pytest.mark.parametrize("np_dtype", [np.uint8, np.float32, np.float64])
@pytest.mark.parametrize("shape", [(1, 1), (15, 300), (17, 257), (999, 1001), (2048, 4100)])
def test_parity_short_bands(monkeypatch, short, np_dtype, shape):
    """16-row-band kernels (chosen automatically for short, wide images)
    forced on and off for every shape."""
    torch = _torch()
    sat = _sat()
    monkeypatch.setenv("SAT_SHORT", short)
    H, W = shape
    x = gen(np_dtype, H, W, seed=2101 + H)
    y = sat.sat(x)
    torch.cuda.synchronize()
    check(y.cpu().numpy(), oracle.sat(x.cpu().numpy()), np_dtype, f"short={short} {shape}")


def test_short_bands_batched_and_carry(monkeypatch):
    """Short-band kernels with batches straddled by clusters and with a band carry-in."""
    torch = _torch()
    sat = _sat()
    monkeypatch.setenv("SAT_SHORT", "1")
    x = torch.empty((9, 37, 1920), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=2201)
    y = sat.sat(x)
    torch.cuda.synchronize()
    xs = x.cpu().numpy()
    for i in range(9):
        check(y[i].cpu().numpy(), oracle.sat(xs[i]), np.uint8, f"frame {i}")
    full = gen(np.float64, 200, 700, seed=2202)
    top = sat.sat(full[:77])
    band = sat.sat_band(full[77:], carry_in=top[-1].contiguous())
    torch.cuda.synchronize()
    check(band.cpu().numpy(), oracle.sat(full.cpu().numpy())[77:], np.float64, "band carry")
